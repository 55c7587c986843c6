# k_sp_fem_box build knobs: the CG iteration's K p pass per variant library
for lib in libnb.so libnb_SFB_MINB4.so libnb_SFB_ZC16.so libnb_SFB_ZC64.so; do
  echo "== $lib"
  NB_LIB=paper_conf_ipps_meneghinmjm22_b200/$lib timeout 300 python tools/sparse_fem_box_ab.py 384 2>&1 | cut -c1-400 | grep -o '"box": {"ms_per_iter": [0-9.]*, "kernel_ms": {"k_sp_fem_q": [0-9.]*'
done
