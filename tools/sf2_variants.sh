# sparse FEM box2 producer back-off variants: CG iteration (full cube / sphere)
for lib in libnb.so libnb_SF2_SLEEP_NS64.so libnb_SF2_SLEEP_NS1024.so; do
  echo "== $lib"
  NB_LIB=paper_conf_ipps_meneghinmjm22_b200/$lib timeout 300 python tools/sparse_fem_box_ab.py 384 2>&1 | grep -o '"box": {"ms_per_iter": [0-9.]*' | tr '\n' ' '; echo
done
