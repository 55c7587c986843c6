P=paper_conf_ipps_meneghinmjm22_b200
for L in $P/libnb_LBM_BX256.so $P/libnb_LBM_BX512.so $P/libnb_LBM_BX256.so; do
  echo "lib=$L"; NB_LIB=$L python tools/power_probe.py lbm 8 2>&1 | head -1
done > gpurun_out/lbmbx.log 2>&1
