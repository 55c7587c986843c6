P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_CG_NTX1.so $P/libnb_CG_NTY2_CG_NST3.so $P/libnb_CG_NTX4_CG_NST3.so; do
  for a in "140 23 1" "67 9 2" "200 5 2"; do NB_LIB=$L python tools/cg_dump.py $a 2>&1 | tail -1; done
done > gpurun_out/dump5.log
for L in "" $P/libnb_CG_NTX1.so $P/libnb_CG_NTY2_CG_NST3.so $P/libnb_CG_NTX4_CG_NST3.so ""; do
  echo "lib=$L"; NB_LIB=$L python tools/power_probe.py cg 60 2>&1 | head -1
  NB_LIB=$L python tools/cg_drift.py 3 2>&1 | tail -1
done > gpurun_out/tile_probe.log 2>&1
