P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_OLD1.so; do
  for a in "70 12 1" "70 12 3"; do NB_LIB=$L python tools/fem_dump.py $a 2>&1 | tail -1; done
  NB_LIB=$L python tools/fem_time.py 384 20 2>&1 | tail -1
  NB_LIB=$L python tools/fem_time.py 384 20 2>&1 | tail -1
done > gpurun_out/femcv.log 2>&1
