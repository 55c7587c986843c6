P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_FEM_PFLAT1.so "" $P/libnb_FEM_PFLAT1.so; do
  NB_LIB=$L python tools/fem_dump.py 70 12 3 2>&1 | tail -1
  NB_LIB=$L python tools/fem_time.py 384 20 2>&1 | tail -1
done > gpurun_out/pflat.log 2>&1
