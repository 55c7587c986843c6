P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_CG_SLEEP1.so; do
  for a in "140 23 1" "67 9 2" "200 5 2" "130 7 3"; do NB_LIB=$L python tools/cg_dump.py $a 2>&1 | tail -1; done
done > gpurun_out/dump10.log
for L in "" $P/libnb_CG_SLEEP1.so "" $P/libnb_CG_SLEEP1.so; do
  echo "lib=$L"; NB_LIB=$L python tools/power_probe.py cg 60 2>&1 | head -1
  NB_LIB=$L python tools/cg_drift.py 3 2>&1 | tail -1
done > gpurun_out/sleep_probe.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_peer.py tests/test_gpu_skeleton.py -x -q > gpurun_out/sleep_tests.log 2>&1; tail -n 2 gpurun_out/sleep_tests.log
