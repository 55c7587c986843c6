P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_LBM_FAST1.so "" $P/libnb_LBM_FAST1.so; do
  echo "lib=$L"; NB_LIB=$L python tools/power_probe.py lbm 12 2>&1 | head -1
done > gpurun_out/lbmfast.log 2>&1
NB_LIB=$P/libnb_LBM_FAST1.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lbm_aa.py tests/test_gpu_lbm_sparse.py tests/test_gpu_fullsize.py -x -q -k "lbm or aa or LBM" 2>&1 | tail -2 >> gpurun_out/lbmfast.log
