python tools/power_probe.py lbm 8 2>&1 | head -1 > gpurun_out/lbm256.log
python tools/aa_prof.py >> gpurun_out/lbm256.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lbm_aa.py tests/test_gpu_lbm_sparse.py tests/test_gpu_fullsize.py tests/test_gpu_peer.py -x -q 2>&1 | tail -1 >> gpurun_out/lbm256.log
