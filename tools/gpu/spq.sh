for e in "" "NB_SP_Q_FLAT=1" ""; do env $e python tools/sparse_time.py 512 20 2>/dev/null | tail -1; done > gpurun_out/spq.log
timeout 600 python -m pytest tests/test_gpu_sparse.py tests/test_gpu_fullsize.py -x -q 2>&1 | tail -1 >> gpurun_out/spq.log
