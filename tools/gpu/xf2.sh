for a in "70 12 1" "70 12 3"; do python tools/fem_dump.py $a 2>&1 | tail -1; done > gpurun_out/xf2.log
python tools/fem_time.py 384 20 2>&1 | tail -1 >> gpurun_out/xf2.log
timeout 600 python -m pytest tests/test_gpu_fem.py -x -q 2>&1 | tail -1 >> gpurun_out/xf2.log
