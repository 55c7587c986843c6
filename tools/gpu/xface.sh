for a in "70 12 1" "70 12 3"; do python tools/fem_dump.py $a 2>&1 | tail -1; NB_FEM_FACES=node python tools/fem_dump.py $a 2>&1 | tail -1; done > gpurun_out/xface.log
timeout 600 python -m pytest tests/test_gpu_fem.py -x -q >> gpurun_out/xface.log 2>&1
python tools/fem_time.py 384 20 2>&1 | tail -1 >> gpurun_out/xface.log
NB_FEM_FACES=node python tools/fem_time.py 384 20 2>&1 | tail -1 >> gpurun_out/xface.log
