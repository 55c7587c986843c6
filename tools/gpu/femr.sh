for e in "" "NB_FEM_R_PLANE=1"; do
  for a in "70 12 1" "70 12 3"; do env $e python tools/fem_dump.py $a 2>&1 | tail -1; done
  env $e python tools/fem_time.py 384 20 2>&1 | tail -1
done > gpurun_out/femr.log 2>&1
timeout 600 python -m pytest tests/test_gpu_fem.py tests/test_gpu_peer.py -x -q 2>&1 | tail -1 >> gpurun_out/femr.log
