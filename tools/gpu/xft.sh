for e in "" "NB_FEM_XFACE_LDG=1"; do
  for a in "70 12 1" "70 12 3" "33 7 2"; do env $e python tools/fem_dump.py $a 2>&1 | tail -1; done
  env $e python tools/fem_time.py 384 20 2>&1 | tail -1
done > gpurun_out/xft.log 2>&1
timeout 600 python -m pytest tests/test_gpu_fem.py -x -q 2>&1 | tail -1 >> gpurun_out/xft.log
