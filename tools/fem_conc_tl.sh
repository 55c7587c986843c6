python tools/timeline.py 384 3 fem 1 --out gpurun_out/tl_fem_conc.json > gpurun_out/tl_fem_conc.txt 2>&1
NB_FEM_CONC=0 python tools/timeline.py 384 3 fem 1 --out gpurun_out/tl_fem_ser.json > gpurun_out/tl_fem_ser.txt 2>&1
