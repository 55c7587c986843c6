# FEM surface kernels concurrent with the surface-free streaming box
# (NB_FEM_CONC, default on) vs serial (NB_FEM_CONC=0): digests, timings.
for p in 1 3; do
  python tools/fem_dump.py 96 9 $p
  NB_FEM_CONC=0 python tools/fem_dump.py 96 9 $p
done
python tools/fem_dump.py 61 9 1
for i in 1 2 3; do
  python tools/fem_time.py 384 20
  NB_FEM_CONC=0 python tools/fem_time.py 384 20
done
python tools/timeline.py 384 3 fem 1 --out gpurun_out/tl_fem_conc.json > gpurun_out/tl_fem_conc.txt 2>&1
