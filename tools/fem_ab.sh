# FEM A/B: the working build (libnb.so) vs variant builds (default
# libnb_BASE1.so): bitwise digests, then interleaved timings (serial FEM
# schedule, NB_FEM_CONC=0, so the per-kernel split is the kernels' own time).
VARS=${VARS:-paper_conf_ipps_meneghinmjm22_b200/libnb_BASE1.so}
for p in 1 3; do
  python tools/fem_dump.py 61 9 $p
  for v in $VARS; do NB_LIB=$v python tools/fem_dump.py 61 9 $p; done
done
export NB_FEM_CONC=0
for i in 1 2 3; do
  python tools/fem_time.py 384 20
  for v in $VARS; do NB_LIB=$v python tools/fem_time.py 384 20; done
done
