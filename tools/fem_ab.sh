# FEM phase-A A/B: the working build (libnb.so) vs variant builds (default
# libnb_BASE1.so); bitwise digests first, then interleaved timings.
VARS=${VARS:-paper_conf_ipps_meneghinmjm22_b200/libnb_BASE1.so}
for p in 1 3; do
  python tools/fem_dump.py 61 9 $p
  for v in $VARS; do NB_LIB=$v python tools/fem_dump.py 61 9 $p; done
done
python tools/fem_dump.py 40 30 2
for v in $VARS; do NB_LIB=$v python tools/fem_dump.py 40 30 2; done
for i in 1 2 3; do
  python tools/fem_time.py 384 20
  for v in $VARS; do NB_LIB=$v python tools/fem_time.py 384 20; done
done
