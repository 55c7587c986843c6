# PDL A/B on the C2 CG chain (programmatic dependent launch on vs NB_NO_PDL=1),
# interleaved within one process by tools/cg_ab.py, 1 and 8 virtual partitions.
for i in 1 2; do
  python tools/cg_ab.py 512 100 NB_NO_PDL=1 | tail -1
  AB_PARTS=8 python tools/cg_ab.py 512 100 NB_NO_PDL=1 | tail -1
  python tools/cg_ab.py 256 200 NB_NO_PDL=1 | tail -1
done
