for i in 1 2; do
for v in 0 1; do
  if [ $v = 1 ]; then export NB_CG_ZC_POW2=1; else unset NB_CG_ZC_POW2; fi
  echo "pow2=$v"
  python tools/cg_slab_time.py 512 512 64 200
  python tools/cg_slab_time.py 512 512 512 100
  AB_PARTS=8 python tools/cg_ab.py 512 100 2>/dev/null | tail -1
done
done
