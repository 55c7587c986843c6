#!/bin/bash
# A/B of the sparse q-pass L2 prefetch distance (NB_SPR_PF blocks ahead) on
# the C4 sphere: ms per CG iteration, q-pass split and the x digest.
for rep in 1 2; do
  for pf in ${PFS:-0 300 600 900 1500 3000}; do
    echo -n "pf=$pf "; NB_SPR_PF=$pf timeout 120 python tools/sparse_time.py 512 30
  done
done
