#!/bin/bash
# Sparse q pass probe: ncu of k_sp_runs without / with the L2 prefetch, then
# segments-per-block variants (NB_LIB) under the prefetch.
mkdir -p gpurun_out
for pf in 0 600; do
  NB_SPR_PF=$pf timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_sp_runs" -s 3 -c 1 \
     -o gpurun_out/spr_pf$pf python tools/prof_driver.py 512 sparse > gpurun_out/spr_ncu_pf$pf.log 2>&1
  ncu -i gpurun_out/spr_pf$pf.ncu-rep --page raw --csv > gpurun_out/spr_pf$pf.raw.csv 2>/dev/null
  ncu -i gpurun_out/spr_pf$pf.ncu-rep --page source --csv > gpurun_out/spr_pf$pf.src.csv 2>/dev/null
  rm -f gpurun_out/spr_pf$pf.ncu-rep
done
L=paper_conf_ipps_meneghinmjm22_b200
for v in "libnb.so 600" "libnb_SPR_NSB1_SPR_MINB8.so 1200" "libnb_SPR_NSB2_SPR_MINB5.so 600" "libnb_SPR_NSB3_SPR_MINB4.so 400" "libnb_SPR_NSB4_SPR_MINB3.so 300" "libnb_SPR_NSB4_SPR_MINB4.so 300"; do
  set -- $v
  echo -n "$1 pf=$2 "; NB_LIB=$L/$1 NB_SPR_PF=$2 timeout 120 python tools/sparse_time.py 512 30
done
