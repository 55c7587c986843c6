#!/bin/bash
# FEM (C5) probe: timing split, then ncu --set full of the K u apply and the
# CG phase A (raw pages + SASS source page of phase A).
mkdir -p gpurun_out
python tools/fem_time.py 384 20 > gpurun_out/fem_time.json 2>&1
cat > /tmp/fem_apply.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
os.environ["NB_NO_GRAPH"] = "1"
import paper_conf_ipps_meneghinmjm22_b200 as nb
g = nb.Grid((384, 384, 384))
u, y = nb.Field(g, card=3), nb.Field(g, card=3)
u.fill_uniform(seed=5); u.halo_update()
for _ in range(3): nb.nb_fem27_apply(u, y, 1.0, 0.3)
g.sync()
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_fem" -c 12 -o gpurun_out/fem_apply python /tmp/fem_apply.py > gpurun_out/fem_apply.log 2>&1
ncu -i gpurun_out/fem_apply.ncu-rep --page raw --csv > gpurun_out/fem_apply.raw.csv 2>/dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_fem_tma" -s 2 -c 1 -o gpurun_out/femA \
    python tools/prof_driver.py 384 fem > gpurun_out/femA.log 2>&1
ncu -i gpurun_out/femA.ncu-rep --page raw --csv > gpurun_out/femA.raw.csv 2>/dev/null
ncu -i gpurun_out/femA.ncu-rep --page source --csv --print-source sass > gpurun_out/femA.sass.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
ls -la gpurun_out/fem*
