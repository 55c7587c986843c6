#!/bin/bash
# GPU-box profiling pass for one round: launch list of the bench command and
# one ncu --set full capture per hot kernel.  Usage: tools/profile_round.sh r1
set -u
R=${1:-r1}
mkdir -p gpurun_out
# every launch of the default bench workload (cold-cache, serialised: compare shares)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/launches_${R}.csv python bench.py --steps 3 --warmup 3 --no-extras \
    > gpurun_out/launches_${R}.log 2>&1
# full sections of each hot kernel (2-4 launches each)
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"k_cgA_tma|k_cgB_tma|k_finalize|k_map_u" -c 12 -o gpurun_out/prof_${R}_dense \
    python tools/prof_driver.py 512 cg > gpurun_out/prof_${R}_dense.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"k_lbm_d3q19" -s 1 -c 2 -o gpurun_out/prof_${R}_lbm \
    python tools/prof_driver.py 512 lbm > gpurun_out/prof_${R}_lbm.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"^k_sp$|k_sp_runs|k_sp_fem|k_fem_tma|k_fem_faces|k_fem_surface|k_fem_xface|k_fem_map|k_fem_r$" -c 60 -o gpurun_out/prof_${R}_sparse_fem \
    python tools/prof_driver.py 512 sparse,fem,spfem > gpurun_out/prof_${R}_sparse_fem.log 2>&1
# raw pages exported here; the reports themselves stay on the box (gpurun
# copies back at most 64 MiB)
for rep in gpurun_out/prof_${R}_*.ncu-rep; do
    ncu -i "$rep" --page raw --csv > "${rep%.ncu-rep}.raw.csv" 2>/dev/null
    rm -f "$rep"
done
echo profile done
# kernel timelines (CUPTI via torch.profiler): 1 partition and 4 virtual partitions
timeout 300 python tools/timeline.py 512 8 cg 1 --out gpurun_out/timeline_${R}_cg_p1.json > /dev/null 2>&1
timeout 300 python tools/timeline.py 512 8 cg 4 0 --out gpurun_out/timeline_${R}_cg_p4.json > /dev/null 2>&1
timeout 300 python tools/timeline.py 512 8 cg 4 1 --out gpurun_out/timeline_${R}_cg_p4_halostream.json > /dev/null 2>&1
timeout 300 python tools/timeline.py 512 4 lbm 4 0 --out gpurun_out/timeline_${R}_lbm_p4.json > /dev/null 2>&1
timeout 300 python tools/timeline.py 512 4 lbm 4 1 --out gpurun_out/timeline_${R}_lbm_p4_halostream.json > /dev/null 2>&1
echo timelines done
