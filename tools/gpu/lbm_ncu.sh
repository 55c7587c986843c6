timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_lbm_d3q19" -s 1 -c 2 -o gpurun_out/prof_r1_lbm python tools/prof_driver.py 512 lbm > gpurun_out/prof_r1_lbm.log 2>&1
ncu -i gpurun_out/prof_r1_lbm.ncu-rep --page raw --csv > gpurun_out/prof_r1_lbm.raw.csv 2>/dev/null
rm -f gpurun_out/prof_r1_lbm.ncu-rep
