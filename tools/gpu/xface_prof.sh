timeout 600 ncu --set full --clock-control none --kernel-name-base demangled -k regex:"k_fem_xface<.int.3|k_fem_surface<.int.3" -s 2 -c 2 -o gpurun_out/xf python tools/prof_driver.py 384 fem > gpurun_out/xf.log 2>&1
ncu -i gpurun_out/xf.ncu-rep --page raw --csv > gpurun_out/xf_raw.csv 2>/dev/null
rm -f gpurun_out/xf.ncu-rep
