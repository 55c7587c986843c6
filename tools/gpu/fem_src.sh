timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_fem_tma<.int.3" -s 1 -c 1 -o gpurun_out/fem_src python tools/prof_driver.py 384 fem > gpurun_out/fem_src.log 2>&1
ncu -i gpurun_out/fem_src.ncu-rep --page source --csv --print-source sass > gpurun_out/fem_src_sass.csv 2>/dev/null
ncu -i gpurun_out/fem_src.ncu-rep --page source --csv --print-source cuda > gpurun_out/fem_src_cuda.csv 2>/dev/null
rm -f gpurun_out/fem_src.ncu-rep
ls -la gpurun_out/fem_src*
