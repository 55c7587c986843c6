timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_cgA_tma<.bool.1, .bool.0" -s 2 -c 1 -o gpurun_out/cga_src python tools/prof_driver.py 512 cg > gpurun_out/cga_src.log 2>&1
ncu -i gpurun_out/cga_src.ncu-rep --page source --csv --print-source sass > gpurun_out/cga_src_sass.csv 2>/dev/null
ncu -i gpurun_out/cga_src.ncu-rep --page raw --csv > gpurun_out/cga_raw.csv 2>/dev/null
rm -f gpurun_out/cga_src.ncu-rep
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_cgB_tma" -s 2 -c 1 -o gpurun_out/cgb_src python tools/prof_driver.py 512 cg > gpurun_out/cgb_src.log 2>&1
ncu -i gpurun_out/cgb_src.ncu-rep --page source --csv --print-source sass > gpurun_out/cgb_src_sass.csv 2>/dev/null
rm -f gpurun_out/cgb_src.ncu-rep
ls -la gpurun_out/cg*_src*
