# ncu (full set) of the AA even and odd steps at 512^3
timeout 900 ncu --set full --clock-control none -k regex:k_lbm_aa -s 4 -c 2 -o gpurun_out/aa_r2 python tools/aa_prof.py > gpurun_out/aa_ncu.log 2>&1
ncu -i gpurun_out/aa_r2.ncu-rep --page raw --csv > gpurun_out/aa_r2.raw.csv 2>>gpurun_out/aa_ncu.log
rm -f gpurun_out/aa_r2.ncu-rep
python tools/aa_prof.py >> gpurun_out/aa_ncu.log 2>&1
