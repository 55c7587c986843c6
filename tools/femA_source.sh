# Per-instruction SASS execution counts of the FEM CG phase A (k_fem_tma<3,...>)
# at 384^3: ncu SourceCounters, exported as the source page (sass view).
set -u
mkdir -p gpurun_out
timeout 900 ncu --section SourceCounters --section WarpStateStats --section LaunchStats --section Occupancy \
    --clock-control none --import-source on -k regex:"k_fem_tma|k_fem_xface|k_fem_surface" -c 9 -o gpurun_out/femA_src \
    python tools/prof_driver.py 384 fem > gpurun_out/femA_src.log 2>&1
ncu -i gpurun_out/femA_src.ncu-rep --page source --csv --print-source sass > gpurun_out/femA_src.csv 2>>gpurun_out/femA_src.log
ncu -i gpurun_out/femA_src.ncu-rep --page details --csv > gpurun_out/femA_details.csv 2>>gpurun_out/femA_src.log
ls -la gpurun_out/femA_src*
