L=paper_conf_ipps_meneghinmjm22_b200/libnb_CG_NTX2.so
for a in "140 23 1" "140 23 3" "67 9 2" "200 5 2"; do python tools/cg_dump.py $a 2>/dev/null; NB_LIB=$L python tools/cg_dump.py $a 2>/dev/null; done > gpurun_out/dump4.log
python tools/power_probe.py cg 60 > gpurun_out/pw_ntx1.log 2>&1
NB_LIB=$L python tools/power_probe.py cg 60 > gpurun_out/pw_ntx2.log 2>&1
python tools/power_probe.py cg 60 > gpurun_out/pw_ntx1b.log 2>&1
NB_LIB=$L python tools/power_probe.py cg 60 > gpurun_out/pw_ntx2b.log 2>&1
NB_LIB=$L python tools/cg_drift.py 6 > gpurun_out/drift_ntx2.log 2>&1
python tools/cg_drift.py 6 > gpurun_out/drift_ntx1.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests2.log 2>&1; tail -2 gpurun_out/gpu_tests2.log
