L=paper_conf_ipps_meneghinmjm22_b200/libnb_ZC64.so
for a in "140 23 1" "140 23 3" "67 9 2"; do python tools/cg_dump.py $a 2>/dev/null; NB_LIB=$L python tools/cg_dump.py $a 2>/dev/null; done > gpurun_out/dump3.log
python tools/power_probe.py cg 60 > gpurun_out/pw_new.log 2>&1
NB_LIB=$L python tools/power_probe.py cg 60 > gpurun_out/pw_zc64.log 2>&1
python tools/power_probe.py cg 60 > gpurun_out/pw_newb.log 2>&1
timeout 600 python bench.py --no-extras > gpurun_out/bench_new.log 2>&1
