L=paper_conf_ipps_meneghinmjm22_b200/libnb_CG_1WAIT1.so
for a in "140 23 1" "140 23 3" "67 9 2"; do NB_LIB=$L python tools/cg_dump.py $a 2>/dev/null; done > gpurun_out/dump2.log
python tools/power_probe.py cg 60 > gpurun_out/pw_v0.log 2>&1
NB_LIB=$L python tools/power_probe.py cg 60 > gpurun_out/pw_1wait.log 2>&1
NB_CG_SMEM_PAD=12000 python tools/power_probe.py cg 60 > gpurun_out/pw_pad12.log 2>&1
NB_CG_SMEM_PAD=24000 python tools/power_probe.py cg 60 > gpurun_out/pw_pad24.log 2>&1
NB_LIB=$L NB_CG_SMEM_PAD=12000 python tools/power_probe.py cg 60 > gpurun_out/pw_1wait_pad12.log 2>&1
python tools/power_probe.py cg 60 > gpurun_out/pw_v0b.log 2>&1
