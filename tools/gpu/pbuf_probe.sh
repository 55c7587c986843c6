set -x
L=paper_conf_ipps_meneghinmjm22_b200/libnb_CGA_PBUF1.so
for lib in "" $L; do
  for a in "140 23 1" "140 23 3" "67 9 2"; do NB_LIB=$lib python tools/cg_dump.py $a; done
done > gpurun_out/dump.log 2>&1
python tools/copy_sustained.py 3 > gpurun_out/copy_sustained.json 2>&1
python tools/power_probe.py cg 60 > gpurun_out/power_cg_v0.log 2>&1
NB_LIB=$L python tools/power_probe.py cg 60 > gpurun_out/power_cg_v1.log 2>&1
python tools/power_probe.py cg 60 > gpurun_out/power_cg_v0b.log 2>&1
cat gpurun_out/dump.log; head -1 gpurun_out/power_cg_v*.log
