for a in "140 23 1" "67 9 2" "200 5 2" "130 7 3"; do python tools/cg_dump.py $a 2>/dev/null | tail -1; done > gpurun_out/c1fin.log
for e in "" "NB_C1_FIN_EACH=1" ""; do env $e python tools/c1_time.py 64 2>/dev/null | tail -1; done >> gpurun_out/c1fin.log
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -1 >> gpurun_out/c1fin.log
