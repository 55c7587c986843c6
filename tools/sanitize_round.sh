#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over
# tools/sanitize_driver.py (every op family, eager launches).  Usage:
# tools/sanitize_round.sh r2  -> gpurun_out/sanitizer_r2.txt
R=${1:-r2}
OUT=gpurun_out/sanitizer_${R}.txt
: > $OUT
for tool in memcheck racecheck synccheck initcheck; do
    echo "== compute-sanitizer --tool $tool python tools/sanitize_driver.py (NB_NO_GRAPH=1)" >> $OUT
    NB_NO_GRAPH=1 timeout 1500 compute-sanitizer --tool $tool python tools/sanitize_driver.py 2>&1 \
        | grep -E "COMPUTE-SANITIZER|SUMMARY|driver done|Invalid|Race|hazard|Error|error" | head -40 >> $OUT
done
