# round-end evidence pass: GPU tests, smoke, bench + reference lines, ncu
# launch list and full captures, timelines, sanitizers, power probes
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/final_tests.log 2>&1; echo "rc=$?" >> gpurun_out/final_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/final_bench.log 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/final_ref.log 2>&1
python tools/copy_sustained.py 3 > gpurun_out/copy_sustained.json 2>&1
python tools/power_probe.py cg 80 > gpurun_out/power_cg.log 2>&1
python tools/power_probe.py lbm 80 > gpurun_out/power_lbm.log 2>&1
for t in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $t python tools/sanitize_driver.py (NB_NO_GRAPH=1, every op family incl. TMA CG / FEM, skeleton, AA / sparse LBM, D2Q9)"
  NB_NO_GRAPH=1 timeout 900 compute-sanitizer --tool $t python tools/sanitize_driver.py 2>&1 | grep -E "COMPUTE-SANITIZER|ERROR SUMMARY|done|Error|error" | head -20
done > gpurun_out/r1_sanitizer.txt 2>&1
bash tools/profile_round.sh r1 > gpurun_out/profile_round.log 2>&1
echo final done
