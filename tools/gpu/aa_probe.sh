timeout 600 python -m pytest tests/test_gpu_lbm_aa.py -x -q > gpurun_out/aa_tests.log 2>&1; tail -3 gpurun_out/aa_tests.log
python tools/aa_prof.py > gpurun_out/aa_prof.log 2>&1
NB_AA_NOROW=1 python tools/aa_prof.py >> gpurun_out/aa_prof.log 2>&1
cat gpurun_out/aa_prof.log
