P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_SPLBM_BX256_D2Q9_BX256.so; do
  NB_LIB=$L python -c "
import bench, json
a = bench.bench_lbm_sparse_run(512, 20, 3, 0)
k = bench.bench_karman(0)
print('$L', a['value'], a['ms_per_step'], [round(r['mlups']) for r in k['rows']])
" 2>&1 | tail -1
done > gpurun_out/splbm.log
NB_LIB=$P/libnb_SPLBM_BX256_D2Q9_BX256.so timeout 600 python -m pytest tests/test_gpu_lbm_sparse.py tests/test_gpu_karman.py -x -q 2>&1 | tail -1 >> gpurun_out/splbm.log
