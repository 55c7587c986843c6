P=paper_conf_ipps_meneghinmjm22_b200
for L in "" $P/libnb_SPLBM_BX64_FSURF_BX64.so $P/libnb_SPLBM_BX32_FSURF_BX32.so; do
  NB_LIB=$L python -c "
import bench
a = bench.bench_lbm_sparse_run(512, 20, 3, 0)
print('$L'.split('/')[-1], 'splbm', round(a['value']), round(a['ms_per_step'], 4))
" 2>&1 | tail -1
  NB_LIB=$L python tools/fem_time.py 384 20 2>&1 | tail -1 | cut -c1-250
done > gpurun_out/w2.log
