for L in "" paper_conf_ipps_meneghinmjm22_b200/libnb_SP_MINB5.so paper_conf_ipps_meneghinmjm22_b200/libnb_SP_NSB2_SP_MINB6.so paper_conf_ipps_meneghinmjm22_b200/libnb_SP_NSB1_SP_MINB8.so paper_conf_ipps_meneghinmjm22_b200/libnb_SP_NSB3_SP_MINB6.so paper_conf_ipps_meneghinmjm22_b200/libnb_SP_NSB2_SP_MINB7.so ""; do
  NB_LIB=$L python tools/sparse_time.py 512 20 2>&1 | tail -1
done > gpurun_out/sp_probe2.log 2>&1
