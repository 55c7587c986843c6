# 2-phase box CG (C4 sphere 512^3) per build variant: ms/iter and kernel split
for lib in libnb.so libnb_SPB_NST6.so libnb_SPB_NST13.so libnb_SPB_MINB4.so; do
  NB_LIB=paper_conf_ipps_meneghinmjm22_b200/$lib timeout 200 python tools/sparse_time.py 512 20 2>&1 | tail -1
done
