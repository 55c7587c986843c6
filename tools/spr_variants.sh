# C4 q-pass build knobs (segments per block, blocks per SM) with the L2 prefetch on
for lib in libnb.so libnb_SPR_MINB5.so libnb_SPR_MINB8.so libnb_SPR_NSB3.so libnb_SPR_NSB1.so libnb.so; do
  NB_LIB=paper_conf_ipps_meneghinmjm22_b200/$lib timeout 200 python tools/sparse_time.py 512 20 2>&1 | tail -1 | python3 -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['lib'], round(d['ms_per_iter'],4), {k: round(v,4) for k,v in d['split'].items()}, d['digest'][:10])"
done
