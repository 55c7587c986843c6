# AA-pattern A/B over build variants (NB_VARIANT libs): digest + time
P=paper_conf_ipps_meneghinmjm22_b200
LIBS="$P/libnb.so $P/libnb_AA_MINB24.so $P/libnb_AA_MINB28.so $P/libnb_AA_MINB32.so"
for L in $LIBS; do
  NB_LIB=$L python -c "
import sys, hashlib; sys.path.insert(0, '.')
import paper_conf_ipps_meneghinmjm22_b200 as nb
g = nb.Grid((70, 37, 45), nparts=2, devices=[0, 0]); f = nb.Field(g, 'f32', 19)
nb.nb_lbm_init(f, 1.0, (0.0, 0.0, 0.0)); nb.nb_lbm_step_aa(f, 0.79, 6)
print('$L'.split('/')[-1], hashlib.sha1(f.download().tobytes()).hexdigest())"
done
for i in 1 2; do for L in $LIBS; do echo -n "${L##*/} "; NB_LIB=$L python tools/aa_prof.py; done; done
