"""Dump x, r-norm after K CG iterations (for bitwise comparison of build
variants: run once per NB_LIB and compare the printed digests)."""
import hashlib
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n, it, parts = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 1
with nb.Grid((n, n + 3, n - 5), nparts=parts, devices=[0] * parts) as g:
    b, x, y = nb.Field(g), nb.Field(g), nb.Field(g)
    b.fill(nb.FILL_UNIFORM, seed=2, a=-1.0, b=1.0)
    x.fill_const(0.0)
    res = nb.nb_cg_solve(x, b, max_iter=it, rtol=0.0)
    xv = x.download()
    x.fill_int(seed=1)
    y.fill_const(0.0)
    dots = nb.nb_map_stencil_reduce(x, y, 0.125, 10, nb.OCC_TWO_WAY)
    print("cg", n, it, parts, res.rr, hashlib.sha1(xv.tobytes()).hexdigest(),
          "c1", hashlib.sha1(x.download().tobytes() + y.download().tobytes() + dots.tobytes()).hexdigest())
    for f in (b, x, y):
        f.close()
