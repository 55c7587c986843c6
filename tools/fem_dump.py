"""Digest of x after K FEM CG iterations (bitwise comparison of build
variants: run once per NB_LIB)."""
import hashlib
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n, it, parts = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 1
g = nb.Grid((n + 2, n - 3, n), nparts=parts, devices=[0] * parts)
b, x = nb.Field(g, card=3), nb.Field(g, card=3)
nb.nb_fem27_rhs(b, 1.0)
x.fill_const(0.0)
res = nb.nb_cg_solve(x, b, max_iter=it, rtol=0.0, op=nb.OP_FEM27)
print("fem", n, it, parts, res.rr, hashlib.sha1(x.download().tobytes()).hexdigest())
x.close(), b.close(), g.close()
