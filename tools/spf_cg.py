"""A few sparse FEM CG iterations (box q pass; NB_SPF_FUSED / NB_SPF_GATHER select
the fused phase A / the gather pass) on the full N^3 cube: an ncu target."""
import os, sys
sys.path.insert(0, os.getcwd())
os.environ.setdefault("NB_NO_GRAPH", "1")
import numpy as np
import paper_conf_ipps_meneghinmjm22_b200 as nb
N = int(sys.argv[1]) if len(sys.argv) > 1 else 384
g = nb.Grid((N, N, N), active=np.ones((N, N, N), np.uint8))
b, x = nb.Field(g, card=3), nb.Field(g, card=3)
nb.nb_fem27_rhs(b, 1.0)
x.fill_const(0.0)
cg = nb.CG(x, b, op=nb.OP_FEM27)
cg.iterate(4)
cg.finish()
g.sync()
print("ok")
