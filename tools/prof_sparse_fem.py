import os, sys
sys.path.insert(0, os.getcwd())
os.environ["NB_NO_GRAPH"] = "1"
import numpy as np
import paper_conf_ipps_meneghinmjm22_b200 as nb
N = 384
m = np.ones((N, N, N), np.uint8)
g = nb.Grid((N, N, N), active=m)
b, x = nb.Field(g, card=3), nb.Field(g, card=3)
nb.nb_fem27_rhs(b, 1.0)
x.fill_const(0.0)
cg = nb.CG(x, b, op=nb.OP_FEM27)
cg.iterate(3)
cg.finish()
g.profile(True)
cg2 = nb.CG(x, b, op=nb.OP_FEM27)
cg2.iterate(3)
for k in ("k_sp_fem_q", "k_sp_cg_map", "k_sp_cg_r", "k_finalize", "k_halo_copy"):
    print(k, g.profile_read(k))
