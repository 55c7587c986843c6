"""One sparse FEM K u (box operator unless NB_SPF_GATHER=1) on the full N^3
cube and on the sphere: the ncu target for k_sp_fem_box."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth
N = int(sys.argv[1]) if len(sys.argv) > 1 else 384
for mask in (np.ones((N, N, N), np.uint8), synth.sphere_mask(N)):
    g = nb.Grid((N, N, N), active=mask)
    u, y = nb.Field(g, card=3), nb.Field(g, card=3)
    u.fill_uniform(seed=5)
    for _ in range(2):
        nb.nb_fem27_apply(u, y)
    g.sync()
    u.close(), y.close(), g.close()
print("ok")
