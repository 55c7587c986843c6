"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): every op family on 3 virtual partitions."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402
import synth  # noqa: E402

dims = (40, 19, 18)
with nb.Grid(dims, nparts=3, devices=[0, 0, 0]) as g:
    x, y, b = nb.Field(g), nb.Field(g), nb.Field(g)
    x.fill_uniform(seed=1)
    y.fill_const(0.0)
    nb.nb_axpby(0.5, x, 2.0, y)
    x.halo_update()
    nb.nb_laplace7(x, y)
    nb.nb_dot(x, y)
    for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_TWO_WAY):
        nb.nb_map_stencil_reduce(x, y, 0.125, 3, occ)
        b.fill_uniform(seed=2)
        x.fill_const(0.0)
        nb.nb_cg_solve(x, b, max_iter=5, occ=occ)
    f0, f1 = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(f0, 1.0, (0, 0, 0))
    nb.nb_lbm_step(f0, f1, 1.1, 3)
    u, v = nb.Field(g, card=3), nb.Field(g, card=3)
    u.fill_uniform(seed=3)
    u.halo_update()
    nb.nb_fem27_apply(u, v)
    nb.nb_fem27_rhs(v)
    u.fill_const(0.0)
    nb.nb_cg_solve(u, v, max_iter=3, op=nb.OP_FEM27)
    for f in (x, y, b, f0, f1, u, v):
        f.close()
m = synth.sphere_mask(20, 0.45)
with nb.Grid((20, 20, 20), nparts=2, devices=[0, 0], active=m) as g:
    x, b = nb.Field(g), nb.Field(g)
    b.fill_uniform(seed=4)
    x.fill_const(0.0)
    nb.nb_cg_solve(x, b, max_iter=4)
    x.halo_update()
    nb.nb_laplace7(x, b)
    nb.nb_dot(x, b)
    x.download()
    x.close(), b.close()
# round-1 additions: TMA FEM (surface kernels), halo-stream mode, skeleton,
# AA-pattern and sparse LBM, D2Q9, borrowed storage, dot_dev
dims = (34, 21, 40)
with nb.Grid(dims, nparts=2, devices=[0, 0]) as g:
    u, v = nb.Field(g, card=3), nb.Field(g, card=3)
    u.fill_uniform(seed=5)
    u.halo_update()
    nb.nb_fem27_apply(u, v)
    g.set_halo_mode(nb.HALO_STREAM)
    x, y = nb.Field(g), nb.Field(g)
    x.fill_uniform(seed=6)
    y.fill_const(0.0)
    nb.nb_map_stencil_reduce(x, y, 0.125, 2, nb.OCC_TWO_WAY)
    g.set_halo_mode(nb.HALO_FUSED)
    with nb.Skeleton(g, nb.OCC_TWO_WAY) as sk:
        for k in range(2):
            sk.axpy(0.125, y, x)
            sk.laplace7(x, y)
            sk.dot(x, y, k)
        sk.run()
        sk.result(1)
    f = nb.Field(g, "f32", 19)
    nb.nb_lbm_init(f, 1.0, (0.01, 0, 0))
    nb.nb_lbm_step_aa(f, 1.1, 4)
    nb.nb_lbm_step_aa(f, 1.1, 2, bc=nb.LBM_PERIODIC)
    for fld in (u, v, x, y, f):
        fld.close()
m = synth.sphere_mask(22)
with nb.Grid((22, 22, 22), nparts=2, devices=[0, 0], active=m) as g:
    a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(a, 1.0, (0.01, 0, 0))
    a, b = nb.nb_lbm_step(a, b, 1.1, 3)
    a.close(), b.close()
with nb.Grid((96, 40, 1)) as g:
    a, b = nb.Field(g, "f32", 9), nb.Field(g, "f32", 9)
    nb.nb_d2q9_init(a, 1.0, 0.05, 0.0)
    nb.nb_d2q9_step(a, b, 1.6, 0.05, (24, 20, 5), 3)
    a.close(), b.close()
print("sanitize driver done")
