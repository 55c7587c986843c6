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
# round-2 additions: sparse q pass on the segment-indexed table, sparse FEM
# (tables, K u, load, CG with OCC on the halo stream), field layouts (AoS /
# plane-major LBM, dots, halo updates), Skeleton Listing 3 CG + LBM, OCC on
# sparse CG, CopyBatch with > 32 descriptors
m = synth.sphere_mask(18, 0.47)
with nb.Grid((18, 18, 18), nparts=3, devices=[0, 0, 0], active=m) as g:
    g.set_halo_mode(nb.HALO_STREAM)
    b, x = nb.Field(g, card=3), nb.Field(g, card=3)
    nb.nb_fem27_rhs(b, 1.0)
    x.fill_const(0.0)
    nb.nb_cg_solve(x, b, max_iter=3, op=nb.OP_FEM27, occ=nb.OCC_TWO_WAY)
    x.halo_update()
    nb.nb_fem27_apply(x, b)
    p, q = nb.Field(g), nb.Field(g)
    p.fill_uniform(seed=2)
    q.fill_const(0.0)
    nb.nb_cg_solve(q, p, max_iter=3, occ=nb.OCC_TWO_WAY)
    for f in (b, x, p, q):
        f.close()
dims = (24, 20, 18)
for layout in (nb.SOA_PLANE, nb.AOS):
    with nb.Grid(dims, nparts=3, devices=[0, 0, 0]) as g:
        a, c = nb.Field(g, "f32", 19, layout=layout), nb.Field(g, "f32", 19, layout=layout)
        nb.nb_lbm_init(a, 1.0, (0, 0, 0))
        a, c = nb.nb_lbm_step(a, c, 1.1, 3)
        rho, u = nb.Field(g, "f32", 1), nb.Field(g, "f32", 3, layout=layout)
        nb.nb_lbm_macroscopic(a, rho, u)
        h = synth.uniform(dims, card=3, seed=3)
        v, w = nb.Field(g, card=3, layout=layout), nb.Field(g, card=3, layout=layout)
        v.upload(h)
        w.upload(h)
        v.halo_update()
        nb.nb_axpby(0.5, v, 2.0, w)
        nb.nb_dot(v, w)
        v.download()
        for f in (a, c, rho, u, v, w):
            f.close()
with nb.Grid((30, 26, 24), nparts=2, devices=[0, 0]) as g:
    b, x, r, p, q = (nb.Field(g) for _ in range(5))
    b.fill_uniform(seed=8)
    for f in (x, p, q):
        f.fill_const(0.0)
    nb.nb_axpby(1.0, b, 0.0, r)
    with nb.Skeleton(g, nb.OCC_TWO_WAY) as s0:
        s0.dot(r, r, 0)
        s0.set_scalar(3, 0.0)
        s0.run()
    with nb.Skeleton(g, nb.OCC_TWO_WAY) as sk:
        sk.axpby_s(1.0, -1, r, 1.0, 3, p)
        sk.poisson(p, q)
        sk.dot(p, q, 1)
        sk.scalar(nb.SC_DIV, 0, 1, 2)
        sk.axpby_s(1.0, 2, p, 1.0, -1, x)
        sk.axpby_s(-1.0, 2, q, 1.0, -1, r)
        sk.dot(r, r, 4)
        sk.scalar(nb.SC_DIV, 4, 0, 3)
        sk.scalar(nb.SC_COPY, 4, 0, 0)
        sk.run()
        sk.run()
    a, c = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(a, 1.0, (0, 0, 0))
    with nb.Skeleton(g, nb.OCC_STANDARD) as sk:
        sk.lbm(a, c, 1.0)
        sk.lbm(c, a, 1.0)
        sk.run()
    f19 = nb.Field(g, card=19)
    f19.fill_uniform(seed=1)
    f19.halo_update()  # 38 plane copies in one batch
    for f in (b, x, r, p, q, a, c, f19):
        f.close()
# round-2b additions: the sparse FEM box operator + list nodes (apply, CG
# q pass, set-up), its fused phase A (NB_SPF_FUSED) and the 7-point 2-phase
# box CG (NB_SP_CG_BOX) on a ragged mask spanning several tiles and z-chunks
m = synth.sphere_mask(70, 0.45)[:36, :45, :].copy()
nz, ny, nx = m.shape
with nb.Grid((nx, ny, nz), nparts=2, devices=[0, 0], active=m) as g:
    u, v = nb.Field(g, card=3), nb.Field(g, card=3)
    u.fill_uniform(seed=7)
    u.halo_update()
    nb.nb_fem27_apply(u, v)
    for env in (None, "NB_SPF_FUSED"):
        if env:
            os.environ[env] = "1"
        nb.nb_fem27_rhs(v, 1.0)
        u.fill_const(0.0)
        nb.nb_cg_solve(u, v, max_iter=3, op=nb.OP_FEM27, occ=nb.OCC_TWO_WAY)
        os.environ.pop("NB_SPF_FUSED", None)
    x, b = nb.Field(g), nb.Field(g)
    b.fill_uniform(seed=8)
    x.fill_const(0.0)
    os.environ["NB_SP_CG_BOX"] = "1"
    nb.nb_cg_solve(x, b, max_iter=3, occ=nb.OCC_TWO_WAY)
    os.environ.pop("NB_SP_CG_BOX", None)
    for f in (u, v, x, b):
        f.close()
print("sanitize driver done")
