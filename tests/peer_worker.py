"""One rank of the multi-process peer-memory transport check (launched by
tests/test_gpu_peer.py under torch.distributed.run, world 2).

Every rank drives its own slabs through libnb's peer transport (CUDA IPC
mappings of the neighbours' halos and of every rank's reduction buffer; the
ranks may share one GPU, which is how the single-GPU test box runs it) and
compares them BITWISE with the same computation done by one process on
virtual partitions of the same partition plan (halos
are bitwise copies and reductions follow the canonical order, so the result
may not depend on how partitions map to processes).  Exits non-zero on the
first mismatch.
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

dist.init_process_group("gloo")
RANK, WORLD = dist.get_rank(), dist.get_world_size()
DEV = int(os.environ.get("LOCAL_RANK", RANK)) % max(nb.nb_device_count(), 1)
torch.cuda.set_device(DEV)
TRANSPORT = os.environ.get("NB_TRANSPORT", "peer")  # "nccl": the NCCL transport (one GPU per rank)
COMM = nb.Comm.from_torch_distributed(DEV, transport=TRANSPORT)
assert COMM.transport == TRANSPORT
checks = 0


def local_planes(g, nparts):
    """Global z planes owned by this rank."""
    zs = []
    for p in range(nparts):
        info = g.partition_info(p)
        if info["local"]:
            zs.extend(range(info["z_begin"], info["z_end"]))
    return zs


def same(name, a, b):
    global checks
    checks += 1
    if not np.array_equal(a, b, equal_nan=True):
        d = np.max(np.abs(np.asarray(a, np.float64) - np.asarray(b, np.float64)))
        raise AssertionError(f"rank {RANK}: {name} differs from the single-process run (max |d| = {d})")


def compare(name, dims, nparts, fn, card_axis=False, active=None):
    def mk(comm):
        if active is not None:
            kw = dict(comm=comm) if comm else dict(devices=[DEV] * nparts)
            g = nb.Grid(dims, nparts=nparts, active=active, **kw)
        else:
            g = nb.Grid(dims, nparts=nparts, comm=comm) if comm else nb.Grid(dims, nparts=nparts,
                                                                             devices=[DEV] * nparts)
        try:
            return fn(g), (local_planes(g, nparts) if comm else None)
        finally:
            g.close()

    (arrays_p, scal_p), zs = mk(COMM)
    (arrays_s, scal_s), _ = mk(None)
    for k, (a, b) in enumerate(zip(arrays_p, arrays_s)):
        sl = (slice(None), zs) if a.ndim == 4 else (zs,)
        same(f"{name}[{k}]", a[sl], b[sl])
    same(f"{name} scalars", np.asarray(scal_p, np.float64), np.asarray(scal_s, np.float64))


# ---- C1: map-stencil-reduce loop (exact regime and real regime) ------------
def c1(seed, integer, occ):
    def fn(g):
        x, y = nb.Field(g), nb.Field(g)
        (x.fill_int(seed) if integer else x.fill_uniform(seed))
        y.fill_const(0.0)
        d = nb.nb_map_stencil_reduce(x, y, 0.125, 10, occ)
        out = [x.download(), y.download()]
        x.close(), y.close()
        return out, list(d)
    return fn


for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_TWO_WAY):
    compare(f"c1 int occ{occ}", (37, 21, 16), WORLD, c1(1, True, occ))
compare("c1 real 4 parts", (40, 24, 20), 2 * WORLD, c1(2, False, nb.OCC_TWO_WAY))


# ---- dot, laplace7 + halo update -------------------------------------------
def dot_lap(g):
    x, y = nb.Field(g), nb.Field(g)
    x.fill_uniform(3)
    y.fill_uniform(4)
    d = nb.nb_dot(x, y)
    x.halo_update()
    nb.nb_laplace7(x, y)
    out = [y.download()]
    x.close(), y.close()
    return out, [d]


compare("dot+laplace7", (45, 19, 22), WORLD, dot_lap)
compare("dot+laplace7 4 parts", (45, 19, 22), 2 * WORLD, dot_lap)


# ---- C2: Poisson CG ----------------------------------------------------------
def cg(occ, iters):
    def fn(g):
        b, x = nb.Field(g), nb.Field(g)
        b.fill(nb.FILL_POISSON_RHS)
        x.fill_const(0.0)
        c = nb.CG(x, b, max_iter=10 ** 6, occ=occ)
        c.iterate(iters)
        r = c.finish()
        c.close()
        out = [x.download()]
        b.close(), x.close()
        return out, [r.rr, r.rr0, r.iters]
    return fn


for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
    compare(f"cg occ{occ}", (32, 32, 32), WORLD, cg(occ, 21))
compare("cg 4 parts", (32, 32, 32), 2 * WORLD, cg(nb.OCC_TWO_WAY, 37))


# ---- C3: D3Q19 LBM (cavity and periodic) ------------------------------------
def lbm(bc, occ, steps):
    def fn(g):
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        nb.nb_lbm_init(a, 1.0, (0.01, -0.02, 0.015) if bc == nb.LBM_PERIODIC else (0.0, 0.0, 0.0))
        a, b = nb.nb_lbm_step(a, b, 0.9, steps, bc=bc, occ=occ)
        out = [a.download()]
        a.close(), b.close()
        return out, []
    return fn


for bc in (nb.LBM_CAVITY, nb.LBM_PERIODIC):
    for occ in (nb.OCC_NONE, nb.OCC_STANDARD):
        compare(f"lbm bc{bc} occ{occ}", (24, 20, 18), WORLD, lbm(bc, occ, 7))
compare("lbm periodic 4 parts", (24, 20, 18), 2 * WORLD, lbm(nb.LBM_PERIODIC, nb.OCC_STANDARD, 6))


def lbm_layout(layout, bc):
    """AoS / plane-major SoA populations: the fused boundary stores go into
    the neighbour's (IPC-mapped) halo with the layout's element stride."""
    def fn(g):
        a, b = nb.Field(g, "f32", 19, layout=layout), nb.Field(g, "f32", 19, layout=layout)
        nb.nb_lbm_init(a, 1.0, (0.01, -0.02, 0.015) if bc == nb.LBM_PERIODIC else (0.0, 0.0, 0.0))
        a, b = nb.nb_lbm_step(a, b, 0.9, 5, bc=bc, occ=nb.OCC_STANDARD)
        out = [a.download()]
        a.close(), b.close()
        return out, []
    return fn


for layout in (nb.SOA_PLANE, nb.AOS):
    compare(f"lbm layout{layout} cavity", (24, 20, 18), WORLD, lbm_layout(layout, nb.LBM_CAVITY))
    compare(f"lbm layout{layout} periodic", (24, 20, 18), WORLD, lbm_layout(layout, nb.LBM_PERIODIC))


def lbm_aa(bc):
    def fn(g):
        a = nb.Field(g, "f32", 19)
        nb.nb_lbm_init(a, 1.0, (0.01, -0.02, 0.015) if bc == nb.LBM_PERIODIC else (0.0, 0.0, 0.0))
        nb.nb_lbm_step_aa(a, 0.9, 6, bc=bc)
        out = [a.download()]
        a.close()
        return out, []
    return fn


if TRANSPORT == "peer":  # the AA pattern needs fused (peer-store) halos
    for bc in (nb.LBM_CAVITY, nb.LBM_PERIODIC):
        compare(f"lbm aa bc{bc}", (24, 20, 18), WORLD, lbm_aa(bc))


# ---- C4: element-sparse CG ---------------------------------------------------
n = 30
zz, yy, xx = np.meshgrid(*(np.arange(n) + 0.5 - n / 2,) * 3, indexing="ij")
sphere = ((xx ** 2 + yy ** 2 + zz ** 2) <= (0.41528 * n) ** 2).astype(np.uint8)


def sparse_cg(occ):
    def fn(g):
        b, x = nb.Field(g), nb.Field(g)
        b.fill_uniform(4)
        x.fill_const(0.0)
        r = nb.nb_cg_solve(x, b, max_iter=12, rtol=0.0, check_every=4, occ=occ)
        d = nb.nb_dot(b, b)
        out = [x.download()]
        b.close(), x.close()
        return out, [r.rr, r.iters, d]
    return fn


for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_TWO_WAY):  # serial, and split around the halo (OCC)
    compare(f"sparse cg occ{occ}", (n, n, n), WORLD, sparse_cg(occ), active=sphere)


# ---- C5: FEM 27-point CG -----------------------------------------------------
def fem_cg(occ):
    def fn(g):
        b, x = nb.Field(g, card=3), nb.Field(g, card=3)
        nb.nb_fem27_rhs(b, 1.0)
        x.fill_const(0.0)
        r = nb.nb_cg_solve(x, b, max_iter=9, rtol=0.0, op=nb.OP_FEM27, check_every=3, occ=occ)
        out = [x.download()]
        b.close(), x.close()
        return out, [r.rr, r.iters]
    return fn


for occ in (nb.OCC_NONE, nb.OCC_TWO_WAY):
    compare(f"fem cg occ{occ}", (12, 11, 14), WORLD, fem_cg(occ))
compare("fem cg 4 parts", (12, 11, 16), 2 * WORLD, fem_cg(nb.OCC_TWO_WAY))
for occ in (nb.OCC_NONE, nb.OCC_TWO_WAY):  # FEM on the element-sparse sphere
    compare(f"sparse fem cg occ{occ}", (n, n, n), WORLD, fem_cg(occ), active=sphere)

# ---- borrowed (torch-owned) storage: IPC handle of the enclosing allocation + offset
def wrapped_cg(g):
    pad = torch.empty(7, dtype=torch.float64, device=f"cuda:{DEV}")  # noqa: F841 (offsets the next blocks)
    b, x = nb.Field.empty_torch(g), nb.Field.empty_torch(g)
    b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0)
    r = nb.nb_cg_solve(x, b, max_iter=15, rtol=0.0, occ=nb.OCC_TWO_WAY)
    out = [x.download()]
    b.close(), x.close()
    return out, [r.rr, r.iters]


compare("wrapped cg", (20, 20, 20), WORLD, wrapped_cg)


# ---- the Skeleton across processes (§V): Listing 3 CG with device
# scalars, the Fig. 4a loop and the LBM step as generated schedules ----------
RR, PQ, ALPHA, BETA, RR2 = 0, 1, 2, 3, 4


def sk_cg(occ):
    def fn(g):
        b, x, r, p, q = (nb.Field(g) for _ in range(5))
        b.fill_uniform(8)
        for f in (x, p, q):
            f.fill_const(0.0)
        nb.nb_axpby(1.0, b, 0.0, r)
        with nb.Skeleton(g, occ) as s0:
            s0.dot(r, r, RR)
            s0.set_scalar(BETA, 0.0)
            s0.run()
        with nb.Skeleton(g, occ) as sk:
            sk.axpby_s(1.0, -1, r, 1.0, BETA, p)
            sk.poisson(p, q)
            sk.dot(p, q, PQ)
            sk.scalar(nb.SC_DIV, RR, PQ, ALPHA)
            sk.axpby_s(1.0, ALPHA, p, 1.0, -1, x)
            sk.axpby_s(-1.0, ALPHA, q, 1.0, -1, r)
            sk.dot(r, r, RR2)
            sk.scalar(nb.SC_DIV, RR2, RR, BETA)
            sk.scalar(nb.SC_COPY, RR2, 0, RR)
            for _ in range(7):
                sk.run()
            rr = sk.result(RR)
        out = [x.download()]
        for f in (b, x, r, p, q):
            f.close()
        return out, [rr]
    return fn


def sk_c1(occ):
    def fn(g):
        x, y = nb.Field(g), nb.Field(g)
        x.fill_uniform(2)
        y.fill_const(0.0)
        with nb.Skeleton(g, occ) as sk:
            for k in range(4):
                sk.axpy(0.125, y, x)
                sk.laplace7(x, y)
                sk.dot(x, y, k)
            sk.run()
            d = [sk.result(k) for k in range(4)]
        out = [x.download(), y.download()]
        x.close(), y.close()
        return out, d
    return fn


def sk_lbm(occ):
    def fn(g):
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        nb.nb_lbm_init(a, 1.0, (0.0, 0.0, 0.0))
        with nb.Skeleton(g, occ) as sk:
            sk.lbm(a, b, 0.9)
            sk.lbm(b, a, 0.9)
            for _ in range(3):
                sk.run()
        out = [a.download()]
        a.close(), b.close()
        return out, []
    return fn


for occ in (nb.OCC_NONE, nb.OCC_TWO_WAY):
    compare(f"skeleton listing3 cg occ{occ}", (28, 26, 24), WORLD, sk_cg(occ))
    compare(f"skeleton c1 occ{occ}", (37, 21, 16), WORLD, sk_c1(occ))
    compare(f"skeleton lbm occ{occ}", (24, 20, 18), WORLD, sk_lbm(occ))
compare("skeleton listing3 cg 4 parts", (28, 26, 24), 2 * WORLD, sk_cg(nb.OCC_STANDARD))


# ---- the peer path really ran: its kernels were launched ---------------------
if TRANSPORT != "peer":
    COMM.close()
    dist.barrier()
    print(f"PEER_OK rank {RANK} checks {checks} transport {TRANSPORT}", flush=True)
    dist.destroy_process_group()
    sys.exit(0)
g = nb.Grid((32, 32, 32), nparts=WORLD, comm=COMM)
b, x = nb.Field(g), nb.Field(g)
b.fill(nb.FILL_POISSON_RHS)
x.fill_const(0.0)
g.profile(True)
c = nb.CG(x, b, max_iter=100, occ=nb.OCC_TWO_WAY)
c.iterate(3)
c.finish()
counts = {k: g.profile_read(k)[0] for k in ("k_peer_signal", "k_peer_wait", "k_peer_round", "k_finalize")}
g.profile(False)
c.close(), b.close(), x.close()
g.close()
assert counts["k_peer_signal"] >= 3 and counts["k_peer_wait"] >= 3 and counts["k_finalize"] >= 6, counts
print(f"rank {RANK} peer kernels {counts}", flush=True)

COMM.close()
dist.barrier()
print(f"PEER_OK rank {RANK} checks {checks}", flush=True)
dist.destroy_process_group()
