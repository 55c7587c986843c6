"""The Skeleton's generated schedules (§V) executed on the GPU
must reproduce the hand-written fused schedule of the same sequential code
bit for bit: the Fig. 4a loop x <- x + a y; y <- L(x);
d_k = <x, y> for 10 iterations, on 1, 2 and 4 partitions under every OCC
mode, against nb_map_stencil_reduce (one fused kernel per iteration) and
the oracle (exact regime)."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu
OCCS = [nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY]


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def run_skeleton(dims, parts, occ, x0, iters=10, a=0.125):
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        x, y = nb.Field(g), nb.Field(g)
        x.upload(x0)
        y.fill_const(0.0)
        with nb.Skeleton(g, occ) as sk:
            for k in range(iters):
                sk.axpy(a, y, x)      # map: x <- x + a y
                sk.laplace7(x, y)     # stencil: y <- L(x)
                sk.dot(x, y, k)       # reduce: d_k = <x, y>
            plan = sk.describe()
            sk.run()
            d = [sk.result(k) for k in range(iters)]
        out = (x.download(), y.download(), np.array(d), plan)
        x.close(), y.close()
    return out


def run_fused(dims, parts, occ, x0, iters=10, a=0.125):
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        x, y = nb.Field(g), nb.Field(g)
        x.upload(x0)
        y.fill_const(0.0)
        d = nb.nb_map_stencil_reduce(x, y, a, iters, occ)
        out = (x.download(), y.download(), np.array(d))
        x.close(), y.close()
    return out


@pytest.mark.parametrize("parts", [1, 2, 4])
@pytest.mark.parametrize("occ", OCCS)
def test_skeleton_c1_bitwise_equals_hand_written(parts, occ):
    dims = (45, 19, 24)
    x0 = synth.uniform(dims, seed=3)
    xs, ys, ds, plan = run_skeleton(dims, parts, occ, x0)
    xf, yf, df = run_fused(dims, parts, occ, x0)
    assert np.array_equal(xs, xf) and np.array_equal(ys, yf)
    assert np.array_equal(ds, df)
    halos = sum(n["op"] == "halo" for n in plan["nodes"])
    assert halos == (10 if parts > 1 else 0)


def test_skeleton_c1_exact_regime_vs_oracle():
    dims = (33, 17, 20)
    x0 = synth.int_uniform(dims, seed=1)
    xs, ys, ds, _ = run_skeleton(dims, 3, nb.OCC_TWO_WAY, x0)
    xo, yo, do = oracle.c1_loop(x0, 0.125, 10)
    assert np.array_equal(xs, xo) and np.array_equal(ys, yo)
    assert np.max(np.abs(ds - do) / np.abs(do)) <= 1e-10


def test_skeleton_runs_twice_and_orders_after_prior_work():
    dims = (40, 16, 16)
    with nb.Grid(dims, nparts=2, devices=[0, 0]) as g:
        x, y = nb.Field(g), nb.Field(g)
        x.fill_uniform(5)   # enqueued on the compute stream before the run
        y.fill_const(0.0)
        with nb.Skeleton(g, nb.OCC_TWO_WAY) as sk:
            sk.axpy(0.125, y, x)
            sk.laplace7(x, y)
            sk.dot(x, y, 0)
            sk.run()
            d1 = sk.result(0)
            sk.run()
            d2 = sk.result(0)
        xs = x.download()
        x.close(), y.close()
    xf, yf, df = run_fused(dims, 2, nb.OCC_TWO_WAY, synth.uniform(dims, seed=5), iters=2)
    assert np.array_equal(xs, xf) and [d1, d2] == list(df)


def test_skeleton_state_errors():
    with nb.Grid((16, 8, 8), nparts=2, devices=[0, 0]) as g:
        x, y = nb.Field(g), nb.Field(g)
        sk = nb.Skeleton(g)
        sk.laplace7(x, y)
        with pytest.raises(nb.NbError):
            sk.laplace7(x, x)  # in-place stencil
        with pytest.raises(nb.NbError):
            g.close()  # a live skeleton keeps the grid
        sk.run()
        with pytest.raises(nb.NbError):
            sk.dot(x, y, 0)  # compiled: no more containers
        sk.close()
        x.close(), y.close()


@pytest.mark.parametrize("parts,occ", [(1, nb.OCC_TWO_WAY), (3, nb.OCC_TWO_WAY), (3, nb.OCC_NONE),
                                       (2, nb.OCC_STANDARD)])
def test_large_c1_tma_chain_bitwise_equals_skeleton(parts, occ):
    """Above 2^21 cells the fused C1 chain runs on the TMA-staged kernel
    (k_cgA_tma<., C1>); it must still equal the unfused generated schedule
    bit for bit (ragged x / y tiles, several 32-plane chunks)."""
    dims = (130, 129, 131)
    x0 = synth.uniform(dims, seed=8)
    xs, ys, ds, _ = run_skeleton(dims, parts, occ, x0, iters=3)
    xf, yf, df = run_fused(dims, parts, occ, x0, iters=3)
    assert np.array_equal(xs, xf) and np.array_equal(ys, yf) and np.array_equal(ds, df)


# ---- Listing 3: the paper's own example --
# slots of the device scalars
RR, PQ, ALPHA, BETA, RR2 = 0, 1, 2, 3, 4


def listing3_iteration(sk, x, r, p, q):
    """One CG iteration written as sequential user code, UpdateP first (L460)."""
    sk.axpby_s(1.0, -1, r, 1.0, BETA, p)      # p <- r + beta p
    sk.poisson(p, q)                          # q <- A p   (A = -L)
    sk.dot(p, q, PQ)                          # pq <- <p, q>
    sk.scalar(nb.SC_DIV, RR, PQ, ALPHA)       # alpha <- rr / pq
    sk.axpby_s(1.0, ALPHA, p, 1.0, -1, x)     # x <- x + alpha p
    sk.axpby_s(-1.0, ALPHA, q, 1.0, -1, r)    # r <- r - alpha q
    sk.dot(r, r, RR2)                         # rr' <- <r, r>
    sk.scalar(nb.SC_DIV, RR2, RR, BETA)       # beta <- rr' / rr
    sk.scalar(nb.SC_COPY, RR2, 0, RR)         # rr <- rr'


def run_listing3(dims, parts, occ, iters, bh):
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        b, x, r, p, q = (nb.Field(g) for _ in range(5))
        b.upload(bh)
        for f in (x, p, q):
            f.fill_const(0.0)
        nb.nb_axpby(1.0, b, 0.0, r)           # r <- b - A x0 with x0 = 0
        with nb.Skeleton(g, occ) as s0:
            s0.dot(r, r, RR)
            s0.set_scalar(BETA, 0.0)
            s0.run()
        with nb.Skeleton(g, occ) as sk:
            listing3_iteration(sk, x, r, p, q)
            plan = sk.describe()
            for _ in range(iters):
                sk.run()
            rr = sk.result(RR)
        out = (x.download(), rr, plan)
        for f in (b, x, r, p, q):
            f.close()
    return out


@pytest.mark.parametrize("parts", [1, 2, 4])
@pytest.mark.parametrize("occ", OCCS)
def test_skeleton_listing3_cg_bitwise_equals_cg_solve(parts, occ):
    """Listing 3 CG as Containers (device-scalar alpha, beta) -> the
    generated schedule gives nb_cg_solve's iterate and <r, r> bit for bit."""
    dims = (45, 19, 37)
    bh = synth.uniform(dims, seed=3)
    iters = 9
    xs, rrs, plan = run_listing3(dims, parts, occ, iters, bh)
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        b, x = nb.Field(g), nb.Field(g)
        b.upload(bh)
        x.fill_const(0.0)
        res = nb.nb_cg_solve(x, b, max_iter=iters, rtol=0.0, occ=occ)
        xc = x.download()
        b.close(), x.close()
    assert res.iters == iters
    assert np.array_equal(xs, xc) and rrs == res.rr, (parts, occ)
    xo, ro, _ = oracle.cg(bh, max_iter=iters)
    assert np.max(np.abs(xs - xo)) <= 1e-11 * np.max(np.abs(xo))
    ops = [n["op"] for n in plan["nodes"]]
    assert ops.count("scalar") == 3 and ops.count("reduce") >= 2
    if parts > 1:
        assert "halo" in ops


@pytest.mark.parametrize("parts,occ", [(1, nb.OCC_NONE), (2, nb.OCC_NONE), (3, nb.OCC_STANDARD),
                                       (4, nb.OCC_TWO_WAY)])
def test_skeleton_lbm_bitwise_equals_lbm_step(parts, occ):
    """The D3Q19 step as a StencilOp container (twoPop: the next container
    swaps fin / fout): halo nodes carry the z-crossing populations, Standard
    OCC splits the step; equal to nb_lbm_step bit for bit."""
    dims = (24, 20, 18)
    from test_gpu_parity import lbm_state
    f0 = lbm_state(dims, 11)
    om = 1.1
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        a.upload(f0)
        with nb.Skeleton(g, occ) as sk:
            sk.lbm(a, b, om)
            sk.lbm(b, a, om)
            plan = sk.describe()
            for _ in range(3):
                sk.run()
        got = a.download()
        a.close(), b.close()
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        a.upload(f0)
        a2, b2 = nb.nb_lbm_step(a, b, om, 6, occ=min(occ, nb.OCC_STANDARD))
        exp = a2.download()
        a.close(), b.close()
    assert np.array_equal(got, exp)
    ops = [n["op"] for n in plan["nodes"]]
    if parts > 1:
        assert ops.count("halo") == 2
        if occ != nb.OCC_NONE:
            assert [n["view"] for n in plan["nodes"] if n["op"] == "stencil"].count("internal") == 2


def test_skeleton_listing3_cg_512_bench_config_bitwise():
    """Listing 3 CG in the bench's skeleton configuration (512^3, 4
    partitions, Two-way OCC): 2 iterations of the generated schedule equal
    nb_cg_solve's bit for bit at full size."""
    dims = (512, 512, 512)
    bh = synth.uniform(dims, seed=3)
    xs, rrs, _ = run_listing3(dims, 4, nb.OCC_TWO_WAY, 2, bh)
    with nb.Grid(dims, nparts=4, devices=[0] * 4) as g:
        b, x = nb.Field(g), nb.Field(g)
        b.upload(bh)
        x.fill_const(0.0)
        res = nb.nb_cg_solve(x, b, max_iter=2, rtol=0.0, occ=nb.OCC_TWO_WAY)
        xc = x.download()
        b.close(), x.close()
    assert res.iters == 2 and rrs == res.rr
    assert np.array_equal(xs, xc)
