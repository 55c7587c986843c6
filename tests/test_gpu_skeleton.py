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
