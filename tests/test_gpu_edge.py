"""Edge cases and degenerate shapes (the parity bar: "empty and ragged
inputs, maximum sizes, the degenerate cases the method has"): one-cell-wide
dense grids, slabs of exactly two planes, sparse masks with empty planes
inside a partition and between partitions, a single active cell, an empty
mask, and FEM / LBM on the thinnest boxes they accept — each against the
oracle or bitwise across partitions."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def lap_scale(x):
    return oracle.laplace7(np.abs(x)) + 12.0 * np.abs(x)


@pytest.mark.parametrize("dims,parts", [((1, 1, 5), 1), ((1, 7, 4), 2), ((33, 1, 6), 3), ((1, 1, 4), 2),
                                        ((2, 3, 8), 4)])
def test_thin_dense_grids_laplace_dot_cg(dims, parts):
    x0 = synth.uniform(dims, seed=3)
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        fx.upload(x0)
        fx.halo_update()
        nb.nb_laplace7(fx, fy)
        y = fy.download()
        d = nb.nb_dot(fx, fy)
        b, x = nb.Field(g), nb.Field(g)
        b.upload(x0)
        x.fill_const(0.0)
        r = nb.nb_cg_solve(x, b, max_iter=6)
        xs = x.download()
        for f in (fx, fy, b, x):
            f.close()
    yo = oracle.laplace7(x0)
    assert np.max(np.abs(y - yo) / lap_scale(x0)) <= 1e-12
    assert abs(d - oracle.dot(x0, yo)) <= 1e-10 * max(abs(oracle.dot(x0, yo)), 1e-300)
    xo, ro, _ = oracle.cg(x0, max_iter=6)
    assert r.iters == ro.iters
    assert np.max(np.abs(xs - xo)) <= 1e-11 * max(np.max(np.abs(xo)), 1e-300)


def gap_mask(n=20):
    """Two blobs separated by empty planes (z = 8..11) and an empty plane
    inside the lower blob (z = 3)."""
    m = np.zeros((n, n, n), np.uint8)
    zz, yy, xx = np.meshgrid(*(np.arange(n) + 0.5 - n / 2,) * 3, indexing="ij")
    m[(xx ** 2 + yy ** 2) < 40] = 1
    m[8:12] = 0
    m[3] = 0
    return m


@pytest.mark.parametrize("parts", [1, 2, 3])
def test_sparse_with_empty_planes(parts):
    m = gap_mask()
    n = m.shape[0]
    b = np.where(m, synth.uniform((n, n, n), seed=6), 0.0)
    with nb.Grid((n, n, n), nparts=parts, devices=[0] * parts, active=m) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        fx.upload(b)
        fx.halo_update()
        nb.nb_laplace7(fx, fy)
        y = fy.download()
        fb, x = nb.Field(g), nb.Field(g)
        fb.upload(b)
        x.fill_const(0.0)
        r = nb.nb_cg_solve(x, fb, max_iter=9)
        xs = x.download()
        for f in (fx, fy, fb, x):
            f.close()
    exp = np.where(m, oracle.laplace7(b), 0.0)
    assert np.max(np.abs(y - exp) / (lap_scale(b) + 1e-300)) <= 1e-12
    xo, ro, _ = oracle.cg(b, max_iter=9, op=oracle.OP_SPARSE7, mask=m)
    assert np.max(np.abs(xs - xo)) <= 1e-11 * np.max(np.abs(xo))
    assert abs(r.rr - ro.rr) <= 1e-9 * ro.rr


def test_sparse_lbm_and_fem_with_empty_planes_partition_invariant():
    m = gap_mask(18)
    n = m.shape[0]
    outs = []
    for parts in (1, 3):
        with nb.Grid((n, n, n), nparts=parts, devices=[0] * parts, active=m) as g:
            a, c = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
            nb.nb_lbm_init(a, 1.0, (0.01, 0.0, 0.0))
            a, c = nb.nb_lbm_step(a, c, 1.1, 4)
            fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
            nb.nb_fem27_rhs(fb, 1.0)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=5, op=nb.OP_FEM27)
            outs.append((a.download(), fx.download(), r.rr))
            for f in (a, c, fb, fx):
                f.close()
    for u, v in zip(outs[0], outs[1]):
        assert np.array_equal(u, v)


def test_single_active_cell_and_empty_mask():
    n = 6
    m = np.zeros((n, n, n), np.uint8)
    m[2, 3, 4] = 1
    with nb.Grid((n, n, n), active=m) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        x0 = np.zeros((n, n, n))
        x0[2, 3, 4] = 2.5
        fx.upload(x0)
        fx.halo_update()
        nb.nb_laplace7(fx, fy)
        y = fy.download()
        assert y[2, 3, 4] == -15.0 and np.count_nonzero(y) == 1
        assert nb.nb_dot(fx, fx) == 6.25
        fx.close(), fy.close()
    with pytest.raises(nb.NbError):
        nb.Grid((n, n, n), active=np.zeros((n, n, n), np.uint8), nparts=2, devices=[0, 0])


def test_two_plane_slabs_lbm_and_fem_bitwise():
    dims = (12, 10, 8)  # 4 partitions of 2 planes
    from test_gpu_parity import lbm_state
    f0 = lbm_state(dims, 2)
    outs = []
    for parts in (1, 4):
        with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
            a, c = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
            a.upload(f0)
            a, c = nb.nb_lbm_step(a, c, 1.2, 3)
            fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
            nb.nb_fem27_rhs(fb, 1.0)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=6, op=nb.OP_FEM27)
            outs.append((a.download(), fx.download(), r.rr))
            for f in (a, c, fb, fx):
                f.close()
    for u, v in zip(outs[0], outs[1]):
        assert np.array_equal(u, v)
