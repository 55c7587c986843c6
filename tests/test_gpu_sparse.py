"""GPU parity of the element-sparse grid (PAPER.md L248,
L472) against the oracle, plus sparse-vs-dense and partition invariance."""
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


def sgrid(mask, parts=1):
    nz, ny, nx = mask.shape
    return nb.Grid((nx, ny, nz), nparts=parts, devices=[0] * parts, active=mask)


def dgrid(dims, parts=1):
    return nb.Grid(dims, nparts=parts, devices=[0] * parts)


def sphere(n, r=0.45):
    return synth.sphere_mask(n, r)


def test_sparse_partition_info_and_roundtrip():
    m = sphere(24)
    x = synth.uniform((24, 24, 24), seed=1)
    for parts in (1, 3):
        with sgrid(m, parts) as g:
            info = [g.partition_info(p) for p in range(parts)]
            assert sum(i["n_cells"] for i in info) == int(m.sum())
            f = nb.Field(g, outside=-7.0)
            f.upload(x)
            got = f.download()
            assert np.array_equal(got, np.where(m, x, -7.0))
            f.fill_uniform(seed=4)
            assert np.array_equal(f.download(), np.where(m, synth.uniform((24, 24, 24), seed=4), -7.0))
            f.close()


@pytest.mark.parametrize("parts", [1, 2, 4])
def test_sparse_laplace_vs_oracle(parts):
    n = 32
    m = sphere(n)
    x = synth.uniform((n, n, n), seed=3)
    exp = oracle.sparse_laplace7(m, x)
    scale = oracle.sparse_laplace7(m, np.abs(x)) + 12 * np.abs(x) + 1e-300
    with sgrid(m, parts) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        fx.upload(x)
        fx.halo_update()
        nb.nb_laplace7(fx, fy, nb.VIEW_INTERNAL)
        nb.nb_laplace7(fx, fy, nb.VIEW_BOUNDARY)
        got = fy.download()
        fx.close(), fy.close()
    assert np.max(np.abs(got - exp)[m.astype(bool)] / scale[m.astype(bool)]) <= 1e-12
    # integer regime: bit-exact
    xi = synth.int_uniform((n, n, n), seed=3)
    with sgrid(m, parts) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        fx.upload(xi)
        fx.halo_update()
        nb.nb_laplace7(fx, fy)
        assert np.array_equal(fy.download(), oracle.sparse_laplace7(m, xi))
        fx.close(), fy.close()


def test_sparse_full_mask_equals_dense_bitwise_and_masked_dense():
    dims = (40, 17, 21)
    x = synth.uniform(dims, seed=8)
    full = np.ones(dims[::-1], dtype=np.uint8)
    with sgrid(full, 2) as g, dgrid(dims, 2) as d:
        fs, ys = nb.Field(g), nb.Field(g)
        fd, yd = nb.Field(d), nb.Field(d)
        fs.upload(x), fd.upload(x)
        fs.halo_update(), fd.halo_update()
        nb.nb_laplace7(fs, ys), nb.nb_laplace7(fd, yd)
        assert np.array_equal(ys.download(), yd.download())
        for f in (fs, ys, fd, yd):
            f.close()
    m = sphere(24)
    x = synth.uniform((24, 24, 24), seed=9)
    with sgrid(m) as g, dgrid((24, 24, 24)) as d:
        fs, ys = nb.Field(g), nb.Field(g)
        fd, yd = nb.Field(d), nb.Field(d)
        fs.upload(x), fd.upload(np.where(m, x, 0.0))
        nb.nb_laplace7(fs, ys), nb.nb_laplace7(fd, yd)
        assert np.array_equal(ys.download(), np.where(m, yd.download(), 0.0))
        for f in (fs, ys, fd, yd):
            f.close()


def test_sparse_dot_exact_real_and_partition_invariant():
    n = 40
    m = sphere(n)
    xi, yi = synth.int_uniform((n, n, n), seed=1), synth.int_uniform((n, n, n), seed=2)
    exact = float(np.sum((xi * yi)[m.astype(bool)]))
    xr, yr = synth.uniform((n, n, n), seed=5), synth.uniform((n, n, n), seed=6)
    o = oracle.dot(np.where(m, xr, 0.0), np.where(m, yr, 0.0))
    vals = []
    for parts in (1, 2, 3, 4):
        with sgrid(m, parts) as g:
            a, b = nb.Field(g), nb.Field(g)
            a.upload(xi), b.upload(yi)
            assert nb.nb_dot(a, b) == exact
            a.upload(xr), b.upload(yr)
            vals.append(nb.nb_dot(a, b))
            a.close(), b.close()
    assert abs(vals[0] - o) <= 1e-10 * abs(o)
    assert len(set(vals)) == 1


def test_sparse_axpby_views():
    n = 24
    m = sphere(n)
    x, y = synth.uniform((n, n, n), seed=1), synth.uniform((n, n, n), seed=2)
    with sgrid(m, 3) as g:
        fx, fy = nb.Field(g), nb.Field(g)
        fx.upload(x), fy.upload(y)
        nb.nb_axpby(0.5, fx, -2.0, fy, nb.VIEW_INTERNAL)
        nb.nb_axpby(0.5, fx, -2.0, fy, nb.VIEW_BOUNDARY)
        exp = np.where(m, oracle.axpby(0.5, x, -2.0, y), 0.0)
        s = np.abs(0.5 * x) + np.abs(2 * y)
        assert np.max(np.abs(fy.download() - exp) / s) <= 1e-12
        fx.close(), fy.close()


def run_sparse_cg(m, b, parts, iters, rtol=0.0, occ=nb.OCC_TWO_WAY, halo=nb.HALO_FUSED):
    with sgrid(m, parts) as g:
        g.set_halo_mode(halo)
        fb, fx = nb.Field(g), nb.Field(g)
        fb.upload(b)
        fx.upload(np.zeros_like(b))
        r = nb.nb_cg_solve(fx, fb, max_iter=iters, rtol=rtol, check_every=8, occ=occ)
        x = fx.download()
        fb.close(), fx.close()
    return x, r


def test_sparse_cg_vs_oracle_and_partition_invariance():
    n = 28
    m = sphere(n)
    b = np.where(m, synth.uniform((n, n, n), seed=4), 0.0)
    xo, ro, _ = oracle.cg(b, max_iter=15, op=oracle.OP_SPARSE7, mask=m)
    ref = None
    for parts in (1, 2, 4):
        x, r = run_sparse_cg(m, b, parts, 15)
        assert r.iters == 15
        assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo))
        assert abs(r.rr - ro.rr) <= 1e-9 * ro.rr
        if ref is None:
            ref = (x, r.rr)
        assert np.array_equal(x, ref[0]) and r.rr == ref[1], parts


def test_sparse_cg_converges_on_sphere():
    n = 20
    m = sphere(n)
    act = m.ravel().astype(bool)
    b = np.where(m, synth.uniform((n, n, n), seed=7), 0.0)
    x, r = run_sparse_cg(m, b, 2, 300, rtol=1e-12)
    assert r.converged == 1
    xo, ro, _ = oracle.cg(b, max_iter=300, op=oracle.OP_SPARSE7, mask=m, rtol=1e-12)
    assert abs(r.iters - ro.iters) <= 1
    assert np.max(np.abs(x.ravel()[act] - xo.ravel()[act])) <= 1e-10 * np.max(np.abs(xo))


def test_sparse_cg_occ_modes_bitwise_equal():
    """OCC on the sparse CG: boundary-plane map, halo of
    p in flight while the interior map and q pass run, then the boundary q
    pass.  Every OCC mode, partition count and halo transport (fused stream
    order or copies on the halo stream) gives the serial schedule's bits."""
    n = 26
    m = sphere(n)
    b = np.where(m, synth.uniform((n, n, n), seed=14), 0.0)
    ref = None
    for parts in (1, 2, 4):
        for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
            for halo in (nb.HALO_FUSED, nb.HALO_STREAM):
                x, r = run_sparse_cg(m, b, parts, 11, occ=occ, halo=halo)
                if ref is None:
                    ref = (x, r.rr)
                assert np.array_equal(x, ref[0]) and r.rr == ref[1], (parts, occ, halo)
    xo, ro, _ = oracle.cg(b, max_iter=11, op=oracle.OP_SPARSE7, mask=m)
    assert np.max(np.abs(ref[0] - xo)) <= 1e-11 * np.max(np.abs(xo))


@pytest.mark.parametrize("parts", [1, 3])
def test_sparse_cg_xruns_bitwise_equal_connectivity_table(parts, monkeypatch):
    """The q pass / set-up on x-runs (24 B per run) and on the per-cell
    connectivity table (NB_SP_CONN=1, 24 B per cell) compute the same
    neighbours in the same order: bitwise equal CG iterates, on the sphere and
    on a mask with holes, runs split by neighbour rows and segment edges."""
    n = 40
    rng = np.random.default_rng(3)
    masks = [sphere(n), (sphere(n) & (rng.random((n, n, n)) < 0.8)).astype(np.uint8)]
    for m in masks:
        b = np.where(m, synth.uniform((n, n, n), seed=6), 0.0)
        monkeypatch.delenv("NB_SP_CONN", raising=False)
        xa, ra = run_sparse_cg(m, b, parts, 9)
        monkeypatch.setenv("NB_SP_CONN", "1")
        xb, rb = run_sparse_cg(m, b, parts, 9)
        monkeypatch.delenv("NB_SP_CONN", raising=False)
        assert np.array_equal(xa, xb) and ra.rr == rb.rr and ra.rr0 == rb.rr0
        xo, ro, _ = oracle.cg(b, max_iter=9, op=oracle.OP_SPARSE7, mask=m)
        assert np.max(np.abs(xa - xo)) <= 1e-11 * np.max(np.abs(xo))


@pytest.mark.parametrize("parts", [1, 2, 3])
def test_sparse_cg_box_schedule_vs_segment_schedule_and_oracle(parts, monkeypatch):
    """The 2-phase box CG (NB_SP_CG_BOX=1: p_new / x / <p, Ap> in phase A,
    A p recomputed in phase B, dots per 32 x 8 tile) and the map / q / r
    segment schedule (default) solve the same system: both within the CG
    tolerance of the oracle (their dot orders differ, so not bitwise); ragged
    tiles, several z-chunks, a mask with holes."""
    rng = np.random.default_rng(5)
    m = synth.sphere_mask(70, 0.45)[:40, :45, :].copy()
    m &= (rng.random(m.shape) < 0.85).astype(np.uint8)
    nz, ny, nx = m.shape
    b = np.where(m, synth.uniform((nx, ny, nz), seed=6), 0.0)
    xo, ro, _ = oracle.cg(b, max_iter=12, op=oracle.OP_SPARSE7, mask=m)
    out = []
    for seg in (False, True):
        if seg:
            monkeypatch.delenv("NB_SP_CG_BOX", raising=False)
        else:
            monkeypatch.setenv("NB_SP_CG_BOX", "1")
        with nb.Grid((nx, ny, nz), nparts=parts, devices=[0] * parts, active=m) as g:
            fb, fx = nb.Field(g), nb.Field(g)
            fb.upload(b)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=12, occ=nb.OCC_TWO_WAY)
            x = fx.download()
            fb.close(), fx.close()
        assert r.iters == 12
        assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo)), seg
        assert abs(r.rr - ro.rr) <= 1e-9 * ro.rr
        out.append(x)
    assert np.max(np.abs(out[0] - out[1])) <= 1e-11 * np.max(np.abs(xo))


@pytest.mark.parametrize("parts", [1, 2])
def test_sparse_box_cg_full_mask_equals_dense_cg_bitwise(parts, monkeypatch):
    """On a full mask the box CG runs the dense CG's arithmetic in the dense
    canonical dot order (32 x 8 tiles, rows in y, tiles by the plane tree):
    its iterates equal the dense grid's bit for bit."""
    monkeypatch.setenv("NB_SP_CG_BOX", "1")
    dims = (40, 21, 19)  # ragged x and y tiles
    m = np.ones(dims[::-1], np.uint8)
    b = synth.uniform(dims, seed=9)
    xs = []
    for active in (None, m):
        with nb.Grid(dims, nparts=parts, devices=[0] * parts, active=active) as g:
            fb, fx = nb.Field(g), nb.Field(g)
            fb.upload(b)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=10, occ=nb.OCC_NONE)
            xs.append((fx.download(), r.rr, r.rr0))
            fb.close(), fx.close()
    assert xs[0][2] == xs[1][2] and xs[0][1] == xs[1][1]
    assert np.array_equal(xs[0][0], xs[1][0])
