"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (single partition, default OCC, graph-launched CG), on outputs the
oracle can compute: whole-grid oracle CG iterations where the oracle takes
seconds (C2 512^3, C4 sparse 512^3), and sampled outputs computed one by one
on small oracle blocks elsewhere (C3 LBM 512^3, C5 FEM 384^3)."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def test_c2_poisson_cg_512_vs_oracle():
    """C2: 512^3 fp64, b = h^2 f (manufactured), x0 = 0: 3 CG iterations on
    the GPU (bench path: nb_cg_create / iterate / finish, graphs) vs the oracle."""
    n, k = 512, 3
    b = synth.poisson_poly_rhs((n, n, n))
    xo, ro, hist = oracle.cg(b, max_iter=k)
    with nb.Grid((n, n, n)) as g:
        fb, fx = nb.Field(g), nb.Field(g)
        fb.fill(nb.FILL_POISSON_RHS)
        fx.fill_const(0.0)
        cg = nb.CG(fx, fb)
        cg.prepare(k)
        cg.iterate(k)
        r = cg.finish()
        cg.close()
        x = fx.download()
        fb.close(), fx.close()
    assert r.iters == k
    assert abs(r.rr0 - hist[0]) <= 1e-12 * hist[0]
    assert abs(r.rr - ro.rr) <= 1e-10 * ro.rr
    assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo))


def test_c4_sparse_cg_512_vs_oracle():
    n, k = 512, 2
    m = synth.sphere_mask(n)
    b = np.where(m, synth.uniform((n, n, n), seed=4), 0.0)
    xo, ro, hist = oracle.cg(b, max_iter=k, op=oracle.OP_SPARSE7, mask=m)
    with nb.Grid((n, n, n), active=m) as g:
        fb, fx = nb.Field(g), nb.Field(g)
        fb.fill_uniform(seed=4)
        fx.fill_const(0.0)
        r = nb.nb_cg_solve(fx, fb, max_iter=k)
        x = fx.download()
        fb.close(), fx.close()
    assert r.iters == k
    assert abs(r.rr0 - hist[0]) <= 1e-12 * hist[0]
    assert abs(r.rr - ro.rr) <= 1e-10 * ro.rr
    assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo))


def _lbm_slab_oracle(f, z, omega, nz):
    """Oracle step for plane z of the full grid from the planes z-1..z+1 of
    the state f ([19][nz][ny][nx] fp32, global), computed on a 3-plane slab
    (2 planes at the global faces): every source of plane z lies in the
    slab, and the slab's own z faces coincide with the global ones where
    the slab is cut by them."""
    z0, z1 = max(z - 1, 0), min(z + 2, nz)
    sub = oracle.lbm_step(f[:, z0:z1], omega)
    return sub[:, z - z0]


def test_c3_lbm_512_sampled_planes_vs_oracle():
    n = 512
    omega = oracle.lbm_omega(n)
    planes = [0, 1, 255, 510, 511]
    with nb.Grid((n, n, n)) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        nb.nb_lbm_init(a, 1.0, (0.0, 0.0, 0.0))
        a, b = nb.nb_lbm_step(a, b, omega, 3)  # a non-trivial state near the lid
        f = a.download()
        a, b = nb.nb_lbm_step(a, b, omega, 1)
        f1 = a.download()
        a.close(), b.close()
    for z in planes:
        exp = _lbm_slab_oracle(f, z, omega, n)
        got = f1[:, z].astype(np.float64)
        assert np.max(np.abs(got - exp) / np.abs(exp)) <= 1e-5, z
    assert np.max(np.abs(f1[:, :, -1] - f[:, :, -1])) > 1e-6  # the lid drives the flow


def test_c5_fem_384_sampled_nodes_vs_oracle():
    n = 384
    rng = np.random.default_rng(0)
    pts = [(0, 0, 0), (n - 1, n - 1, n - 1), (1, 2, 1), (n // 2, n // 2, n // 2), (0, 200, 383), (383, 0, 1)]
    pts += [tuple(int(v) for v in rng.integers(0, n, 3)) for _ in range(10)]
    with nb.Grid((n, n, n)) as g:
        u, y = nb.Field(g, card=3), nb.Field(g, card=3)
        u.fill_uniform(seed=5)
        nb.nb_fem27_apply(u, y)
        ug, yg = u.download(), y.download()
        u.close(), y.close()
    for (x, yy, z) in pts:
        sl = [slice(max(c - 1, 0), min(c + 2, n)) for c in (z, yy, x)]
        blk = ug[:, sl[0], sl[1], sl[2]]
        exp = oracle.fem_apply(blk, 1.0, 0.3, dirichlet_z0=(sl[0].start == 0))
        loc = (z - sl[0].start, yy - sl[1].start, x - sl[2].start)
        e = exp[:, loc[0], loc[1], loc[2]]
        got = yg[:, z, yy, x]
        assert np.max(np.abs(got - e)) <= 1e-13 * max(1.0, np.max(np.abs(e))), (x, yy, z)


def test_c2_poisson_cg_1024_max_size_vs_oracle():
    """Maximum-size case: 1024^3 fp64 (8 x the C2 bench grid; 8.6 GB per
    field, the buffer offsets pass 2^33 bytes), 2 CG iterations on the bench
    path vs the oracle on the whole grid."""
    n, k = 1024, 2
    b = synth.poisson_poly_rhs((n, n, n))
    xo, ro, hist = oracle.cg(b, max_iter=k)
    del b
    with nb.Grid((n, n, n)) as g:
        fb, fx = nb.Field(g), nb.Field(g)
        fb.fill(nb.FILL_POISSON_RHS)
        fx.fill_const(0.0)
        cg = nb.CG(fx, fb)
        cg.prepare(k)
        cg.iterate(k)
        r = cg.finish()
        cg.close()
        fb.close()
        x = fx.download()
        fx.close()
    assert r.iters == k
    assert abs(r.rr0 - hist[0]) <= 1e-12 * hist[0]
    assert abs(r.rr - ro.rr) <= 1e-10 * ro.rr
    assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo))


@pytest.mark.parametrize("shape", ["sphere", "cube"])
def test_f4_sparse_fem_384_sampled_nodes_vs_oracle(shape):
    """FEM on element-sparse grids at the C5 size (384^3) through the box
    operator and its list nodes, in the bench's launch configuration: the
    C4-recipe sphere (30 % of the box) and the full cube (Dirichlet plane,
    faces, edges).  Sampled nodes — interior ones (box kernel) and surface /
    gz <= 1 ones (list kernel) — against the masked oracle on the 3x3x3
    neighbourhood block (a node's K u row only involves its 8 elements)."""
    n = 384
    m = synth.sphere_mask(n) if shape == "sphere" else np.ones((n, n, n), np.uint8)
    rng = np.random.default_rng(1)
    act = np.argwhere(m)
    pts = [tuple(int(v) for v in act[i][::-1]) for i in rng.integers(0, len(act), 12)]
    # surface nodes: the first and last active x of a few rows
    for (z, y) in ((n // 2, n // 2), (n // 3, n // 2 + 7), (2 * n // 3, n // 4 + 40)):
        xs = np.flatnonzero(m[z, y])
        if xs.size:
            pts += [(int(xs[0]), y, z), (int(xs[-1]), y, z)]
    if shape == "cube":
        pts += [(0, 0, 0), (n - 1, n - 1, n - 1), (5, 7, 1), (n // 2, 0, 2), (n - 1, n // 2, n // 2)]
    with nb.Grid((n, n, n), active=m) as g:
        u, y = nb.Field(g, card=3), nb.Field(g, card=3)
        u.fill_uniform(seed=5)
        nb.nb_fem27_apply(u, y)
        ug, yg = u.download(), y.download()
        u.close(), y.close()
    for (x, yy, z) in pts:
        assert m[z, yy, x]
        sl = [slice(max(c - 1, 0), min(c + 2, n)) for c in (z, yy, x)]
        mb = np.ascontiguousarray(m[sl[0], sl[1], sl[2]])
        blk = np.ascontiguousarray(ug[:, sl[0], sl[1], sl[2]])
        exp = oracle.fem_apply(blk, 1.0, 0.3, dirichlet_z0=(sl[0].start == 0), mask=mb)
        loc = (z - sl[0].start, yy - sl[1].start, x - sl[2].start)
        e = exp[:, loc[0], loc[1], loc[2]]
        got = yg[:, z, yy, x]
        assert np.max(np.abs(got - e)) <= 1e-13 * max(1.0, np.max(np.abs(e))), (shape, x, yy, z)


def test_f2_sparse_lbm_512_sphere_sampled_planes_vs_oracle():
    """D3Q19 on the element-sparse C4 sphere at the bench size (512^3, 40.3M
    active cells; bounce-back at the domain surface), a uniform initial flow
    and 3 steps, then one more: sampled
    planes (the bottom cap, the equator, near the top) against the masked
    oracle on the 3-plane slab around each."""
    n = 512
    m = synth.sphere_mask(n)
    omega = oracle.lbm_omega(n)
    zs = np.flatnonzero(m.reshape(n, -1).any(axis=1))
    planes = [int(zs[0]) + 1, n // 2, int(zs[-1]) - 2]
    with nb.Grid((n, n, n), active=m) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        # a uniform flow (the rest state would be a fixed point): the
        # bounce-back surface makes the state non-trivial after 3 steps
        nb.nb_lbm_init(a, 1.0, (0.05, 0.03, 0.02))
        a, b = nb.nb_lbm_step(a, b, omega, 3, u_lid=0.05)
        f = a.download()
        a, b = nb.nb_lbm_step(a, b, omega, 1, u_lid=0.05)
        f1 = a.download()
        a.close(), b.close()
    assert np.max(np.abs(f1[:, n // 2] - f[:, n // 2])) > 1e-4  # the surface keeps changing the state
    for z in planes:
        z0, z1 = max(z - 1, 0), min(z + 2, n)
        sub = oracle.lbm_step(f[:, z0:z1], omega, active=np.ascontiguousarray(m[z0:z1]))
        exp = sub[:, z - z0]
        act = m[z].astype(bool)
        got = f1[:, z].astype(np.float64)
        assert np.max(np.abs(got[:, act] - exp[:, act]) / np.abs(exp[:, act])) <= 1e-5, z


def test_f3_aa_pattern_512_equals_twopop_bitwise():
    """The AA pattern at the bench size (512^3, one 10.2 GB buffer) against
    twoPop (two buffers) after 4 steps of the lid-driven cavity from a
    uniform flow: bit for bit on sampled planes (the lid plane, the walls,
    the middle), and twoPop's planes against the oracle on a slab."""
    n = 512
    omega = oracle.lbm_omega(n)
    planes = [0, 1, n // 2, n - 2, n - 1]
    with nb.Grid((n, n, n)) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        nb.nb_lbm_init(a, 1.0, (0.02, 0.01, 0.0))
        a, b = nb.nb_lbm_step(a, b, omega, 3)
        f3 = np.ascontiguousarray(a.download()[:, n // 2 - 1:n // 2 + 2])
        a, b = nb.nb_lbm_step(a, b, omega, 1)
        two = a.download()
        a.close(), b.close()
    with nb.Grid((n, n, n)) as g:
        f = nb.Field(g, "f32", 19)
        nb.nb_lbm_init(f, 1.0, (0.02, 0.01, 0.0))
        nb.nb_lbm_step_aa(f, omega, 4)
        aa = f.download()
        f.close()
    for z in planes:
        assert np.array_equal(aa[:, z], two[:, z]), z
    # the middle plane of step 4 from step 3's planes (interior slab: no z wall)
    sub = oracle.lbm_step(f3, omega)
    exp = sub[:, 1]
    got = two[:, n // 2].astype(np.float64)
    assert np.max(np.abs(got - exp) / np.abs(exp)) <= 1e-5


def test_f4_karman_32768x8192_sampled_rows_vs_oracle():
    """The largest PAPER.md Table I domain (32768 x 8192, 268M cells) in the
    bench's configuration (D2Q9 channel, cylinder r = ny/10 at (nx/5, ny/2),
    Re 150): after 4 + 1 steps from the uniform inflow, sampled rows (the
    walls, through the cylinder, between) against the oracle's D2Q9 step on
    the 3-row slab around each (the cylinder shifted into the slab)."""
    nx, ny = 32768, 8192
    u = 0.08
    cyl = (nx // 5, ny // 2, ny // 10)
    omega = 1.0 / (3 * u * 2 * cyl[2] / 150.0 + 0.5)
    rows = [0, 1, cyl[1] - cyl[2] - 1, cyl[1], cyl[1] + cyl[2], ny - 2, ny - 1]
    with nb.Grid((nx, ny, 1)) as g:
        a, b = nb.Field(g, "f32", 9), nb.Field(g, "f32", 9)
        nb.nb_d2q9_init(a, 1.0, u, 0.0)
        a, b = nb.nb_d2q9_step(a, b, omega, u, cyl, 4)
        f = a.download()[:, 0]
        a, b = nb.nb_d2q9_step(a, b, omega, u, cyl, 1)
        f1 = a.download()[:, 0]
        a.close(), b.close()
    assert np.max(np.abs(f1[:, cyl[1]] - f[:, cyl[1]])) > 1e-5  # the cylinder perturbs the flow
    for y in rows:
        y0, y1 = max(y - 1, 0), min(y + 2, ny)
        sub = np.ascontiguousarray(f[:, y0:y1])
        exp = oracle.d2q9_step(sub, omega, u, (cyl[0], cyl[1] - y0, cyl[2]))[:, y - y0]
        got = f1[:, y].astype(np.float64)
        nz = exp != 0
        assert np.all(got[~nz] == 0), y
        assert np.max(np.abs(got[nz] - exp[nz]) / np.abs(exp[nz])) <= 1e-5, y
