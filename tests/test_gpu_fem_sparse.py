"""FEM on element-sparse grids:
nodes = active cells, an element exists iff its 8 nodes are active (the
oracle's reading).  The GPU K u, consistent pressure load and CG must match
the masked oracle (or_fem_apply / or_fem_rhs / or_cg); a full mask must give
the dense operator bit for bit; partitions, OCC modes and halo transports
must not change a bit."""
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


def masks():
    n = 14
    rng = np.random.default_rng(7)
    sph = synth.sphere_mask(n, 0.47)
    holes = (np.ones((n, n, n), bool) & (rng.random((n, n, n)) < 0.9)).astype(np.uint8)
    step = np.ones((12, 11, 13), np.uint8)
    step[7:, :, 5:] = 0  # a stepped top: exposed faces on two levels
    return {"sphere": sph, "holes": holes, "step": step}


def sgrid(mask, parts=1):
    nz, ny, nx = mask.shape
    return nb.Grid((nx, ny, nz), nparts=parts, devices=[0] * parts, active=mask)


@pytest.mark.parametrize("name", ["sphere", "holes", "step"])
@pytest.mark.parametrize("parts", [1, 3])
def test_sparse_fem_apply_and_rhs_vs_oracle(name, parts):
    m = masks()[name]
    nz, ny, nx = m.shape
    u = synth.uniform((nx, ny, nz), card=3, seed=5) * m[None]
    yo = oracle.fem_apply(u, 1.0, 0.3, mask=m)
    bo = oracle.fem_rhs((nx, ny, nz), 1.0, mask=m)
    with sgrid(m, parts) as g:
        fu, fy, fb = (nb.Field(g, card=3) for _ in range(3))
        fu.upload(u)
        fu.halo_update()
        nb.nb_fem27_apply(fu, fy)
        y = fy.download()
        nb.nb_fem27_rhs(fb, 1.0)
        b = fb.download()
        for f in (fu, fy, fb):
            f.close()
    assert np.max(np.abs(y - yo)) <= 1e-13 * max(np.max(np.abs(yo)), 1.0)
    assert np.array_equal(b, bo)  # dyadic loads in the oracle's order: bit-exact


def test_sparse_fem_full_mask_equals_dense_bitwise():
    dims = (13, 11, 12)
    m = np.ones(dims[::-1], np.uint8)
    u = synth.uniform(dims, card=3, seed=8)
    outs = []
    for active in (None, m):
        with nb.Grid(dims, nparts=2, devices=[0, 0], active=active) as g:
            fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
            fu.upload(u)
            fu.halo_update()
            nb.nb_fem27_apply(fu, fy)
            outs.append(fy.download())
            fu.close(), fy.close()
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("name", ["sphere", "step"])
def test_sparse_fem_cg_vs_oracle_and_invariance(name):
    m = masks()[name]
    nz, ny, nx = m.shape
    bo = oracle.fem_rhs((nx, ny, nz), 1.0, mask=m)
    xo, ro, _ = oracle.cg(bo, max_iter=12, op=oracle.OP_FEM27, mask=m)
    ref = None
    for parts in (1, 2, 3):
        for occ in (nb.OCC_NONE, nb.OCC_TWO_WAY):
            for halo in (nb.HALO_FUSED, nb.HALO_STREAM):
                with sgrid(m, parts) as g:
                    g.set_halo_mode(halo)
                    fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
                    nb.nb_fem27_rhs(fb, 1.0)
                    fx.fill_const(0.0)
                    r = nb.nb_cg_solve(fx, fb, max_iter=12, op=nb.OP_FEM27, occ=occ)
                    x = fx.download()
                    fb.close(), fx.close()
                if ref is None:
                    ref = (x, r.rr)
                    assert np.max(np.abs(x - xo)) <= 1e-10 * np.max(np.abs(xo))
                    assert abs(r.rr - ro.rr) <= 1e-9 * ro.rr
                assert np.array_equal(x, ref[0]) and r.rr == ref[1], (parts, occ, halo)


def test_sparse_fem_cg_converges():
    m = masks()["step"]
    nz, ny, nx = m.shape
    with sgrid(m, 2) as g:
        fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
        nb.nb_fem27_rhs(fb, 1.0)
        fx.fill_const(0.0)
        r = nb.nb_cg_solve(fx, fb, max_iter=3000, rtol=1e-10, op=nb.OP_FEM27)
        x = fx.download()
        fb.close(), fx.close()
    assert r.converged == 1
    b = oracle.fem_rhs((nx, ny, nz), 1.0, mask=m)
    res = oracle.fem_apply(x, 1.0, 0.3, mask=m) - b
    assert np.max(np.abs(res)) <= 1e-8 * np.max(np.abs(b))
    assert np.all(x[:, 0] == 0.0)


def _run_both(fn, modes=("NB_SPF_NONE", "NB_SPF_GATHER")):
    """fn() under each switch in `modes` set to 1 (NB_SPF_NONE: the default,
    the shared-memory box operator (warp-specialised, two rows per thread)
    after a separate map, <p, q> in a separate segment-order pass;
    NB_SFB_NR1: the single-role one-row box kernel; NB_SPF_TILEDOT: <p, q> in
    tile order inside the box kernel; NB_SPF_GATHER: the gather pass;
    NB_SPF_FUSED: the box operator's fused CG phase A)."""
    import os
    outs = []
    for m in modes:
        os.environ[m] = "1"
        try:
            outs.append(fn())
        finally:
            os.environ.pop(m, None)
    return outs


@pytest.mark.parametrize("name", ["sphere", "holes", "step", "wide"])
@pytest.mark.parametrize("parts", [1, 2, 3])
def test_sparse_fem_box_equals_gather_bitwise(name, parts):
    """The shared-memory box operator (k_sp_fem_box: 32 x 8 tiles, z-chunks,
    ragged x / y tiles) and the gather pass compute the same K u and the
    same CG iterates bit for bit (same per-node arithmetic, same dot)."""
    if name == "wide":  # several tiles in x and y, a ragged last tile, > 1 z-chunk
        m = synth.sphere_mask(70, 0.45)[:, :45, :]
        m = np.ascontiguousarray(m[:40])
    else:
        m = masks()[name]
    nz, ny, nx = m.shape
    u = synth.uniform((nx, ny, nz), card=3, seed=11) * m[None]

    def apply():
        with sgrid(m, parts) as g:
            fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
            fu.upload(u)
            fu.halo_update()
            nb.nb_fem27_apply(fu, fy)
            y = fy.download()
            fu.close(), fy.close()
        return y

    ya, yb, yc = _run_both(apply, ("NB_SPF_NONE", "NB_SPF_GATHER", "NB_SFB_NR1"))
    assert np.array_equal(ya, yb) and np.array_equal(ya, yc)
    yo = oracle.fem_apply(u, 1.0, 0.3, mask=m)
    assert np.max(np.abs(ya - yo)) <= 1e-13 * max(np.max(np.abs(yo)), 1.0)

    def cg():
        with sgrid(m, parts) as g:
            fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
            nb.nb_fem27_rhs(fb, 1.0)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=9, op=nb.OP_FEM27, occ=nb.OCC_TWO_WAY)
            x = fx.download()
            fb.close(), fx.close()
        return x, r.rr, r.iters

    # the segment-order dot schedules: bitwise equal (same per-node arithmetic, same dots)
    (xa, rra, ia), (xb, rrb, ib), (xc, rrc, ic) = _run_both(cg, ("NB_SPF_NONE", "NB_SPF_GATHER", "NB_SPF_FUSED"))
    assert ia == ib == ic and rra == rrb == rrc
    assert np.array_equal(xa, xb) and np.array_equal(xa, xc)
    # <p, q> in tile order (NB_SPF_TILEDOT): the same solve up to the dot's rounding
    (xd, rrd, idd), = _run_both(cg, ("NB_SPF_TILEDOT",))
    assert idd == ia and abs(rrd - rra) <= 1e-12 * rra
    assert np.max(np.abs(xd - xa)) <= 1e-12 * np.max(np.abs(xa))


def test_sparse_fem_degenerate_masks():
    """Degenerate element-sparse FEM domains through the box operator: lone
    nodes (no element: K u = 0 off the Dirichlet plane, the identity on it),
    a single element (8 active nodes), and a one-node-thick sheet (no
    element anywhere) — against the masked oracle."""
    n = 9
    cases = {}
    m = np.zeros((n, n, n), np.uint8)
    m[4, 3, 5] = 1
    m[0, 2, 2] = 1
    cases["lone"] = m
    m = np.zeros((n, n, n), np.uint8)
    m[3:5, 4:6, 1:3] = 1
    cases["one_element"] = m
    m = np.zeros((n, n, n), np.uint8)
    m[5, :, :] = 1
    cases["sheet"] = m
    for name, m in cases.items():
        u = synth.uniform((n, n, n), card=3, seed=13) * m[None]
        yo = oracle.fem_apply(u, 1.0, 0.3, mask=m)
        with sgrid(m, 1) as g:
            fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
            fu.upload(u)
            fu.halo_update()
            nb.nb_fem27_apply(fu, fy)
            y = fy.download()
            fu.close(), fy.close()
        assert np.max(np.abs(y - yo)) <= 1e-13 * max(np.max(np.abs(yo)), 1.0), name
        if name == "lone":
            assert np.all(y[:, 4, 3, 5] == 0.0) and np.array_equal(y[:, 0, 2, 2], u[:, 0, 2, 2])
