"""GPU parity of the matrix-free Q1 linear-elastic operator and its CG
 against the oracle."""
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


def grid(dims, parts=1):
    return nb.Grid(dims, nparts=parts, devices=[0] * parts)


@pytest.mark.parametrize("dims,parts", [((9, 7, 8), 1), ((12, 11, 10), 2), ((33, 9, 12), 3)])
def test_fem_apply_vs_oracle(dims, parts):
    u = synth.uniform(dims, card=3, seed=2)
    exp = oracle.fem_apply(u, 1.0, 0.3)
    with grid(dims, parts) as g:
        fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
        fu.upload(u)
        fu.halo_update()
        nb.nb_fem27_apply(fu, fy, 1.0, 0.3)
        got = fy.download()
        fu.close(), fy.close()
    assert np.max(np.abs(got - exp)) <= 1e-13 * np.max(np.abs(exp))


def test_fem_apply_partition_invariant_bitwise():
    dims = (17, 13, 16)
    u = synth.uniform(dims, card=3, seed=3)
    ref = None
    for parts in (1, 2, 4):
        with grid(dims, parts) as g:
            fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
            fu.upload(u)
            fu.halo_update()
            nb.nb_fem27_apply(fu, fy, 1.0, 0.3)
            got = fy.download()
            fu.close(), fy.close()
        ref = got if ref is None else ref
        assert np.array_equal(got, ref), parts


def test_fem_rigid_translation_and_rhs():
    dims = (10, 9, 8)
    nx, ny, nz = dims
    with grid(dims) as g:
        fu, fy, fb = nb.Field(g, card=3), nb.Field(g, card=3), nb.Field(g, card=3)
        # rigid translation in x: zero force away from the Dirichlet layer
        u = np.zeros((3, nz, ny, nx))
        u[0] = 1.0
        fu.upload(u)
        nb.nb_fem27_apply(fu, fy)
        y = fy.download()
        assert np.max(np.abs(y[:, 2:])) < 1e-13
        nb.nb_fem27_rhs(fb, 1.0)
        b = fb.download()
        assert np.array_equal(b, oracle.fem_rhs(dims, 1.0))
        assert abs(b[2].sum() - (nx - 1) * (ny - 1)) < 1e-12
        for f in (fu, fy, fb):
            f.close()


def run_fem_cg(dims, parts, iters, rtol=0.0, occ=nb.OCC_TWO_WAY, halo=nb.HALO_FUSED):
    with grid(dims, parts) as g:
        g.set_halo_mode(halo)
        fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
        nb.nb_fem27_rhs(fb, 1.0)
        fx.upload(np.zeros((3,) + dims[::-1]))
        r = nb.nb_cg_solve(fx, fb, max_iter=iters, rtol=rtol, op=nb.OP_FEM27, check_every=16, occ=occ)
        x = fx.download()
        fb.close(), fx.close()
    return x, r


def test_fem_cg_vs_oracle_iterates_and_partitions():
    dims = (10, 9, 12)
    b = oracle.fem_rhs(dims, 1.0)
    xo, ro, _ = oracle.cg(b, max_iter=25, op=oracle.OP_FEM27)
    ref = None
    for parts in (1, 2, 3):
        x, r = run_fem_cg(dims, parts, 25)
        assert r.iters == 25
        assert np.max(np.abs(x - xo)) <= 1e-10 * np.max(np.abs(xo))
        if ref is None:
            ref = (x, r.rr)
        assert np.array_equal(x, ref[0]) and r.rr == ref[1], parts


def test_fem_cg_converges():
    dims = (8, 8, 8)
    x, r = run_fem_cg(dims, 2, 2000, rtol=1e-10)
    assert r.converged == 1
    b = oracle.fem_rhs(dims, 1.0)
    res = oracle.fem_apply(x, 1.0, 0.3) - b
    assert np.max(np.abs(res)) <= 1e-8 * np.max(np.abs(b))
    assert np.all(x[:, 0] == 0.0)        # Dirichlet plane stays fixed
    assert x[2, -1].mean() > 0           # the top moves outward (+z) under the pressure


@pytest.mark.parametrize("dims,parts", [((17, 13, 40), 1), ((34, 19, 37), 3), ((9, 10, 5), 1), ((20, 70, 13), 2),
                                        ((2, 9, 6), 1), ((98, 27, 70), 1), ((70, 20, 100), 2)])
def test_fem_kernels_bitwise_equal(dims, parts, monkeypatch):
    """The TMA-staged z-march (default), the register z-march and the
    one-node-per-thread kernel must agree bit for bit: each output receives
    the same FMA chain.  Chunks of 16 planes, ragged tails, partition
    edges, surface nodes and the Dirichlet plane are all covered; so are the
    CG dots."""
    u = synth.uniform(dims, card=3, seed=9)
    out = {}
    # kernel variants (NB_FEM_KERNEL), the z-marching face-column kernel
    # (NB_FEM_FACES=col), x-face nodes in the one-thread-per-node surface
    # kernel instead of the shared-memory x-face kernel (NB_FEM_FACES=node)
    # and the 3-pass CG schedule (NB_FEM_3PASS: map -> q = K p -> r), and
    # the one-CTA-per-plane residual kernel (NB_FEM_R_PLANE), and the
    # surface-node kernels serialised before the streaming kernel instead of
    # concurrent with its surface-free box (NB_FEM_CONC=0; the last two
    # shapes have >= 3 x 3 tiles and surface-free z-chunks) against the
    # default fused schedule
    envs = {None: {}, "zmarch": {"NB_FEM_KERNEL": "zmarch"}, "plain": {"NB_FEM_KERNEL": "plain"},
            "faces_col": {"NB_FEM_FACES": "col"}, "faces_node": {"NB_FEM_FACES": "node"},
            "3pass": {"NB_FEM_3PASS": "1"}, "r_plane": {"NB_FEM_R_PLANE": "1"}, "serial": {"NB_FEM_CONC": "0"}}
    for variant, env in envs.items():
        for k in ("NB_FEM_KERNEL", "NB_FEM_FACES", "NB_FEM_3PASS", "NB_FEM_R_PLANE", "NB_FEM_CONC"):
            if k in env:
                monkeypatch.setenv(k, env[k])
            else:
                monkeypatch.delenv(k, raising=False)
        with grid(dims, parts) as g:
            fu, fy = nb.Field(g, card=3), nb.Field(g, card=3)
            fu.upload(u)
            fu.halo_update()
            nb.nb_fem27_apply(fu, fy, 1.0, 0.3)
            y = fy.download()
            fb, fx = nb.Field(g, card=3), nb.Field(g, card=3)
            nb.nb_fem27_rhs(fb, 1.0)
            fx.fill_const(0.0)
            r = nb.nb_cg_solve(fx, fb, max_iter=7, rtol=0.0, op=nb.OP_FEM27)
            out[variant] = (y, fx.download(), r.rr)
            for f in (fu, fy, fb, fx):
                f.close()
    for v in ("zmarch", "plain", "faces_col", "faces_node", "3pass", "r_plane", "serial"):
        assert np.array_equal(out[None][0], out[v][0]), v
        assert np.array_equal(out[None][1], out[v][1]) and out[None][2] == out[v][2], v


def test_fem_cg_occ_modes_bitwise_equal():
    """OCC on the FEM CG: the p_new halo is
    sent after the boundary-plane map while phase A runs on the planes whose
    neighbours are own planes; the boundary planes follow the wait.  Every
    OCC mode, partition count (2-plane slabs included) and halo transport
    gives the serial schedule's bits."""
    dims = (13, 11, 16)
    ref = None
    for parts in (1, 2, 4, 8):
        for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_TWO_WAY):
            for halo in (nb.HALO_FUSED, nb.HALO_STREAM):
                x, r = run_fem_cg(dims, parts, 9, occ=occ, halo=halo)
                if ref is None:
                    ref = (x, r.rr)
                assert np.array_equal(x, ref[0]) and r.rr == ref[1], (parts, occ, halo)
    b = oracle.fem_rhs(dims, 1.0)
    xo, _, _ = oracle.cg(b, max_iter=9, op=oracle.OP_FEM27)
    assert np.max(np.abs(ref[0] - xo)) <= 1e-10 * np.max(np.abs(xo))
