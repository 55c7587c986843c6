"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle on the
same seeded inputs, element by element, at sizes spanning several tiles with
ragged tails; bit-identity across partition counts and OCC schedules.

Tolerances:
  maps / stencils (fp64): max_i |g_i - o_i| / s_i <= 1e-12, s_i = sum of |terms|
  dots (fp64):            |g - o| / |o| <= 1e-10
  LBM (fp32 vs fp64 oracle from the same fp32 state): pointwise rel <= 1e-5
  exact regimes (integers, dyadic scalars): bit-exact
"""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu

SHAPES = [(45, 19, 37), (64, 64, 64), (33, 8, 5)]  # (nx, ny, nz): ragged x/y tiles, z chunks


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def grid(dims, parts=1):
    return nb.Grid(dims, nparts=parts, devices=[0] * parts)


def field(g, host=None, dtype="f64", card=1, outside=0.0):
    f = nb.Field(g, dtype, card, outside)
    if host is not None:
        f.upload(host)
    return f


def lap_scale(x, outside=0.0):
    """s_i = sum_j |x_j| + 6|x_i| (out-of-domain terms = |outside|)."""
    return oracle.laplace7(np.abs(x), outside=abs(outside)) + 12.0 * np.abs(x)


# ---- generator, layout, I/O -----------------------------------------------
@pytest.mark.parametrize("dims", SHAPES)
@pytest.mark.parametrize("parts", [1, 3])
def test_fill_matches_synth_bytewise(dims, parts):
    if dims[2] < 2 * parts:
        pytest.skip("slab too thin")
    with grid(dims, parts) as g:
        f = field(g)
        f.fill_uniform(seed=7, lo=-1.0, hi=2.0)
        assert np.array_equal(f.download(), synth.uniform(dims, seed=7, lo=-1.0, hi=2.0))
        f.fill_int(seed=3, lo=-8, hi=8)
        assert np.array_equal(f.download(), synth.int_uniform(dims, seed=3))
        f32 = field(g, dtype="f32", card=3)
        f32.fill_uniform(seed=5)
        assert np.array_equal(f32.download(), synth.uniform(dims, card=3, seed=5, dtype=np.float32))
        f.close(), f32.close()


def test_poisson_rhs_matches_synth_bytewise():
    n = 40
    with grid((n, n, n), 3) as g:
        b = field(g)
        b.fill(nb.FILL_POISSON_RHS)
        assert np.array_equal(b.download(), synth.poisson_poly_rhs((n, n, n)))
        b.close()


def test_upload_download_roundtrip_multi_partition():
    dims = (37, 11, 23)
    h = synth.uniform(dims, card=2, seed=1)
    with grid(dims, 4) as g:
        f = field(g, h, card=2)
        assert np.array_equal(f.download(), h)
        f.close()


# ---- maps (eq. L104) --------------------------------------------------------
@pytest.mark.parametrize("parts", [1, 2])
def test_axpy_dyadic_bit_exact(parts):
    dims = (45, 19, 37)
    x, y = synth.int_uniform(dims, seed=1), synth.int_uniform(dims, seed=2)
    with grid(dims, parts) as g:
        fx, fy = field(g, x), field(g, y)
        nb.nb_axpy(0.125, fx, fy)
        assert np.array_equal(fy.download(), oracle.axpy(0.125, x, y))
        fx.close(), fy.close()


def test_axpby_real_and_views():
    dims = (45, 19, 37)
    x, y = synth.uniform(dims, seed=3), synth.uniform(dims, seed=4)
    a, b = 0.3, -1.7
    with grid(dims, 3) as g:
        fx, fy = field(g, x), field(g, y)
        nb.nb_axpby(a, fx, b, fy, nb.VIEW_INTERNAL)
        nb.nb_axpby(a, fx, b, fy, nb.VIEW_BOUNDARY)
        got = fy.download()
        exp = oracle.axpby(a, x, b, y)
        s = np.abs(a * x) + np.abs(b * y)
        assert np.max(np.abs(got - exp) / s) <= 1e-12
        # b == 0 is copy/scale: y's old contents (NaN) are not read
        fy.fill_const(np.nan)
        nb.nb_axpby(2.0, fx, 0.0, fy)
        assert np.array_equal(fy.download(), 2.0 * x)
        fx.close(), fy.close()


def test_views_partition_cells():
    dims = (16, 16, 20)
    with grid(dims, 3) as g:
        x = field(g, np.ones(dims[::-1]))
        y = field(g, np.zeros(dims[::-1]))
        nb.nb_axpy(1.0, x, y, nb.VIEW_INTERNAL)
        got = y.download()
        zb = nb.nb_partition_plan(20, 3)
        bnd = {zb[1] - 1, zb[1], zb[2] - 1, zb[2]}
        for z in range(20):
            assert np.all(got[z] == (0.0 if z in bnd else 1.0)), z
        nb.nb_axpy(1.0, x, y, nb.VIEW_BOUNDARY)
        assert np.all(y.download() == 1.0)
        info = [g.partition_info(p) for p in range(3)]
        assert sum(i["n_cells"] for i in info) == 16 * 16 * 20
        assert info[0]["n_bnd_lo"] == 0 and info[2]["n_bnd_hi"] == 0
        x.close(), y.close()


# ---- reduce (eq. L129) ------------------------------------------------------
def test_dot_integer_exact_and_partition_invariant():
    dims = (45, 19, 37)
    x, y = synth.int_uniform(dims, seed=1), synth.int_uniform(dims, seed=2)
    exact = float(np.sum(x.astype(np.int64) * y.astype(np.int64)))
    for parts in (1, 2, 3, 4):
        with grid(dims, parts) as g:
            fx, fy = field(g, x), field(g, y)
            assert nb.nb_dot(fx, fy) == exact
            fx.close(), fy.close()


def test_dot_real_vs_oracle_and_bitwise_partition_invariance():
    dims = (64, 64, 64)
    x, y = synth.uniform(dims, seed=5), synth.uniform(dims, seed=6)
    o = oracle.dot(x, y)
    vals = []
    for parts in (1, 2, 4, 8):
        with grid(dims, parts) as g:
            fx, fy = field(g, x), field(g, y)
            vals.append(nb.nb_dot(fx, fy))
            fx.close(), fy.close()
    assert abs(vals[0] - o) / abs(o) <= 1e-10
    assert len(set(vals)) == 1, vals


# ---- 7-point stencil (Listing 2) ------------------------------------------
@pytest.mark.parametrize("dims", SHAPES)
def test_laplace_quadratic_bit_exact(dims):
    nx, ny, nz = dims
    Z, Y, X = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    u = (X * X + Y * Y + Z * Z).astype(np.float64)
    with grid(dims) as g:
        fu, fy = field(g, u), field(g)
        nb.nb_laplace7(fu, fy)
        assert np.array_equal(fy.download(), oracle.laplace7(u))
        fu.close(), fy.close()


@pytest.mark.parametrize("dims", SHAPES)
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_laplace_real_vs_oracle(dims, dtype):
    npdt = np.float64 if dtype == "f64" else np.float32
    x = synth.uniform(dims, seed=11, dtype=npdt)
    outside = 0.25
    with grid(dims) as g:
        fx, fy = field(g, x, dtype, outside=outside), field(g, dtype=dtype)
        nb.nb_laplace7(fx, fy)
        got = fy.download().astype(np.float64)
        exp = oracle.laplace7(x.astype(np.float64), outside=outside)
        tol = 1e-12 if dtype == "f64" else 1e-5
        assert np.max(np.abs(got - exp) / lap_scale(x.astype(np.float64), outside)) <= tol
        fx.close(), fy.close()


def test_laplace_multi_partition_halo_bitwise():
    dims = (45, 19, 37)
    x = synth.uniform(dims, seed=12)
    ref = None
    for parts in (1, 2, 3, 5):
        with grid(dims, parts) as g:
            fx, fy = field(g, x), field(g)
            fx.halo_update()
            nb.nb_laplace7(fx, fy, nb.VIEW_INTERNAL)
            nb.nb_laplace7(fx, fy, nb.VIEW_BOUNDARY)
            got = fy.download()
            ref = got if ref is None else ref
            assert np.array_equal(got, ref), parts
            fx.close(), fy.close()
    assert np.max(np.abs(ref - oracle.laplace7(x)) / lap_scale(x)) <= 1e-12


# ---- config C1: map -> stencil -> reduce ----------------------------------
def test_c1_exact_regime_bit_exact_vs_oracle():
    dims = (64, 64, 64)
    x0 = synth.int_uniform(dims, seed=1)
    ox, oy, od = oracle.c1_loop(x0, 0.125, 10)
    with grid(dims) as g:
        fx, fy = field(g, x0), field(g, np.zeros_like(x0))
        dots = nb.nb_map_stencil_reduce(fx, fy, 0.125, 10, nb.OCC_TWO_WAY)
        assert np.array_equal(fx.download(), ox)
        assert np.array_equal(fy.download(), oy)
        assert np.max(np.abs(dots - od) / np.abs(od)) <= 1e-12
        fx.close(), fy.close()


@pytest.mark.parametrize("parts", [1, 3])
def test_c1_graph_replay_and_rebuild_bit_exact(parts, monkeypatch):
    """nb_map_stencil_reduce replays its loop as a CUDA graph: repeated calls
    on the same fields (replay), odd iteration counts (results copied back
    from the ping-pong partners), a changed scalar and changed fields
    (rebuild) must all equal the oracle, and the eager path bit for bit."""
    dims = (64, 40, 37)
    x0 = synth.int_uniform(dims, seed=3)
    # oracle: 4 + 4 iterations at a = 1/8, then 3 at a = 1/4 (dyadic scalars,
    # integer start: every operation is exact, so the order cannot matter)
    ox, oy, od1 = oracle.c1_loop(x0, 0.125, 4)
    ox, oy, od2 = oracle.c1_loop(ox, 0.125, 4, y0=oy)
    ox, oy, od3 = oracle.c1_loop(ox, 0.25, 3, y0=oy)
    out = {}
    for mode in ("graph", "graph_fin_each", "eager", "eager_fin_each"):
        # the loop's dots: one finalize per call over per-iteration slices
        # (default, single process) or one finalize per iteration
        if mode.startswith("eager"):
            monkeypatch.setenv("NB_NO_GRAPH", "1")
        if mode.endswith("fin_each"):
            monkeypatch.setenv("NB_C1_FIN_EACH", "1")
        else:
            monkeypatch.delenv("NB_C1_FIN_EACH", raising=False)
        with grid(dims, parts) as g:
            fx, fy = field(g, x0), field(g, np.zeros_like(x0))
            d1 = nb.nb_map_stencil_reduce(fx, fy, 0.125, 4, nb.OCC_TWO_WAY)
            d2 = nb.nb_map_stencil_reduce(fx, fy, 0.125, 4, nb.OCC_TWO_WAY)
            d3 = nb.nb_map_stencil_reduce(fx, fy, 0.25, 3, nb.OCC_TWO_WAY)
            gx, gy = fx.download(), fy.download()
            # other fields on the same grid: the cached graph must not be reused
            hx, hy = field(g, x0), field(g, np.zeros_like(x0))
            e1 = nb.nb_map_stencil_reduce(hx, hy, 0.125, 4, nb.OCC_TWO_WAY)
            assert np.array_equal(e1, d1)
            out[mode] = (gx, gy, d1, d2, d3)
            for f in (fx, fy, hx, hy):
                f.close()
        assert np.array_equal(gx, ox) and np.array_equal(gy, oy), mode
        for d, o in ((d1, od1), (d2, od2), (d3, od3)):
            assert np.max(np.abs(d - o) / np.abs(o)) <= 1e-12, mode
    for m in ("graph_fin_each", "eager", "eager_fin_each"):
        for a, b in zip(out["graph"], out[m]):
            assert np.array_equal(a, b), m


def test_c1_real_regime_vs_oracle():
    dims = (45, 19, 37)
    x0 = synth.uniform(dims, seed=1)
    ox, oy, od = oracle.c1_loop(x0, 0.125, 10)
    with grid(dims) as g:
        fx, fy = field(g, x0), field(g, np.zeros_like(x0))
        dots = nb.nb_map_stencil_reduce(fx, fy, 0.125, 7 + 3, nb.OCC_NONE)
        gx, gy = fx.download(), fy.download()
        scale = np.max(np.abs(ox))
        assert np.max(np.abs(gx - ox)) <= 1e-12 * scale * 10
        assert np.max(np.abs(gy - oy)) <= 1e-12 * np.max(np.abs(oy)) * 10
        assert np.max(np.abs(dots - od) / np.abs(od)) <= 1e-10
        fx.close(), fy.close()


@pytest.mark.parametrize("iters", [10, 3])
def test_c1_partition_and_occ_invariance_bitwise(iters):
    dims = (45, 19, 37)
    x0 = synth.uniform(dims, seed=2)
    ref = None
    for parts in (1, 2, 3, 4):
        for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
            with grid(dims, parts) as g:
                fx, fy = field(g, x0), field(g, np.zeros_like(x0))
                d = nb.nb_map_stencil_reduce(fx, fy, 0.125, iters, occ)
                out = (fx.download(), fy.download(), d)
                fx.close(), fy.close()
            if ref is None:
                ref = out
            for a, b in zip(out, ref):
                assert np.array_equal(a, b), (parts, occ)


# ---- CG (Listing 3, UpdateP first) ------------------------------------------
def run_cg(dims, parts, occ, iters, b_host=None, rtol=0.0, kind="poly"):
    with grid(dims, parts) as g:
        b = field(g)
        if kind == "poly":
            b.fill(nb.FILL_POISSON_RHS)
        else:
            b.upload(b_host)
        x = field(g, np.zeros(dims[::-1]))
        r = nb.nb_cg_solve(x, b, max_iter=iters, rtol=rtol, occ=occ, check_every=8)
        out = x.download()
        x.close(), b.close()
    return out, r


def test_cg_manufactured_solution():
    n = 32
    x, r = run_cg((n, n, n), 1, nb.OCC_TWO_WAY, 300, rtol=1e-12)
    xo, ro, _ = oracle.cg(synth.poisson_poly_rhs((n, n, n)), max_iter=300, rtol=1e-12)
    assert r.converged == 1 and r.iters == ro.iters
    assert np.max(np.abs(x - synth.poisson_poly_solution(n))) < 1e-12
    assert np.max(np.abs(x - xo)) < 1e-13
    # both stop at the same iteration once rr <= rtol^2 rr0 (the values there
    # are rounding noise, so only the criterion is compared)
    assert r.rr <= 1e-24 * r.rr0 and ro.rr <= 1e-24 * ro.rr0


def test_cg_random_rhs_vs_oracle_iterates():
    dims = (45, 19, 37)
    bh = synth.uniform(dims, seed=2)
    for k in (1, 2, 7, 20):
        x, r = run_cg(dims, 1, nb.OCC_TWO_WAY, k, b_host=bh, kind="host")
        xo, ro, _ = oracle.cg(bh, max_iter=k)
        assert r.iters == k
        assert np.max(np.abs(x - xo)) <= 1e-11 * np.max(np.abs(xo)), k
        assert abs(r.rr - ro.rr) <= 1e-9 * ro.rr, k


def test_cg_partition_and_occ_invariance_bitwise():
    dims = (45, 19, 37)
    bh = synth.uniform(dims, seed=3)
    ref = None
    for parts in (1, 2, 3, 4):
        for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
            x, r = run_cg(dims, parts, occ, 12, b_host=bh, kind="host")
            out = (x, r.rr, r.iters)
            ref = out if ref is None else ref
            assert np.array_equal(out[0], ref[0]) and out[1] == ref[1] and out[2] == ref[2], (parts, occ)


def test_cg_zero_rhs_and_eigenvector():
    n = 12
    x, r = run_cg((n, n, n), 2, nb.OCC_TWO_WAY, 5, b_host=np.zeros((n, n, n)), kind="host", rtol=1e-10)
    assert r.iters == 0 and r.converged == 2 and np.all(x == 0)
    s = np.sin(np.pi * np.arange(1, n + 1) / (n + 1))
    u = s[:, None, None] * s[None, :, None] * s[None, None, :]
    lam = 3 * (2 - 2 * np.cos(np.pi / (n + 1)))
    x, r = run_cg((n, n, n), 2, nb.OCC_TWO_WAY, 5, b_host=lam * u, kind="host", rtol=1e-13)
    assert r.iters == 1 and np.max(np.abs(x - u)) < 1e-14


def test_cg_iterate_in_pieces_equals_one_shot():
    dims = (33, 20, 17)
    with grid(dims) as g:
        b = field(g)
        b.fill_uniform(seed=9)
        x1, x2 = field(g, np.zeros(dims[::-1])), field(g, np.zeros(dims[::-1]))
        cg = nb.CG(x1, b)
        for n in (1, 4, 16, 3):
            cg.iterate(n)
        r1 = cg.finish()
        cg.close()
        r2 = nb.nb_cg_solve(x2, b, max_iter=24)
        assert r1.iters == r2.iters == 24 and r1.rr == r2.rr
        assert np.array_equal(x1.download(), x2.download())
        for f in (b, x1, x2):
            f.close()


# ---- D3Q19 BGK (L447-L456) ----------------------------------------------------
def lbm_state(dims, seed, amp=0.03):
    """Near-equilibrium fp32 state: feq(rho, u) with seeded rho, u, times a
    1 % seeded perturbation (post-collision populations stay well away from
    0, so pointwise relative error is meaningful)."""
    c, w, _ = oracle.lbm_lattice()
    rho = 1.0 + amp * synth.uniform(dims, seed=seed)
    u = amp * synth.uniform(dims, card=3, seed=seed + 1)
    cu = np.einsum("ia,a...->i...", c.astype(float), u)
    usq = (u * u).sum(0)
    f = w[:, None, None, None] * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * usq)
    f = f * (1 + 0.01 * synth.uniform(dims, card=19, seed=seed + 2))
    return f.astype(np.float32)


@pytest.mark.parametrize("bc", [nb.LBM_CAVITY, nb.LBM_PERIODIC])
@pytest.mark.parametrize("dims", [(37, 29, 23), (128, 3, 4)])
def test_lbm_one_step_vs_oracle(bc, dims):
    f0 = lbm_state(dims, 4)
    omega = 1.3
    with grid(dims) as g:
        a, b = field(g, f0, "f32", 19), field(g, dtype="f32", card=19)
        a2, _ = nb.nb_lbm_step(a, b, omega, 1, u_lid=0.05, bc=bc)
        got = a2.download().astype(np.float64)
        a.close(), b.close()
    exp = oracle.lbm_step(f0, omega, u_lid=0.05, bc=bc)
    assert np.max(np.abs(got - exp) / np.abs(exp)) <= 1e-5


def test_lbm_cavity_many_steps_and_mass():
    n = 24
    omega = oracle.lbm_omega(n)
    with grid((n, n, n)) as g:
        a, b = field(g, dtype="f32", card=19), field(g, dtype="f32", card=19)
        nb.nb_lbm_init(a, 1.0, (0.0, 0.0, 0.0))
        f0 = a.download().astype(np.float64)
        a, b = nb.nb_lbm_step(a, b, omega, 50)
        got = a.download().astype(np.float64)
        a.close(), b.close()
    exp = f0
    for _ in range(50):
        exp = oracle.lbm_step(exp, omega)
    assert np.max(np.abs(got - exp) / np.abs(exp)) <= 1e-5
    assert abs(got.sum() - f0.sum()) / f0.sum() <= 1e-5


@pytest.mark.parametrize("bc", [nb.LBM_CAVITY, nb.LBM_PERIODIC])
def test_lbm_partition_and_occ_invariance_bitwise(bc):
    dims = (37, 29, 23)
    f0 = lbm_state(dims, 8)
    ref = None
    for parts in (1, 2, 3):
        for occ in (nb.OCC_NONE, nb.OCC_STANDARD):
            with grid(dims, parts) as g:
                a, b = field(g, f0, "f32", 19), field(g, dtype="f32", card=19)
                a2, _ = nb.nb_lbm_step(a, b, 1.2, 5, bc=bc, occ=occ)
                got = a2.download()
                a.close(), b.close()
            ref = got if ref is None else ref
            assert np.array_equal(got, ref), (parts, occ)


def test_lbm_macroscopic_vs_oracle():
    dims = (20, 12, 9)
    f0 = lbm_state(dims, 5)
    with grid(dims) as g:
        a = field(g, f0, "f32", 19)
        rho, u = field(g, dtype="f32"), field(g, dtype="f32", card=3)
        nb.nb_lbm_macroscopic(a, rho, u)
        orho, ou = oracle.lbm_macroscopic(f0)
        assert np.max(np.abs(rho.download() - orho) / orho) <= 1e-6
        assert np.max(np.abs(u.download() - ou)) <= 1e-6
        a.close(), rho.close(), u.close()


# ---- error behaviour --------------------------------------------------------
def test_errors_are_reported_not_crashing():
    with grid((8, 8, 8)) as g:
        f = field(g)
        h = field(g, dtype="f32")
        with pytest.raises(nb.NbError) as e:
            nb.nb_axpy(1.0, f, h)
        assert e.value.status == nb.NB_EMISMATCH
        with pytest.raises(nb.NbError) as e:
            g.close()
        assert e.value.status == nb.NB_ESTATE
        f.close(), h.close()
    with pytest.raises(nb.NbError) as e:
        nb.Grid((8, 8, 3), nparts=2, devices=[0, 0])
    assert e.value.status == nb.NB_EUNSUPPORTED


# ---- halo transport: fused stores vs copies on the halo stream -------------
def test_halo_stream_mode_bitwise_equals_fused():
    """NB_HALO_STREAM (device copies on the halo stream, ordered by events and
    overlapped with the interior) must give the same bits as the fused halo
    stores, for CG, C1 and LBM under every OCC mode."""
    dims = (45, 19, 37)
    bh = synth.uniform(dims, seed=3)
    f0 = lbm_state(dims, 8)
    for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED):
        outs = []
        for mode in (nb.HALO_FUSED, nb.HALO_STREAM):
            with grid(dims, 3) as g:
                g.set_halo_mode(mode)
                b = field(g, bh)
                x = field(g, np.zeros(dims[::-1]))
                r = nb.nb_cg_solve(x, b, max_iter=9, occ=occ)
                y = field(g, np.zeros(dims[::-1]))
                x2 = field(g, bh)
                d = nb.nb_map_stencil_reduce(x2, y, 0.125, 4, occ)
                a, c = field(g, f0, "f32", 19), field(g, dtype="f32", card=19)
                a2, _ = nb.nb_lbm_step(a, c, 1.2, 4, occ=min(occ, nb.OCC_STANDARD))
                outs.append((x.download(), r.rr, x2.download(), y.download(), d, a2.download()))
                for f in (b, x, y, x2, a, c):
                    f.close()
        for u, v in zip(outs[0], outs[1]):
            assert np.array_equal(u, v), occ


def test_lbm_halo_stream_many_partitions_bitwise_equals_fused():
    """HALO_STREAM LBM on 6 virtual partitions puts 10 messages x 5
    populations = 50 plane copies into one exchange (more than 32 CopyBatch
    descriptors); it must equal the fused halo stores bit for bit."""
    dims = (24, 20, 30)
    f0 = lbm_state(dims, 5)
    outs = []
    for mode in (nb.HALO_FUSED, nb.HALO_STREAM):
        with grid(dims, 6) as g:
            g.set_halo_mode(mode)
            a, c = field(g, f0, "f32", 19), field(g, dtype="f32", card=19)
            a2, _ = nb.nb_lbm_step(a, c, 1.1, 3, occ=nb.OCC_STANDARD)
            outs.append(a2.download())
            a.close(), c.close()
    assert np.array_equal(outs[0], outs[1])
    exp = f0.astype(np.float64)
    for _ in range(3):
        exp = oracle.lbm_step(exp, 1.1)
    assert np.max(np.abs(outs[0] - exp) / np.abs(exp)) < 1e-5


@pytest.mark.parametrize("parts,occ", [(1, nb.OCC_TWO_WAY), (3, nb.OCC_EXTENDED), (2, nb.OCC_NONE)])
def test_large_c1_tma_chain_exact_regime_vs_oracle(parts, occ):
    """Above 2^21 cells the fused C1 chain runs on the TMA-staged kernel
    (k_cgA_tma<., C1>).  In the exact regime (integer x0, a = 1/8, SURVEY
    §8(c) c9 pin 1) x_10 and y_10 must equal the oracle bit for bit."""
    dims = (130, 129, 131)
    assert dims[0] * dims[1] * dims[2] > 2 ** 21
    x0 = synth.int_uniform(dims, seed=5)
    ox, oy, od = oracle.c1_loop(x0, 0.125, 10)
    with grid(dims, parts) as g:
        fx, fy = field(g, x0), field(g, np.zeros_like(x0))
        dots = nb.nb_map_stencil_reduce(fx, fy, 0.125, 10, occ)
        assert np.array_equal(fx.download(), ox)
        assert np.array_equal(fy.download(), oy)
        assert np.max(np.abs(dots - od) / np.abs(od)) <= 1e-12
        fx.close(), fy.close()
