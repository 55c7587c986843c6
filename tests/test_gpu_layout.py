"""Field layouts ("SoA or AoS organizations without impacting
the application code", L256 2 vs 2n halo transfers; include/nb.h nb_layout):
SOA [c][z][y][x], SOA_PLANE [z][c][y][x] and AOS [z][y][x][c] must give the
same bits for every operation that takes them — fills, host transfers,
maps, dots, halo updates, the D3Q19 step (fused and halo-stream transports,
OCC) and the FEM CG — and the operations that do not take a layout must say
so (NB_EUNSUPPORTED)."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu
LAYOUTS = [nb.SOA, nb.SOA_PLANE, nb.AOS]


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def grid(dims, parts=1):
    return nb.Grid(dims, nparts=parts, devices=[0] * parts)


@pytest.mark.parametrize("layout", LAYOUTS)
@pytest.mark.parametrize("parts", [1, 3])
def test_fill_and_roundtrip_every_layout(layout, parts):
    dims = (45, 19, 23)
    with grid(dims, parts) as g:
        f = nb.Field(g, card=3, layout=layout)
        assert f.layout == layout
        f.fill_uniform(seed=7, lo=-1.0, hi=2.0)
        assert np.array_equal(f.download(), synth.uniform(dims, card=3, seed=7, lo=-1.0, hi=2.0))
        h = synth.uniform(dims, card=3, seed=9)
        f.upload(h)
        assert np.array_equal(f.download(), h)
        s = nb.Field(g, "f32", 19, layout=layout)
        s.fill_uniform(seed=5)
        assert np.array_equal(s.download(), synth.uniform(dims, card=19, seed=5, dtype=np.float32))
        one = nb.Field(g, layout=layout)
        assert one.layout == nb.SOA  # one component: the layouts coincide
        f.close(), s.close(), one.close()


@pytest.mark.parametrize("parts", [1, 2, 4])
def test_maps_dots_halo_bitwise_across_layouts(parts):
    dims = (37, 21, 16)
    x0 = synth.uniform(dims, card=3, seed=1)
    y0 = synth.uniform(dims, card=3, seed=2)
    outs = []
    for layout in LAYOUTS:
        with grid(dims, parts) as g:
            x, y = nb.Field(g, card=3, layout=layout), nb.Field(g, card=3, layout=layout)
            x.upload(x0), y.upload(y0)
            nb.nb_axpby(0.3, x, -1.7, y, nb.VIEW_INTERNAL)
            nb.nb_axpby(0.3, x, -1.7, y, nb.VIEW_BOUNDARY)
            nb.nb_axpy(0.125, y, x)
            d = nb.nb_dot(x, y)
            outs.append((x.download(), y.download(), d))
            x.close(), y.close()
    for o in outs[1:]:
        for a, b in zip(outs[0], o):
            assert np.array_equal(a, b)
    ex = x0 + 0.125 * (0.3 * x0 - 1.7 * y0)
    assert np.max(np.abs(outs[0][0] - ex)) < 1e-14
    ref = oracle.dot(outs[0][0], outs[0][1])
    assert abs(outs[0][2] - ref) <= 1e-12 * abs(ref)


def torch_halo_planes(f, g, p):
    """The halo planes of partition p read back through the layout formula."""
    ptr, pitch, ps, cs = f.partition_ptr(p)
    buf = f.buffers[p].cpu().numpy()
    nx, ny, _ = g.dims
    es = f.card if f.layout == nb.AOS else 1
    info = g.partition_info(p)
    nzl = info["z_end"] - info["z_begin"]
    out = {}
    for zl in (-1, nzl):
        idx = (np.arange(f.card)[:, None, None] * cs
               + (((zl + 1) * ps + np.arange(ny)[:, None] * pitch + np.arange(nx)[None, :]) * es)[None])
        out[zl] = buf[idx]
    return out


@pytest.mark.parametrize("layout", LAYOUTS)
def test_halo_update_every_layout(layout):
    torch = pytest.importorskip("torch")  # noqa: F841
    dims = (33, 12, 20)
    h = synth.uniform(dims, card=5, seed=4)
    with grid(dims, 3) as g:
        f = nb.Field.empty_torch(g, card=5, outside=-2.0, layout=layout)
        f.upload(h)
        f.halo_update()
        g.sync()
        for p in range(3):
            info = g.partition_info(p)
            z0, z1 = info["z_begin"], info["z_end"]
            hp = torch_halo_planes(f, g, p)
            for zl, zg in ((-1, z0 - 1), (z1 - z0, z1)):
                exp = h[:, zg] if 0 <= zg < dims[2] else np.full((5,) + dims[1::-1], -2.0)
                assert np.array_equal(hp[zl], exp), (p, zl)
        f.close()


@pytest.mark.parametrize("parts,occ,halo", [(1, nb.OCC_NONE, nb.HALO_FUSED), (3, nb.OCC_STANDARD, nb.HALO_FUSED),
                                            (3, nb.OCC_STANDARD, nb.HALO_STREAM), (2, nb.OCC_NONE, nb.HALO_STREAM)])
@pytest.mark.parametrize("bc", [nb.LBM_CAVITY, nb.LBM_PERIODIC])
def test_lbm_bitwise_across_layouts(parts, occ, halo, bc):
    from test_gpu_parity import lbm_state
    dims = (24, 20, 18)
    f0 = lbm_state(dims, 6)
    outs = []
    for layout in LAYOUTS:
        with grid(dims, parts) as g:
            g.set_halo_mode(halo)
            a, b = nb.Field(g, "f32", 19, layout=layout), nb.Field(g, "f32", 19, layout=layout)
            a.upload(f0)
            a2, b2 = nb.nb_lbm_step(a, b, 1.05, 5, bc=bc, occ=occ)
            rho, u = nb.Field(g, "f32", 1), nb.Field(g, "f32", 3, layout=layout)
            nb.nb_lbm_macroscopic(a2, rho, u)
            outs.append((a2.download(), rho.download(), u.download()))
            for f in (a, b, rho, u):
                f.close()
    for o in outs[1:]:
        for x, y in zip(outs[0], o):
            assert np.array_equal(x, y)
    exp = f0.astype(np.float64)
    for _ in range(5):
        exp = oracle.lbm_step(exp, 1.05, bc=bc)
    assert np.max(np.abs(outs[0][0] - exp) / np.abs(exp)) < 1e-5


def test_lbm_init_every_layout():
    dims = (16, 12, 10)
    outs = []
    for layout in LAYOUTS:
        with grid(dims, 2) as g:
            a = nb.Field(g, "f32", 19, layout=layout)
            nb.nb_lbm_init(a, 1.02, (0.01, -0.02, 0.03))
            outs.append(a.download())
            a.close()
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


@pytest.mark.parametrize("parts", [1, 3])
def test_fem_cg_soa_plane_bitwise_equals_soa(parts):
    dims = (11, 10, 13)
    outs = []
    for layout in (nb.SOA, nb.SOA_PLANE):
        with grid(dims, parts) as g:
            u, y = nb.Field(g, card=3, layout=layout), nb.Field(g, card=3, layout=layout)
            u.upload(synth.uniform(dims, card=3, seed=3))
            u.halo_update()
            nb.nb_fem27_apply(u, y)
            b, x = nb.Field(g, card=3, layout=layout), nb.Field(g, card=3, layout=layout)
            nb.nb_fem27_rhs(b, 1.0)
            x.fill_const(0.0)
            r = nb.nb_cg_solve(x, b, max_iter=8, op=nb.OP_FEM27)
            outs.append((y.download(), x.download(), r.rr))
            for f in (u, y, b, x):
                f.close()
    for a, b in zip(outs[0], outs[1]):
        assert np.array_equal(a, b)


def test_unsupported_layouts_are_reported():
    dims = (16, 12, 10)
    with grid(dims) as g:
        u, y = nb.Field(g, card=3, layout=nb.AOS), nb.Field(g, card=3, layout=nb.AOS)
        with pytest.raises(nb.NbError) as e:
            nb.nb_fem27_apply(u, y)
        assert e.value.status == nb.NB_EUNSUPPORTED
        f = nb.Field(g, "f32", 19, layout=nb.SOA_PLANE)
        with pytest.raises(nb.NbError) as e:
            nb.nb_lbm_step_aa(f, 1.0, 2)
        assert e.value.status == nb.NB_EUNSUPPORTED
        v = nb.Field(g, card=3)
        with pytest.raises(nb.NbError) as e:
            nb.nb_axpy(1.0, u, v)  # layouts differ
        assert e.value.status == nb.NB_EMISMATCH
        for h in (u, y, f, v):
            h.close()
    m = synth.sphere_mask(12)
    with nb.Grid((12, 12, 12), active=m) as g:
        with pytest.raises(nb.NbError) as e:
            nb.Field(g, card=3, layout=nb.AOS)
        assert e.value.status == nb.NB_EUNSUPPORTED


def test_lbm_layouts_512_bench_config_bitwise():
    """The bench's layout lines at full size (512^3 cavity, 1 partition):
    3 steps of the D3Q19 step from a uniform flow on SoA, plane-major SoA
    and AoS populations give the same bits on sampled planes."""
    n = 512
    omega = oracle.lbm_omega(n)
    planes = [0, 1, n // 2, n - 1]
    outs = []
    for layout in LAYOUTS:
        with nb.Grid((n, n, n)) as g:
            a, b = nb.Field(g, "f32", 19, layout=layout), nb.Field(g, "f32", 19, layout=layout)
            nb.nb_lbm_init(a, 1.0, (0.02, 0.01, 0.0))
            a, b = nb.nb_lbm_step(a, b, omega, 3)
            f = a.download()
            outs.append([np.ascontiguousarray(f[:, z]) for z in planes])
            del f
            a.close(), b.close()
    for o in outs[1:]:
        for x, y in zip(outs[0], o):
            assert np.array_equal(x, y)
