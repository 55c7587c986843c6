"""Borrowed storage (include/nb.h nb_field_required_elems / nb_field_wrap,
SURVEY.md §8(b) "field (borrowed)": PyTorch owns the memory) and the
device-resident dot (nb_dot_dev).  A field over torch tensors must behave
bit for bit like a library-allocated one."""
import numpy as np
import pytest

import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def test_required_elems_matches_layout():
    with nb.Grid((45, 19, 37), nparts=3, devices=[0] * 3) as g:
        for p in range(3):
            info = g.partition_info(p)
            nz = info["z_end"] - info["z_begin"]
            assert nb.Field.required_elems(g, 2, p) == 64 * 19 * (nz + 2) * 2  # pitch 64
        f = nb.Field.empty_torch(g, card=2)
        for p in range(3):
            ptr, pitch, ps, cs = f.partition_ptr(p)
            assert ptr == f.buffers[p].data_ptr() and pitch == 64 and ps == 64 * 19
        f.close()


@pytest.mark.parametrize("parts", [1, 3])
@pytest.mark.parametrize("outside", [0.0, 2.5])
def test_wrapped_field_bitwise_equals_owned(parts, outside):
    dims = (45, 19, 23)
    x0 = synth.uniform(dims, seed=11)
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        xo, yo = nb.Field(g, outside=outside), nb.Field(g)
        xw, yw = nb.Field.empty_torch(g, outside=outside), nb.Field.empty_torch(g)
        for f in (xo, xw):
            f.upload(x0)
            f.halo_update()
        nb.nb_laplace7(xo, yo)
        nb.nb_laplace7(xw, yw)
        assert np.array_equal(yo.download(), yw.download())
        d_host = nb.nb_dot(xw, yw)
        out = torch.full((1,), float("nan"), dtype=torch.float64, device="cuda")
        nb.nb_dot_dev(xw, yw, out.data_ptr())
        g.sync()
        assert out.item() == d_host == nb.nb_dot(xo, yo)
        for f in (xo, yo, xw, yw):
            f.close()


def test_wrapped_cg_and_sparse_bitwise():
    n = 24
    with nb.Grid((n, n, n), nparts=2, devices=[0, 0]) as g:
        res = []
        for mk in (lambda: nb.Field(g), lambda: nb.Field.empty_torch(g)):
            b, x = mk(), mk()
            b.fill(nb.FILL_POISSON_RHS)
            x.fill_const(0.0)
            r = nb.nb_cg_solve(x, b, max_iter=30, rtol=0.0)
            res.append((x.download(), r.rr))
            b.close(), x.close()
        assert np.array_equal(res[0][0], res[1][0]) and res[0][1] == res[1][1]
    zz, yy, xx = np.meshgrid(*(np.arange(n) + 0.5 - n / 2,) * 3, indexing="ij")
    m = ((xx ** 2 + yy ** 2 + zz ** 2) <= (0.41528 * n) ** 2).astype(np.uint8)
    with nb.Grid((n, n, n), nparts=3, devices=[0] * 3, active=m) as g:
        res = []
        for mk in (lambda: nb.Field(g), lambda: nb.Field.empty_torch(g)):
            b, x = mk(), mk()
            b.fill_uniform(4)
            x.fill_const(0.0)
            r = nb.nb_cg_solve(x, b, max_iter=12, rtol=0.0)
            res.append((x.download(), r.rr))
            b.close(), x.close()
        assert np.array_equal(res[0][0], res[1][0]) and res[0][1] == res[1][1]


def test_wrap_rejects_bad_pointers():
    with nb.Grid((16, 8, 8), nparts=1, devices=[0]) as g:
        n = nb.Field.required_elems(g, 1, 0)
        t = torch.empty(n + 2, dtype=torch.float64, device="cuda")
        with pytest.raises(nb.NbError):
            nb.Field.wrap(g, [t[1:]])  # 8-byte aligned only
        with pytest.raises(nb.NbError):
            nb.Field.wrap(g, [torch.empty(n, dtype=torch.float64)])  # host memory


@pytest.mark.parametrize("card,parts", [(19, 2), (19, 3), (3, 7)])
def test_halo_update_many_descriptors_fills_every_halo_plane(card, parts):
    """nb_halo_update batches all device-local plane copies of one exchange
    into ONE launch (CopyBatch): 19 components x 2 partitions is 38
    descriptors, 19 x 3 is 76 (more than one batch) — every halo plane of
    every component must equal the neighbour's boundary plane bit for bit
    (descriptors 32..47 once copied only a quarter of their plane)."""
    dims = (45, 19, 23)
    h = synth.uniform(dims, card=card, seed=21)
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        f = nb.Field.empty_torch(g, card=card, outside=-3.0)
        f.upload(h)
        f.halo_update()
        g.sync()
        nx, ny, _ = dims
        for p in range(parts):
            info = g.partition_info(p)
            z0, z1 = info["z_begin"], info["z_end"]
            _, pitch, ps, cs = f.partition_ptr(p)
            buf = f.buffers[p]
            for c in range(card):
                for zl, zg in ((-1, z0 - 1), (z1 - z0, z1)):
                    plane = buf[c * cs + (zl + 1) * ps: c * cs + (zl + 2) * ps].view(ny, pitch)[:, :nx]
                    got = plane.cpu().numpy()
                    exp = h[c, zg] if 0 <= zg < dims[2] else np.full((ny, nx), -3.0)
                    assert np.array_equal(got, exp), (p, c, zl)
        f.close()
