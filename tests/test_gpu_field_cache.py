"""The grid's field buffer cache: a destroyed field's device
buffer is handed to the next field of the same size, a new field still
starts at its outside value, other sizes allocate, NB_NO_FIELD_CACHE frees
at once, nb_grid_trim returns the cached bytes."""
import numpy as np
import pytest

import paper_conf_ipps_meneghinmjm22_b200 as nb

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def _ptr(f):
    return f.partition_ptr(0)[0]


@pytest.mark.parametrize("sparse", [False, True])
def test_field_buffers_are_reused_and_reset(sparse):
    dims = (20, 18, 16)
    m = np.ones(dims[::-1], np.uint8) if sparse else None
    with nb.Grid(dims, active=m) as g:
        a = nb.Field(g)
        a.fill_uniform(seed=3)
        pa = _ptr(a)
        a.close()
        b = nb.Field(g)  # same size: the cached buffer, reset to the outside value (0)
        assert _ptr(b) == pa
        assert np.count_nonzero(b.download()) == 0
        c = nb.Field(g, card=3)  # another size: a fresh allocation
        assert _ptr(c) != pa
        b.close(), c.close()
        assert g.trim() > 0
        assert g.trim() == 0


def test_no_field_cache_frees_at_once(monkeypatch):
    monkeypatch.setenv("NB_NO_FIELD_CACHE", "1")
    with nb.Grid((16, 16, 16)) as g:
        a = nb.Field(g)
        a.close()
        assert g.trim() == 0
