"""CPU-side checks of the C-ABI boundary: libnb.so loads, exports every
symbol include/nb.h declares, the pure host logic (partition plans) works
without a GPU, and GPU calls fail loudly (no CPU fallback)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_meneghinmjm22_b200 as nb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "nb.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(nb_[a-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def built():
    import __graft_entry__
    __graft_entry__.build()
    return nb.lib()


def test_every_declared_symbol_is_exported(built):
    syms = header_symbols()
    assert len(syms) >= 40
    missing = [s for s in syms if not hasattr(built, s)]
    assert not missing, missing
    # the binding declares a signature for every one of them
    assert set(syms) <= set(nb.SIGNATURES), set(syms) - set(nb.SIGNATURES)


def test_library_is_sm100a(built):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", nb.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_device_count(built):
    assert "sm_100a" in nb.nb_version()
    assert nb.nb_device_count() >= 0


@pytest.mark.parametrize("nz,parts", [(512, 1), (512, 8), (100, 3), (7, 7), (9, 4)])
def test_partition_plan_even_split(built, nz, parts):
    zb = nb.nb_partition_plan(nz, parts)
    sizes = np.diff(zb)
    assert zb[0] == 0 and zb[-1] == nz and len(zb) == parts + 1
    assert sizes.max() - sizes.min() <= 1 and sizes.min() >= 1
    # remainder goes to the lowest partitions
    assert list(sizes) == sorted(sizes, reverse=True)


def test_partition_plan_rejects_bad_input(built):
    with pytest.raises(nb.NbError) as e:
        nb.nb_partition_plan(4, 5)
    assert e.value.status == nb.NB_EINVAL
    with pytest.raises(nb.NbError):
        nb.nb_partition_plan(4, 0)


def test_weighted_plan_balances_sphere(built):
    import synth
    n = 128
    m = synth.sphere_mask(n)
    counts = m.reshape(n, -1).sum(1).astype(np.int64)
    for parts in (1, 2, 4, 8):
        zb = nb.nb_partition_plan_weighted(counts, parts)
        loads = [counts[zb[i]:zb[i + 1]].sum() for i in range(parts)]
        assert min(np.diff(zb)) >= 1
        # plane granularity: no slab exceeds the ideal load by more than one plane
        assert max(loads) <= counts.sum() / parts + counts.max()


def test_weighted_plan_all_empty_planes(built):
    zb = nb.nb_partition_plan_weighted(np.zeros(10, dtype=np.int64), 3)
    assert zb[0] == 0 and zb[-1] == 10 and min(np.diff(zb)) >= 1


@pytest.mark.skipif(nb.nb_device_count() if os.path.exists(nb.LIB_PATH) else 1,
                    reason="only meaningful on a host without a GPU")
def test_no_cpu_fallback(built):
    with pytest.raises(nb.NbError) as e:
        nb.Grid((8, 8, 8))
    assert e.value.status == nb.NB_ECUDA
