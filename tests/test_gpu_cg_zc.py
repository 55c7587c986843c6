"""The CG phase kernels choose how many planes each CTA marches (a wave
model); the dot partials are per plane and tile, so every
choice must give the same bits.  Each choice is forced per process
(NB_CG_ZC), so the runs are separate processes of tools/cg_dump.py, which
prints a digest of x after K CG iterations and of a C1 loop."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()


def digest(args, zc):
    env = dict(os.environ)
    env.pop("NB_CG_ZC", None)
    if zc:
        env["NB_CG_ZC"] = str(zc)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "cg_dump.py"), *map(str, args)], env=env,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    return out.stdout.strip().splitlines()[-1]


@pytest.mark.parametrize("args", [(67, 9, 2), (140, 11, 1)])
def test_planes_per_cta_bitwise(args):
    ref = digest(args, None)
    for zc in (2, 5, 32):
        assert digest(args, zc) == ref, zc
