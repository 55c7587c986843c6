"""Multi-process peer-memory transport (include/nb.h nb_comm_create_peer):
two processes, one slab range each, CUDA IPC halos + flag signalling +
cross-rank deterministic reductions — bitwise equal to one process running
the same partition plan (tests/peer_worker.py holds the cases: C1, dot,
laplace7 + halo update, CG under all OCC modes, LBM cavity / periodic,
sparse CG, FEM CG).  On the single-GPU test box both ranks share cuda:0,
which exercises the same IPC mappings, stores and flags (NVLink peers on a
multi-GPU node)."""
import os
import socket
import subprocess
import sys

import pytest

import paper_conf_ipps_meneghinmjm22_b200 as nb

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world", [2, 3])
def test_peer_transport_multi_process_bitwise(world):
    """world 3: the middle rank has two remote neighbours (distinct ranks)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.join(ROOT, "tests", "peer_worker.py")]
    env = dict(os.environ, OMP_NUM_THREADS="1")
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    out = p.stdout + p.stderr
    assert p.returncode == 0, out[-6000:]
    assert out.count("PEER_OK") == world, out[-6000:]
