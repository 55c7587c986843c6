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


# ---- schedule robustness:
# the halo and reduction protocol is ordered by flags / events only, so a
# delay injected anywhere on either side must leave every result bitwise
# equal (NB_DELAY_* knobs, csrc/nb_peer.cu) --------------------------------
DELAYS = [
    # (world, where, rank, jitter): producer-side delay before the halo signal
    (2, 1, 0, 0),
    # consumer-side delay after the halo wait (tests the WAR ping-pong)
    (2, 2, 1, 0),
    # the middle rank of three delays its reduction flags and its halo copies
    (3, 4 | 8, 1, 0),
    # every injection point on every rank, jittered
    (3, 15, -1, 1),
]


@pytest.mark.parametrize("world,where,rank,jitter", DELAYS)
def test_peer_transport_with_injected_delays_bitwise(world, where, rank, jitter):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.join(ROOT, "tests", "peer_worker.py")]
    env = dict(os.environ, OMP_NUM_THREADS="1", NB_DELAY_US="150", NB_DELAY_WHERE=str(where),
               NB_DELAY_RANK=str(rank), NB_DELAY_JITTER=str(jitter))
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    out = p.stdout + p.stderr
    assert p.returncode == 0, out[-6000:]
    assert out.count("PEER_OK") == world, out[-6000:]


def test_halo_stream_with_delayed_copies_bitwise():
    """One process, NB_HALO_STREAM: the batched halo copies on the halo
    stream start 300 us late; the events that order them against the
    interior / boundary kernels must keep every result bitwise equal to the
    fused stores (the parity test, rerun under the delay)."""
    env = dict(os.environ, NB_DELAY_US="300", NB_DELAY_WHERE="8")
    cmd = [sys.executable, "-m", "pytest", "-q", "-m", "gpu", "-p", "no:cacheprovider",
           os.path.join(ROOT, "tests", "test_gpu_parity.py") + "::test_halo_stream_mode_bitwise_equals_fused",
           os.path.join(ROOT, "tests", "test_gpu_parity.py") +
           "::test_lbm_halo_stream_many_partitions_bitwise_equals_fused"]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, (p.stdout + p.stderr)[-6000:]
    assert "2 passed" in p.stdout, p.stdout[-3000:]


@pytest.mark.parametrize("world", [2])
def test_nccl_transport_multi_process_bitwise(world):
    """The NCCL transport (include/nb.h nb_comm_create: grouped ncclSend /
    ncclRecv halos on the halo stream, ncclAllReduce of zero-padded plane
    sums) on the same cases, bitwise equal to one process.  NCCL refuses
    two ranks on one GPU, so this needs one visible device per rank."""
    if nb.nb_device_count() < world:
        pytest.skip(f"NCCL transport needs {world} GPUs (one per rank); {nb.nb_device_count()} visible")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.join(ROOT, "tests", "peer_worker.py")]
    env = dict(os.environ, OMP_NUM_THREADS="1", NB_TRANSPORT="nccl")
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    out = p.stdout + p.stderr
    assert p.returncode == 0, out[-6000:]
    assert out.count("PEER_OK") == world, out[-6000:]
