"""Multi-process (N > 1) host logic on CPU: world-size-2 `gloo` process groups.

The GPU path runs one process per GPU and moves halo planes with NCCL
send/recv in the order `nb_halo_plan` (product host code, C ABI) prescribes,
and combines reductions by an all-reduce of zero-padded per-plane sums
followed by a fixed-order total.  These tests execute exactly
that plan and protocol with gloo on numpy slabs and check (a) every send is
matched by the peer's receive in order, (b) the halos equal the neighbours'
planes, (c) a stencil over the exchanged slabs equals the undecomposed one,
(d) the reduction is bit-identical on every rank and to one process."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_ipps_meneghinmjm22_b200 as nb


@pytest.fixture(scope="module", autouse=True)
def _built():
    import __graft_entry__
    __graft_entry__.build()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(fn, world, *args):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, fn, args, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get() for _ in procs]
    for p in procs:
        p.join(60)
    errs = [r for r in res if isinstance(r, str)]
    assert not errs, errs
    return res


def _worker(rank, world, port, fn, args, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        q.put(fn(rank, world, *args))
        dist.destroy_process_group()
    except Exception as e:  # report to the parent
        import traceback
        q.put(f"rank {rank}: {e!r}\n{traceback.format_exc()}")


def lap_numpy(u, halo_lo, halo_hi):
    """7-point Laplacian of a slab [nz][ny][nx] given its two halo planes
    (test-side stand-in for the GPU kernel; outside value 0 in x/y)."""
    ext = np.concatenate([halo_lo[None], u, halo_hi[None]])
    p = np.pad(ext, ((0, 0), (1, 1), (1, 1)))
    c = p[1:-1, 1:-1, 1:-1]
    s = p[1:-1, 1:-1, :-2] + p[1:-1, 1:-1, 2:]
    s = s + p[1:-1, :-2, 1:-1]
    s = s + p[1:-1, 2:, 1:-1]
    s = s + p[:-2, 1:-1, 1:-1]
    s = s + p[2:, 1:-1, 1:-1]
    return s - 6.0 * c


# ---- (a) plan consistency ---------------------------------------------------
def _plans(rank, world, nz, nparts, periodic):
    return nb.nb_halo_plan(nz, nparts, world, rank, periodic)


@pytest.mark.parametrize("nparts,periodic", [(2, True), (4, False), (6, True)])
def test_plan_sends_match_receives_in_order(nparts, periodic):
    world = 2
    plans = _run(_plans, world, 40, nparts, periodic)
    for a in range(world):
        for b in range(world):
            if a == b:
                continue
            sent = [(m["src_part"], m["dst_part"], m["up"]) for m in plans[a]
                    if m["src_rank"] == a and m["dst_rank"] == b]
            recv = [(m["src_part"], m["dst_part"], m["up"]) for m in plans[b]
                    if m["src_rank"] == a and m["dst_rank"] == b]
            assert sent == recv and len(sent) > 0


@pytest.mark.parametrize("world,nparts", [(1, 1), (1, 4), (2, 4), (4, 4), (4, 8), (8, 8)])
@pytest.mark.parametrize("periodic", [False, True])
def test_plan_all_ranks_consistent(world, nparts, periodic):
    allm = nb.nb_halo_plan(64, nparts, world, -1, periodic)
    npairs = nparts if periodic else nparts - 1
    assert len(allm) == 2 * npairs
    for r in range(world):
        mine = nb.nb_halo_plan(64, nparts, world, r, periodic)
        assert mine == [m for m in allm if r in (m["src_rank"], m["dst_rank"])]
    for a in range(world):
        for b in range(world):
            seq_a = [m for m in nb.nb_halo_plan(64, nparts, world, a, periodic)
                     if m["src_rank"] == a and m["dst_rank"] == b]
            seq_b = [m for m in nb.nb_halo_plan(64, nparts, world, b, periodic)
                     if m["src_rank"] == a and m["dst_rank"] == b]
            assert seq_a == seq_b


# ---- (b, c) executing the plan: halos and stencil -------------------------------
def _exchange_and_stencil(rank, world, dims, nparts, periodic):
    import synth
    nx, ny, nz = dims
    glob = synth.uniform(dims, seed=5)
    zb = nb.nb_partition_plan(nz, nparts)
    k = nparts // world
    mine = range(rank * k, (rank + 1) * k)
    slabs = {p: glob[zb[p]:zb[p + 1]].copy() for p in mine}
    halo = {p: [np.zeros((ny, nx)), np.zeros((ny, nx))] for p in mine}  # [low, high], outside = 0
    reqs = []
    for m in nb.nb_halo_plan(nz, nparts, world, rank, periodic):
        src_plane = m["src_plane"]
        if m["src_rank"] == rank and m["dst_rank"] == rank:
            halo[m["dst_part"]][0 if m["up"] else 1] = slabs[m["src_part"]][src_plane].copy()
        elif m["src_rank"] == rank:
            reqs.append(dist.isend(torch.from_numpy(slabs[m["src_part"]][src_plane].copy()), m["dst_rank"]))
        else:
            buf = torch.empty((ny, nx), dtype=torch.float64)
            dist.recv(buf, m["src_rank"])
            halo[m["dst_part"]][0 if m["up"] else 1] = buf.numpy()
    for r in reqs:
        r.wait()
    out = {}
    for p in mine:
        lo_ref = glob[zb[p] - 1] if zb[p] > 0 else (glob[-1] if periodic else np.zeros((ny, nx)))
        hi_ref = glob[zb[p + 1]] if zb[p + 1] < nz else (glob[0] if periodic else np.zeros((ny, nx)))
        assert np.array_equal(halo[p][0], lo_ref) and np.array_equal(halo[p][1], hi_ref), p
        out[p] = lap_numpy(slabs[p], halo[p][0], halo[p][1])
    return {p: v.tolist() for p, v in out.items()}


@pytest.mark.parametrize("nparts,periodic", [(2, False), (4, True)])
def test_plan_exchange_reproduces_global_stencil(nparts, periodic):
    import synth
    dims = (9, 7, 21)
    res = _run(_exchange_and_stencil, 2, dims, nparts, periodic)
    parts = {}
    for r in res:
        parts.update({int(k): np.array(v) for k, v in r.items()})
    got = np.concatenate([parts[p] for p in range(nparts)])
    glob = synth.uniform(dims, seed=5)
    if periodic:
        ref = lap_numpy(glob, glob[-1], glob[0])
    else:
        ref = lap_numpy(glob, np.zeros(glob.shape[1:]), np.zeros(glob.shape[1:]))
    assert np.array_equal(got, ref)


# ---- (d) deterministic cross-rank reduction ----------------------------------
def _tree(v):
    """Fixed 256-wide block tree of DESIGN.md §6 (host mirror for the test)."""
    acc = np.zeros(256)
    for t in range(256):
        s = 0.0
        for i in range(t, len(v), 256):
            s = s + v[i]
        acc[t] = s
    w = 128
    while w:
        acc[:w] = acc[:w] + acc[w:2 * w]
        w //= 2
    return acc[0]


def _reduce(rank, world, nz, nparts):
    import synth
    x = synth.uniform((16, 8, nz), seed=3)
    zb = nb.nb_partition_plan(nz, nparts)
    k = nparts // world
    send = np.zeros(nz)
    for p in range(rank * k, (rank + 1) * k):
        for z in range(zb[p], zb[p + 1]):
            send[z] = _tree((x[z] * x[z]).ravel())
    t = torch.from_numpy(send)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(_tree(t.numpy()))


@pytest.mark.parametrize("nparts", [4])
def test_reduction_protocol_bitwise(nparts):
    nz = 12
    vals = _run(_reduce, 2, nz, nparts)
    single = _run(_reduce, 1, nz, nparts)[0]
    assert vals[0] == vals[1] == single
