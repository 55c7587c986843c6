#!/usr/bin/env python
"""bench.py — headline benchmark of the B200 Neon map-stencil hot path.

Default workload (BASELINE.json configs[1], the config the metric is quoted
on): Poisson finite-difference CG, 7-point, fp64, 512^3 dense grid, strong
scaling over N GPUs (one process per GPU, torchrun).  One "step" is one full
CG iteration (UpdateP, stencil, <p,q>, x/r updates, <r,r>; DESIGN.md "CG
schedule").  value = MLUPS = cells * steps / t / 1e6 over the whole job.

The same JSON line carries, at N = 1, the D3Q19 LBM cavity (configs[2],
512^3 fp32) and the config-C1 loop (configs[0]) results under "also".

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl nb|reference]
                  [--workload cg|lbm] [--n 512]

--impl reference times the CPU oracle (oracle/, plain C fp64) on the host
cores — the tier's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MLUPS & HBM GB/s (% roofline) at 1/2/4/8 B200; weak/strong scaling eff."
CG_BYTES_PER_CELL = 64      # 2-phase schedule, DESIGN.md "CG schedule"
CG_A_BYTES = 40             # phase A: read x, r, p_old; write x, p_new
CG_B_BYTES = 24             # phase B: read r, p_new; write r
LBM_BYTES_PER_CELL = 152    # 19 x (4 B read + 4 B write)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu, self.rows, self.proc, self.start = gpu, [], None, 0

    def mark(self):
        """Samples from here on belong to the timed region."""
        self.start = len(self.rows)

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        rows = self.rows[self.start:] or self.rows[-1:]  # the timed region (at least the last sample)
        sm = [float(r[1]) for r in rows if len(r) > 8 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) > 8 and r[2].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            if len(r) > 8:
                for nm, v in zip(names, r[5:9]):
                    if v.strip().lower() == "active":
                        reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------
def setup_dist(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import torch
    # one process per GPU; if there are fewer GPUs than local ranks (a
    # single-GPU box exercising the multi-process path) ranks share GPUs and
    # the timing plumbing uses gloo (NCCL refuses two ranks on one GPU)
    ndev = max(torch.cuda.device_count(), 1)
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    global _SHARED_GPU
    _SHARED_GPU = local_world > ndev
    local = local % ndev
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if _SHARED_GPU:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return world, rank, local


_SHARED_GPU = False


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(world, v):
    if world == 1:
        return v
    import torch
    import torch.distributed as dist
    t = torch.tensor([v], dtype=torch.float64, device="cpu" if _SHARED_GPU else "cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def timed(world, stream, fn, gpu):
    """Barrier + sync on both sides; CUDA events on the launching stream.  The
    clock sampler (nvidia-smi) is started first and given time to initialise
    (NVML start-up holds driver locks that would otherwise stall this
    process's enqueues inside the timed region)."""
    import torch
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(gpu) as clk:
        t0 = time.perf_counter()
        while not clk.rows and time.perf_counter() - t0 < 3.0:
            time.sleep(0.02)
        barrier(world)
        torch.cuda.synchronize()
        clk.mark()
        ev0.record(stream)
        fn()
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier(world)
    ms = ev0.elapsed_time(ev1)
    return max_over_ranks(world, ms), clk.summary()


def ncu_traffic(kernel: str):
    """dram bytes per launch of `kernel` from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    return d.get(kernel)


# ---------------------------------------------------------------------------
def comm_profile(g, iters):
    """Per-iteration device time of the communication kernels from a profiled
    (event-bracketed, eager) pass: reductions (k_finalize: plane sums, the
    cross-rank exchange of the peer transport, alpha / beta) and halo
    signalling / waiting (k_peer_*) or batched halo copies (k_halo_copy).
    The halo planes themselves are stored by the boundary kernels (fused
    transport), so their bytes are inside the compute kernels' time."""
    out = {}
    for key, name in (("reduction", "k_finalize"), ("halo_sync", "k_peer_"), ("halo_copy", "k_halo_copy")):
        k, ms = g.profile_read(name)
        out[key + "_ms_per_iter"] = ms / max(iters, 1)
        out[key + "_launches_per_iter"] = k / max(iters, 1)
    return out


def bench_cg(args, world, rank, local, weak=False, with_e2e=True):
    """C2 Poisson CG.  Strong scaling: the n^3 grid split over `world` ranks;
    weak: n x n x (n * world), an n^3 slab per rank."""
    import numpy as np
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    n = args.n
    dims = (n, n, n * world) if weak else (n, n, n)
    cells = dims[0] * dims[1] * dims[2]
    steps = args.steps
    comm = nb.Comm.from_torch_distributed(local) if world > 1 else None
    g = nb.Grid(dims, nparts=world, comm=comm) if comm else nb.Grid(dims, nparts=1, devices=[local])
    stream = torch.cuda.ExternalStream(g.stream())
    b, x = nb.Field(g), nb.Field(g)
    if weak:  # POISSON_RHS needs a cube: a seeded uniform right-hand side
        b.fill_uniform(seed=2)
    else:
        b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0)
    occ = nb.OCC_NAMES[args.occ]
    cg = nb.CG(x, b, occ=occ)
    cg.iterate(args.warmup)
    cg.prepare(steps)  # graph instantiation outside the timed region
    g.sync()
    l0 = g.launch_count()
    ms, clocks = timed(world, stream, lambda: cg.iterate(steps), local)
    launches = g.launch_count() - l0
    res = cg.finish()
    cg.close()
    t = ms / 1e3
    mlups = cells * steps / t / 1e6
    hbm, peak_kind = peaks()
    # per-kernel durations: a profiled (event-bracketed, eager) pass; the
    # roofline divides one iteration's algorithmic bytes by the SUM of that
    # kernel's launches in one iteration (at N > 1 phase A is an interior
    # launch plus boundary-plane launches)
    x.fill_const(0.0)
    cg = nb.CG(x, b, occ=occ)
    cg.iterate(1)
    g.profile(True)
    it = args.prof_steps
    cg.iterate(it)
    na, msa = g.profile_read("k_msr_cgA")
    nbb, msb = g.profile_read("k_cg_B")
    comm_t = comm_profile(g, it)
    g.profile(False)
    cg.finish()
    cg.close()
    local_cells = cells // world
    a_it, b_it = msa / it, msb / it
    dom = ("k_msr_cgA", CG_A_BYTES, a_it, na / it) if msa >= msb else ("k_cg_B", CG_B_BYTES, b_it, nbb / it)
    achieved = dom[1] * local_cells / (dom[2] / 1e3) / 1e9
    tr = ncu_traffic(dom[0])
    kind = "weak" if weak else "strong"
    out = {
        "metric": METRIC, "value": mlups, "unit": "MLUPS", "n_gpus": world, "steps": steps,
        "warmup": args.warmup, "ms_per_step": ms / steps, "higher_is_better": True, "scaling": kind,
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": (f"C2 Poisson FD CG 7-point fp64 {n}^3 per GPU, weak scaling "
                                f"({dims[0]}x{dims[1]}x{dims[2]})" if weak else
                                f"C2 Poisson FD CG 7-point fp64 {n}^3 dense (configs[1])"),
                   "rhs": "uniform[-1,1) seed 2" if weak else "b = h^2 f, manufactured u* = g(x)g(y)g(z)",
                   "x0": 0, "parts": world, "occ": args.occ, "schedule": "2-phase, 64 B/cell/iter",
                   "l2": "inputs larger than L2 (5 fp64 fields of %.2f GB per GPU)" % (local_cells * 8 / 1e9)},
        "hbm_gbs": CG_BYTES_PER_CELL * cells * steps / t / 1e9,
        "hbm_frac": CG_BYTES_PER_CELL * cells * steps / t / 1e9 / hbm / world,
        "roofline": {"bound": "hbm", "kernel": dom[0], "achieved": achieved, "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "peak_kind": peak_kind, "traffic": tr,
                     "algorithmic_bytes_per_iter": dom[1] * local_cells,
                     "kernel_ms_per_iter": dom[2], "launches_per_iter": dom[3],
                     "per_rank": world > 1,
                     "kernel_ms": {"k_msr_cgA": a_it, "k_cg_B": b_it}},
        "comm": comm_t,
        "gpu_launches": int(launches), "clocks": clocks,
        "cg_state": {"iters": res.iters, "rr0": res.rr0, "rr": res.rr},
    }
    if _SHARED_GPU:
        out["note"] = SHARED_NOTE
    if with_e2e:
        # ---- e2e: public API, host buffers, H2D and D2H inside the timed
        # region (every rank holds the dense host logical view;
        # nb_field_upload / download move only its own slab)
        import synth
        bh = torch.from_numpy(synth.poisson_poly_rhs(dims).reshape(-1)).pin_memory()
        xh = torch.zeros(cells, dtype=torch.float64).pin_memory()
        local_bytes = cells * 8 // world

        def e2e():
            b.upload_async(bh.data_ptr())
            x.upload_async(xh.data_ptr())
            s = nb.CG(x, b, occ=occ)
            s.prepare(steps)
            s.iterate(steps)
            s.finish()
            s.close()
            x.download(xh)
        e2e()  # warm
        ms_e, _ = timed(world, stream, e2e, local)
        out["e2e"] = {"value": cells * steps / (ms_e / 1e3) / 1e6, "unit": "MLUPS",
                      "h2d_bytes_per_step": 2 * local_bytes / steps, "d2h_bytes_per_step": local_bytes / steps,
                      "h2d_bytes_per_call": 2 * local_bytes, "d2h_bytes_per_call": local_bytes,
                      "note": "per rank: upload b and x0 (own slab) from pinned host, CG create (r = b - Ax0), "
                              "steps iterations, finish (deferred x update), download x (own slab); "
                              "one e2e call (a whole solve of `steps` iterations) per timed region, max over "
                              "ranks; bytes per step = bytes per call / steps"}
    b.close(), x.close()
    g.close()
    if comm:
        comm.close()
    return out


SHARED_NOTE = ("ranks share one GPU (fewer GPUs than ranks): kernels of different ranks overlap and the "
               "peer-flag waits spin, so per-kernel times, communication times and the roofline are not "
               "meaningful here")


def lbm_omega(nx, u_lid=0.05, re=100.0):
    """Cavity set-up (SURVEY.md §8(c) c6 reading): nu = u_lid Nx / Re."""
    nu = u_lid * nx / re
    return 1.0 / (3.0 * nu + 0.5)


def bench_lbm_layouts(n, steps, local):
    """SURVEY f3 / PAPER L248: the C3 twoPop step with the populations in
    each field layout (SoA, plane-major SoA, AoS), 1 GPU, same bits."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    hbm, peak_kind = peaks()
    rows = {}
    for name, layout in (("soa", nb.SOA), ("soa_plane", nb.SOA_PLANE), ("aos", nb.AOS)):
        g = nb.Grid((n, n, n), devices=[local])
        stream = torch.cuda.ExternalStream(g.stream())
        st = {"a": nb.Field(g, "f32", 19, layout=layout), "b": nb.Field(g, "f32", 19, layout=layout)}
        nb.nb_lbm_init(st["a"], 1.0, (0.0, 0.0, 0.0))
        om = lbm_omega(n)

        def run(k):
            st["a"], st["b"] = nb.nb_lbm_step(st["a"], st["b"], om, k)
        run(3)
        g.sync()
        ms, clocks = timed(1, stream, lambda: run(steps), local)
        gbs = LBM_BYTES_PER_CELL * n ** 3 * steps / (ms / 1e3) / 1e9
        rows[name] = {"mlups": n ** 3 * steps / (ms / 1e3) / 1e6, "ms_per_step": ms / steps, "hbm_gbs": gbs,
                      "hbm_frac": gbs / hbm, "clocks": clocks}
        st["a"].close(), st["b"].close()
        g.close()
    return {"workload": f"C3 D3Q19 cavity {n}^3 fp32 twoPop, populations as SoA [c][z][y][x], plane-major SoA "
                        "[z][c][y][x] and AoS [z][y][x][c] (PAPER L248; bitwise equal results)",
            "rows": rows, "peak_kind": peak_kind}


def bench_lbm_run(n, steps, warmup, world, local, occ="standard"):
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    dims = (n, n, n * world)  # weak scaling: 512^3 per GPU
    comm = nb.Comm.from_torch_distributed(local) if world > 1 else None
    g = nb.Grid(dims, nparts=world, comm=comm) if comm else nb.Grid(dims, nparts=1, devices=[local])
    stream = torch.cuda.ExternalStream(g.stream())
    fa, fb = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(fa, 1.0, (0.0, 0.0, 0.0))
    om = lbm_omega(n)
    st = {"a": fa, "b": fb}

    def run(k):
        st["a"], st["b"] = nb.nb_lbm_step(st["a"], st["b"], om, k, u_lid=0.05, occ=nb.OCC_NAMES[occ])
    run(warmup)
    g.sync()
    l0 = g.launch_count()
    ms, clocks = timed(world, stream, lambda: run(steps), local)
    launches = g.launch_count() - l0
    g.profile(True)
    run(3)
    nk, msk = g.profile_read("k_lbm_d3q19")
    comm_t = comm_profile(g, 3)
    g.profile(False)
    cells = n * n * n * world
    t = ms / 1e3
    hbm, peak_kind = peaks()
    local_cells = n * n * n
    # per step: the sum of the step's launches (boundary planes + interior
    # under Standard OCC at N > 1; one launch at N = 1)
    per_step_ms = msk / 3.0
    achieved = LBM_BYTES_PER_CELL * local_cells / (per_step_ms / 1e3) / 1e9
    res = {
        "value": cells * steps / t / 1e6, "unit": "MLUPS", "n_gpus": world, "steps": steps, "warmup": warmup,
        "ms_per_step": ms / steps, "scaling": "weak", "dtype": "f32",
        "config": {"workload": f"C3 D3Q19 BGK lid-driven cavity fp32 SoA twoPop, {n}^3 per GPU (configs[2])",
                   "omega": om, "u_lid": 0.05, "Re": 100, "occ": occ,
                   "l2": "inputs larger than L2 (2 x %.1f GB)" % (19 * 4 * n ** 3 / 1e9)},
        "hbm_gbs": LBM_BYTES_PER_CELL * cells * steps / t / 1e9,
        "hbm_frac": LBM_BYTES_PER_CELL * cells * steps / t / 1e9 / hbm,
        "roofline": {"bound": "hbm", "kernel": "k_lbm_d3q19", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "peak_kind": peak_kind, "traffic": ncu_traffic("k_lbm_d3q19"),
                     "algorithmic_bytes_per_step": LBM_BYTES_PER_CELL * local_cells,
                     "kernel_ms_per_step": per_step_ms, "launches_per_step": nk / 3.0, "per_rank": world > 1},
        "comm": comm_t,
        "gpu_launches": int(launches), "clocks": clocks,
    }
    if _SHARED_GPU:
        res["note"] = SHARED_NOTE
    st["a"].close(), st["b"].close()
    g.close()
    if comm:
        comm.close()
    return res


def bench_lbm_aa_run(n, steps, warmup, local):
    """the AA pattern — the C3 cavity on ONE population buffer
    updated in place (half of twoPop's memory), 1 GPU."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    g = nb.Grid((n, n, n), devices=[local])
    stream = torch.cuda.ExternalStream(g.stream())
    f = nb.Field(g, "f32", 19)
    nb.nb_lbm_init(f, 1.0, (0.0, 0.0, 0.0))
    om = lbm_omega(n)
    nb.nb_lbm_step_aa(f, om, warmup + (warmup & 1))
    g.sync()
    steps += steps & 1
    ms, clocks = timed(1, stream, lambda: nb.nb_lbm_step_aa(f, om, steps), local)
    hbm, peak_kind = peaks()
    cells = n ** 3
    gbs = LBM_BYTES_PER_CELL * cells * steps / (ms / 1e3) / 1e9
    f.close()
    g.close()
    return {"workload": f"C3 D3Q19 cavity {n}^3 fp32, AA pattern (one in-place buffer, {19 * 4 * n ** 3 / 1e9:.1f} GB "
                        f"instead of {2 * 19 * 4 * n ** 3 / 1e9:.1f} GB) (SURVEY f3)",
            "value": cells * steps / (ms / 1e3) / 1e6, "unit": "MLUPS", "ms_per_step": ms / steps,
            "hbm_gbs": gbs, "hbm_frac": gbs / hbm, "peak_kind": peak_kind, "clocks": clocks}


def bench_karman(local, steps=20):
    """the 2-D Kármán vortex street of PAPER.md Table I (D2Q9,
    fp32, 72 B/cell/step) at the table's four domain sizes, 1 GPU."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    hbm, peak_kind = peaks()
    rows = []
    for nx, ny in ((4096, 1024), (8192, 2048), (16384, 4096), (32768, 8192)):
        g = nb.Grid((nx, ny, 1), devices=[local])
        stream = torch.cuda.ExternalStream(g.stream())
        st = {"a": nb.Field(g, "f32", 9), "b": nb.Field(g, "f32", 9)}
        u = 0.08
        cyl = (nx // 5, ny // 2, ny // 10)
        omega = 1.0 / (3 * u * 2 * cyl[2] / 150.0 + 0.5)  # Re 150 on the diameter
        nb.nb_d2q9_init(st["a"], 1.0, u, 0.0)

        def run(k):
            st["a"], st["b"] = nb.nb_d2q9_step(st["a"], st["b"], omega, u, cyl, k)
        run(4)
        g.sync()
        ms, _ = timed(1, stream, lambda: run(steps), local)
        cells = nx * ny
        gbs = 72 * cells * steps / (ms / 1e3) / 1e9
        rows.append({"domain": f"{nx}x{ny}", "mlups": cells * steps / (ms / 1e3) / 1e6, "ms_per_step": ms / steps,
                     "hbm_gbs": gbs, "hbm_frac": gbs / hbm})
        st["a"].close(), st["b"].close()
        g.close()
    return {"workload": "2-D Karman vortex street, D2Q9 BGK fp32, cylinder r = ny/10 at (nx/5, ny/2), Re 150 "
                        "(PAPER.md Table I sizes; SURVEY f4)", "rows": rows, "peak_kind": peak_kind,
            "paper_context": "Table I reports 33-206 'LUPS' on 1 A100 (units garbled in the extraction; context only)"}


LBM_SPARSE_BYTES_PER_CELL = 152 + 18 * 4  # 19 loads + 19 stores fp32, + the 18-direction source table


def bench_lbm_sparse_run(n, steps, warmup, local):
    """D3Q19 on an element-sparse domain — the C4 sphere (30 % of
    the n^3 box) as the fluid region, bounce-back on its surface, 1 GPU."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    import synth
    m = synth.sphere_mask(n)
    g = nb.Grid((n, n, n), devices=[local], active=m)
    active = int(m.sum(dtype="int64"))
    stream = torch.cuda.ExternalStream(g.stream())
    st = {"a": nb.Field(g, "f32", 19), "b": nb.Field(g, "f32", 19)}
    nb.nb_lbm_init(st["a"], 1.0, (0.01, 0.0, 0.0))
    om = lbm_omega(n)

    def run(k):
        st["a"], st["b"] = nb.nb_lbm_step(st["a"], st["b"], om, k)
    run(warmup)
    g.sync()
    ms, clocks = timed(1, stream, lambda: run(steps), local)
    g.profile(True)
    run(3)
    nk, msk = g.profile_read("k_sp_lbm")
    g.profile(False)
    hbm, peak_kind = peaks()
    k_ms = msk / max(nk, 1)
    achieved = LBM_SPARSE_BYTES_PER_CELL * active / (k_ms / 1e3) / 1e9
    st["a"].close(), st["b"].close()
    g.close()
    return {"workload": f"D3Q19 BGK on the element-sparse sphere ({active} active cells of {n}^3, 30 %), fp32, "
                        "bounce-back at the surface (SURVEY f2)",
            "value": active * steps / (ms / 1e3) / 1e6, "unit": "MLUPS (active cells)", "ms_per_step": ms / steps,
            "roofline": {"bound": "hbm", "kernel": "k_sp_lbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "peak_kind": peak_kind,
                         "algorithmic_bytes_per_cell": LBM_SPARSE_BYTES_PER_CELL, "launch_ms": k_ms},
            "clocks": clocks}


# per active cell: map reads r, p_old, x and writes x, p (40 B); q reads p and
# the 16-byte segment-indexed neighbour entry and writes q (32 B; the six
# neighbour values are cache hits of the same p stream); r reads q, r and
# writes r (24 B)
SPARSE_BYTES = {"k_sp_cg_map": 40, "k_sp_cg_q": 32, "k_sp_cg_r": 24}
# fused FEM CG schedule, per node of 3 fp64 components:
# phase A reads x, r, p_old, writes x, p_new, q; phase B reads r, q, writes r
FEM_BYTES = {"k_fem_cg_a": 144, "k_fem_r": 72}
FEM_FLOPS_PER_NODE = 306  # 153 nonzero stencil coefficients x 2
FP64_PEAK_DERIVED = 148 * 64 * 2 * 1.965e9 / 1e12  # SMs x FP64 lanes x 2 x max clock


def fp64_peak():
    """Measured FP64 FMA throughput (tools/fp64_peak.cu, profiles/fp64_peak_r1.jsonl),
    else the derived unit-count figure."""
    p = os.path.join(ROOT, "profiles", "fp64_peak_r1.jsonl")
    if os.path.exists(p):
        v = max(json.loads(line)["fp64_tflops"] for line in open(p) if line.strip())
        return v, "measured: tools/fp64_peak.cu (DFMA chains, all SMs), profiles/fp64_peak_r1.jsonl"
    return FP64_PEAK_DERIVED, "derived: 148 SMs x 64 FP64 lanes x 2 flop x 1.965 GHz"


def _profiled_kernels(g, run, names, comm_iters=0):
    g.profile(True)
    run()
    out = {}
    for nm in names:
        k, ms = g.profile_read(nm)
        out[nm] = (k, ms)
    if comm_iters:
        out["comm"] = comm_profile(g, comm_iters)
    g.profile(False)
    return out


def bench_sparse_run(n, steps, warmup, world, local):
    """C4 (configs[3]): element-sparse sphere (~30 % of the n^3 box), 7-point
    CG fp64, active-balanced z cuts."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    import synth
    mask = synth.sphere_mask(n)
    nact = int(mask.sum(dtype="int64"))
    comm = nb.Comm.from_torch_distributed(local) if world > 1 else None
    g = nb.Grid((n, n, n), nparts=world, comm=comm, active=mask) if comm else \
        nb.Grid((n, n, n), nparts=1, devices=[local], active=mask)
    stream = torch.cuda.ExternalStream(g.stream())
    b, x = nb.Field(g), nb.Field(g)
    b.fill_uniform(seed=4)
    x.fill_const(0.0)
    cg = nb.CG(x, b)
    cg.iterate(warmup)
    cg.prepare(steps)
    g.sync()
    l0 = g.launch_count()
    ms, clocks = timed(world, stream, lambda: cg.iterate(steps), local)
    launches = g.launch_count() - l0
    cg.finish()
    cg.close()
    x.fill_const(0.0)
    cg = nb.CG(x, b)
    cg.iterate(1)
    pit = 5
    prof = _profiled_kernels(g, lambda: cg.iterate(pit), list(SPARSE_BYTES), comm_iters=pit)
    comm_t = prof.pop("comm")
    cg.finish()
    cg.close()
    hbm, peak_kind = peaks()
    t = ms / 1e3
    local_act = nact // world
    dom = max(prof, key=lambda k: prof[k][1])
    dk, dms = prof[dom]
    achieved = SPARSE_BYTES[dom] * local_act / (dms / pit / 1e3) / 1e9
    b.close(), x.close()
    g.close()
    if comm:
        comm.close()
    per_cell = sum(SPARSE_BYTES.values())
    return {"value": nact * steps / t / 1e6, "unit": "MLUPS (active cells)", "n_gpus": world, "steps": steps,
            "ms_per_step": ms / steps, "scaling": "strong", "dtype": "f64",
            "config": {"workload": f"C4 element-sparse sphere r=0.41528N in {n}^3 ({nact} active, "
                                   f"{nact / n ** 3:.2%}), 7-point CG fp64 (configs[3])",
                       "schedule": f"3 passes, {per_cell} B/active cell/iter incl. the 16 B segment-indexed neighbour table"},
            "hbm_gbs": per_cell * nact * steps / t / 1e9, "hbm_frac": per_cell * nact * steps / t / 1e9 / hbm,
            # 96 B/active/iter is the minimum of a 24-B
            # connectivity schedule; the iteration time against it
            "survey_96B_frac": 96 * nact * steps / t / 1e9 / hbm / world,
            "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "peak_kind": peak_kind, "traffic": ncu_traffic(dom),
                         "per_rank": world > 1, "local_active_cells": local_act,
                         "kernel_ms_per_iter": {k: v[1] / pit for k, v in prof.items()},
                         "launches_per_iter": {k: v[0] / pit for k, v in prof.items()}},
            "comm": comm_t, "gpu_launches": int(launches), "clocks": clocks,
            **({"note": SHARED_NOTE} if _SHARED_GPU else {})}


def bench_fem_run(n, steps, warmup, world, local):
    """C5 (configs[4]): matrix-free Q1 linear-elastic CG on n^3 nodes x 3 fp64
    (fused schedule: surface nodes + phase A, then phase B)."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    comm = nb.Comm.from_torch_distributed(local) if world > 1 else None
    dims = (n, n, n)
    g = nb.Grid(dims, nparts=world, comm=comm) if comm else nb.Grid(dims, nparts=1, devices=[local])
    stream = torch.cuda.ExternalStream(g.stream())
    b, x = nb.Field(g, card=3), nb.Field(g, card=3)
    nb.nb_fem27_rhs(b, 1.0)
    x.fill_const(0.0)
    cg = nb.CG(x, b, op=nb.OP_FEM27)
    cg.iterate(warmup)
    cg.prepare(steps)
    g.sync()
    l0 = g.launch_count()
    ms, clocks = timed(world, stream, lambda: cg.iterate(steps), local)
    launches = g.launch_count() - l0
    cg.finish()
    cg.close()
    x.fill_const(0.0)
    # per-kernel times from the serial schedule (NB_FEM_CONC=0: same kernels,
    # same bits; the timed step runs the surface kernels concurrently with the
    # surface-free part of phase A, whose stream spans would overlap)
    conc_env = os.environ.get("NB_FEM_CONC")
    os.environ["NB_FEM_CONC"] = "0"
    cg = nb.CG(x, b, op=nb.OP_FEM27)
    cg.iterate(1)  # the first iteration has no deferred x update: profile steady-state ones
    pit = 5
    prof = _profiled_kernels(g, lambda: cg.iterate(pit), list(FEM_BYTES) + ["k_fem_surface"], comm_iters=pit)
    comm_t = prof.pop("comm")
    cg.finish()
    cg.close()
    # K u alone (nb_fem27_apply): the FP64-ALU-bound stencil kernel
    u, y = nb.Field(g, card=3), nb.Field(g, card=3)
    u.fill_uniform(seed=5)
    u.halo_update()
    nb.nb_fem27_apply(u, y, 1.0, 0.3)
    aprof = _profiled_kernels(g, lambda: [nb.nb_fem27_apply(u, y, 1.0, 0.3) for _ in range(5)], ["k_fem_apply"])
    if conc_env is None:
        os.environ.pop("NB_FEM_CONC", None)
    else:
        os.environ["NB_FEM_CONC"] = conc_env
    u.close(), y.close()
    hbm, peak_kind = peaks()
    f64, f64_kind = fp64_peak()
    t = ms / 1e3
    nodes = n ** 3
    local_nodes = nodes // world
    ak, ams = prof["k_fem_cg_a"]
    a_avg = ams / pit / 1e3  # per iteration (interior + boundary launches)
    achieved = FEM_BYTES["k_fem_cg_a"] * local_nodes / a_avg / 1e9
    qk, qms = aprof["k_fem_apply"]
    flops = FEM_FLOPS_PER_NODE * local_nodes / (qms / 5 / 1e3) / 1e12  # per nb_fem27_apply call
    per_node = sum(FEM_BYTES.values())
    b.close(), x.close()
    g.close()
    if comm:
        comm.close()
    return {"value": nodes * steps / t / 1e6, "unit": "MLUPS (nodes)", "n_gpus": world, "steps": steps,
            "ms_per_step": ms / steps, "scaling": "strong", "dtype": "f64",
            "config": {"workload": f"C5 FEM Q1 linear elastic CG, {n}^3 nodes x 3 fp64, E=1 nu=0.3, "
                                   "Dirichlet z=0, pressure 1 on z=N-1 (configs[4])",
                       "schedule": f"fused: surface nodes, phase A (p, x, q = K p, <p,q>), phase B; "
                                   f"{per_node} B/node/iter"},
            "hbm_gbs": per_node * nodes * steps / t / 1e9, "hbm_frac": per_node * nodes * steps / t / 1e9 / hbm,
            "roofline": {"bound": "hbm", "kernel": "k_fem_cg_a", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "peak_kind": peak_kind, "traffic": ncu_traffic("k_fem_cg_a"),
                         "algorithmic_bytes_per_node": FEM_BYTES["k_fem_cg_a"], "per_rank": world > 1,
                         "kernel_times": "serial schedule (NB_FEM_CONC=0); the timed step overlaps the "
                                         "surface kernels with phase A",
                         "kernel_ms_per_iter": {k: v[1] / pit for k, v in prof.items()},
                         "launches_per_iter": {k: v[0] / pit for k, v in prof.items()}},
            "apply_alu": {"bound": "alu", "kernel": "k_fem_apply (interior K u, surface nodes excluded)",
                          "achieved": flops, "peak": f64, "unit": "TFLOP/s", "frac": flops / f64,
                          "peak_kind": f64_kind, "flop_per_node": FEM_FLOPS_PER_NODE},
            "comm": comm_t, "gpu_launches": int(launches), "clocks": clocks,
            **({"note": SHARED_NOTE} if _SHARED_GPU else {})}


def bench_fem_sparse_run(n, steps, local):
    """f4: the C5 FEM CG on element-
    sparse grids at n^3 — the full cube (every node active: against the dense
    C5 line) and the C4-recipe sphere (~30 % of the box) — with the K p
    pass's FP64 roofline (box operator + list nodes, profiled serially)."""
    import numpy as np
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    import synth
    out = {"unit": "MLUPS (active nodes)", "n_gpus": 1, "steps": steps, "dtype": "f64", "scaling": "strong",
           "config": {"workload": f"f4 FEM Q1 linear elastic CG on element-sparse grids, {n}^3 box, 3 fp64 dof, "
                                  "E=1 nu=0.3, Dirichlet z=0, pressure on exposed top faces",
                      "schedule": "map 120 B + K p 48 B (box operator) + <p,q> 48 B + r 72 B per node"}}
    f64, f64_kind = fp64_peak()
    for name, mask in (("full_cube", np.ones((n, n, n), np.uint8)), ("sphere", synth.sphere_mask(n))):
        act = int(mask.sum(dtype="int64"))
        g = nb.Grid((n, n, n), nparts=1, devices=[local], active=mask)
        stream = torch.cuda.ExternalStream(g.stream())
        b, x = nb.Field(g, card=3), nb.Field(g, card=3)
        nb.nb_fem27_rhs(b, 1.0)
        x.fill_const(0.0)
        cg = nb.CG(x, b, op=nb.OP_FEM27)
        cg.iterate(3)
        cg.prepare(steps)
        g.sync()
        ms, clocks = timed(1, stream, lambda: cg.iterate(steps), local)
        os.environ["NB_SPF_SERIAL"] = "1"  # list nodes after the box kernel: separable kernel times
        pit = 3
        prof = _profiled_kernels(g, lambda: cg.iterate(pit), ["k_sp_fem_q", "k_sp_fem_dot", "k_sp_cg_map",
                                                                "k_sp_cg_r"])
        os.environ.pop("NB_SPF_SERIAL", None)
        cg.finish()
        cg.close(), b.close(), x.close(), g.close()
        kp = prof["k_sp_fem_q"][1] / pit
        out[name] = {"active_nodes": act, "value": act * steps / (ms / 1e3) / 1e6, "ms_per_step": ms / steps,
                     "kernel_ms_per_iter": {k: v[1] / pit for k, v in prof.items()},
                     "k_p_roofline": {"bound": "alu", "kernel": "k_sp_fem_box + k_sp_fem_list (q = K p)",
                                      "achieved": FEM_FLOPS_PER_NODE * act / (kp / 1e3) / 1e12, "peak": f64,
                                      "unit": "TFLOP/s",
                                      "frac": FEM_FLOPS_PER_NODE * act / (kp / 1e3) / 1e12 / f64,
                                      "peak_kind": f64_kind, "hbm_gbs_48B_per_node": 48 * act / (kp / 1e3) / 1e9},
                     "clocks": clocks}
    out["value"] = out["sphere"]["value"]
    out["ms_per_step"] = out["sphere"]["ms_per_step"]
    return out


def bench_c1(local):
    """Config C1 (64^3 fp64, 10 map-stencil-reduce iterations, 1 GPU): a
    launch/latency-bound case.  Timed per synchronous nb_map_stencil_reduce
    call (device events on the grid stream, and host wall clock)."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    n = 64
    g = nb.Grid((n, n, n), devices=[local])
    stream = torch.cuda.ExternalStream(g.stream())
    x, y = nb.Field(g), nb.Field(g)
    reps = 50

    def run():
        for _ in range(reps):
            nb.nb_map_stencil_reduce(x, y, 0.125, 10, nb.OCC_TWO_WAY)
    x.fill_int(seed=1)
    y.fill_const(0.0)
    run()
    g.sync()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    ev0.record(stream)
    run()
    ev1.record(stream)
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / reps
    dev = ev0.elapsed_time(ev1) / 1e3 / reps
    x.close(), y.close()
    g.close()
    return {"workload": "C1 AXPY + 7-pt + dot, 64^3 fp64, 10 iterations (configs[0])",
            "ms_per_loop": dev * 1e3, "wall_ms_per_loop": wall * 1e3, "value": n ** 3 * 10 / dev / 1e6,
            "unit": "MLUPS", "note": "per synchronous nb_map_stencil_reduce call (10 fused iterations + dots "
                                    "to host); latency-bound: 2 MB fields live in L2"}


def bench_skeleton(local, n=512, parts=4, iters=10):
    """the Skeleton's generated schedule (separate map / stencil /
    reduce containers, halo nodes, Two-way OCC, BFS streams + events) against
    the hand-written fused schedule of the same sequential code (the Fig. 4a
    loop), on `parts` virtual partitions; bit-identical results
    (test_gpu_skeleton.py), device time per iteration on the compute stream."""
    import torch

    import paper_conf_ipps_meneghinmjm22_b200 as nb
    g = nb.Grid((n, n, n), nparts=parts, devices=[local] * parts)
    stream = torch.cuda.ExternalStream(g.stream())
    x, y = nb.Field(g), nb.Field(g)
    x.fill_uniform(seed=1)
    y.fill_const(0.0)
    sk = nb.Skeleton(g, nb.OCC_TWO_WAY)
    for k in range(iters):
        sk.axpy(0.125, y, x)
        sk.laplace7(x, y)
        sk.dot(x, y, k)
    sk.compile()
    plan = sk.describe()

    def t(fn):
        fn()
        g.sync()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        fn()
        ev1.record(stream)
        torch.cuda.synchronize()
        return ev0.elapsed_time(ev1) / iters

    ms_sk = t(sk.run)
    ms_fused = t(lambda: nb.nb_map_stencil_reduce(x, y, 0.125, iters, nb.OCC_TWO_WAY))
    sk.close()
    # Listing 3 CG as containers with device scalars,
    # against the hand-fused 2-phase CG on the same grid (bitwise equal:
    # tests/test_gpu_skeleton.py)
    RR, PQ, AL, BE, RR2 = 0, 1, 2, 3, 4
    b, r, p, q = nb.Field(g), nb.Field(g), nb.Field(g), nb.Field(g)
    b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0), p.fill_const(0.0), q.fill_const(0.0)
    nb.nb_axpby(1.0, b, 0.0, r)
    with nb.Skeleton(g, nb.OCC_TWO_WAY) as s0:
        s0.dot(r, r, RR)
        s0.set_scalar(BE, 0.0)
        s0.run()
    cgk = nb.Skeleton(g, nb.OCC_TWO_WAY)
    cgk.axpby_s(1.0, -1, r, 1.0, BE, p)
    cgk.poisson(p, q)
    cgk.dot(p, q, PQ)
    cgk.scalar(nb.SC_DIV, RR, PQ, AL)
    cgk.axpby_s(1.0, AL, p, 1.0, -1, x)
    cgk.axpby_s(-1.0, AL, q, 1.0, -1, r)
    cgk.dot(r, r, RR2)
    cgk.scalar(nb.SC_DIV, RR2, RR, BE)
    cgk.scalar(nb.SC_COPY, RR2, 0, RR)
    cplan = cgk.describe()

    def run_cg_sk():
        for _ in range(iters):
            cgk.run()
    ms_cg_sk = t(run_cg_sk)
    cgk.close()
    x.fill_const(0.0)
    cg = nb.CG(x, b, occ=nb.OCC_TWO_WAY)
    cg.prepare(iters)
    ms_cg_fused = t(lambda: cg.iterate(iters))
    cg.close()
    for f in (b, r, p, q):
        f.close()
    x.close(), y.close()
    g.close()
    cells = n ** 3
    return {"workload": f"Fig. 4a loop (axpy, 7-pt, dot) x {iters}, {n}^3 fp64, {parts} partitions, Two-way OCC",
            "skeleton_ms_per_iter": ms_sk, "fused_ms_per_iter": ms_fused,
            "skeleton_gbs": 56 * cells / ms_sk / 1e6, "fused_gbs": 32 * cells / ms_fused / 1e6,
            "nodes": len(plan["nodes"]), "streams": plan["streams"], "events": plan["events"],
            "note": "skeleton = unfused containers (24 + 16 + 16 = 56 B/cell/iter), as Neon generates them; "
                    "fused = one kernel per iteration (32 B/cell/iter)",
            "listing3_cg": {"workload": f"Listing 3 CG (UpdateP first, device-scalar alpha / beta), {n}^3 fp64, "
                                        f"{parts} partitions, Two-way OCC",
                            "skeleton_ms_per_iter": ms_cg_sk, "fused_ms_per_iter": ms_cg_fused,
                            "skeleton_mlups": cells / ms_cg_sk / 1e3, "fused_mlups": cells / ms_cg_fused / 1e3,
                            "skeleton_gbs": 112 * cells / ms_cg_sk / 1e6, "fused_gbs": 64 * cells / ms_cg_fused / 1e6,
                            "nodes": len(cplan["nodes"]), "streams": cplan["streams"], "events": cplan["events"],
                            "note": "skeleton = the paper's 6 containers + 3 scalar steps (112 B/cell/iter); fused "
                                    "= 2 phase kernels (64 B/cell/iter); bitwise equal iterates"}}


# ---------------------------------------------------------------------------
def host_info():
    """CPU model, logical cores and RAM of the host running the oracle."""
    model, mem = None, None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                mem = round(int(line.split()[1]) / 1024 / 1024, 1)
                break
    except OSError:
        pass
    return {"cpu_model": model, "logical_cores": os.cpu_count(), "ram_gib": mem,
            "sched_affinity_cores": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else None}


def _oracle_threads(nthreads):
    """The oracle on `nthreads` host threads (torchrun sets OMP_NUM_THREADS=1
    in each rank; the reference arm and cpu_baseline run on rank 0 alone)."""
    import oracle
    oracle.set_num_threads(nthreads)
    return oracle


def _oracle_all_cores():
    return _oracle_threads(os.cpu_count() or 1)


def _time_oracle_cg(n, iters, nthreads):
    import synth
    oracle = _oracle_threads(nthreads)
    b = synth.poisson_poly_rhs((n, n, n))
    t0 = time.perf_counter()
    oracle.cg(b, max_iter=0)
    t1 = time.perf_counter()
    oracle.cg(b, max_iter=iters)
    t2 = time.perf_counter()
    per_iter = max((t2 - t1) - (t1 - t0), 1e-9) / iters
    return n ** 3 / per_iter / 1e6, oracle.num_threads(), per_iter


def cpu_baseline_cg(n, iters=3):
    """The oracle (plain C, fp64, OpenMP over planes), as it stands, on the
    host cores: CG iterations on the full n^3 grid (setup subtracted), on
    every core and on one thread (SURVEY §8(d) "CPU oracle timing")."""
    v_all, cores, per_all = _time_oracle_cg(n, iters, os.cpu_count() or 1)
    v_one, _, per_one = _time_oracle_cg(n, 1, 1)
    return {"value": v_all, "unit": "MLUPS", "cores": cores, "kind": "oracle",
            "sample": f"{iters} CG iterations on the full {n}^3 grid on {cores} threads, and 1 iteration on "
                      "1 thread (oracle.cg; set-up time subtracted)",
            "ms_per_iter": per_all * 1e3,
            "one_thread": {"value": v_one, "unit": "MLUPS", "cores": 1, "ms_per_iter": per_one * 1e3},
            "host": host_info()}


def cpu_baseline_lbm(n=256, steps=2):
    import numpy as np

    out = {}
    for label, nth in (("all", os.cpu_count() or 1), ("one", 1)):
        oracle = _oracle_threads(nth)
        c, w, _ = oracle.lbm_lattice()
        f = np.broadcast_to(w[:, None, None, None], (19, n, n, n)).astype(np.float32)
        om = lbm_omega(n)
        k = steps if label == "all" else 1
        t0 = time.perf_counter()
        for _ in range(k):
            f = oracle.lbm_step(f, om)
        out[label] = ((time.perf_counter() - t0) / k, oracle.num_threads())
    dt, cores = out["all"]
    return {"value": n ** 3 / dt / 1e6, "unit": "MLUPS", "cores": cores, "kind": "oracle",
            "sample": f"{steps} cavity steps at {n}^3 on {cores} threads, 1 step on 1 thread "
                      "(512^3 x 19 fp64 does not fit the bounded sample)",
            "one_thread": {"value": n ** 3 / out["one"][0] / 1e6, "unit": "MLUPS", "cores": 1}}


def reference_arm(args, world, rank):
    """--impl reference: the oracle as it stands, on the host cores, same
    config / metric / unit; each step = one CG iteration on the full grid."""
    if rank != 0:
        return None
    import synth
    oracle = _oracle_all_cores()
    n = args.n
    b = synth.poisson_poly_rhs((n, n, n))
    # W untimed warm-up iterations, then K timed ones (capped at 400: ~0.35 s
    # each on 16 host cores at 512^3, so the arm stays within a few minutes)
    w = max(args.warmup, 3)
    k = max(1, min(args.steps, 400))
    t0 = time.perf_counter()
    oracle.cg(b, max_iter=w)
    t1 = time.perf_counter()
    oracle.cg(b, max_iter=w + k)
    t2 = time.perf_counter()
    per = ((t2 - t1) - (t1 - t0)) / k
    v = n ** 3 / per / 1e6
    return {"metric": METRIC, "value": v, "unit": "MLUPS", "n_gpus": world, "steps": k, "warmup": w,
            "ms_per_step": per * 1e3, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": f"C2 Poisson FD CG 7-point fp64 {n}^3 dense (configs[1])", "parts": 1},
            "cpu_baseline": {"value": v, "unit": "MLUPS", "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"{k} CG iterations on the full {n}^3 grid after {w} warm-up "
                                       "(time of cg(w+k) minus cg(w))", "host": host_info()},
            "e2e": {"value": v, "unit": "MLUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def relaunch_under_torchrun(args) -> int:
    """`bench.py --gpus N` (N > 1) outside torchrun: start N ranks, one per
    GPU, with torch.distributed.run on this node (rendezvous on 127.0.0.1)."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="nb", choices=["nb", "reference"])
    ap.add_argument("--workload", default="cg", choices=["cg", "lbm", "sparse", "fem"])
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--occ", default="two_way", choices=list(("none", "standard", "extended", "two_way")))
    ap.add_argument("--prof-steps", type=int, default=10)
    ap.add_argument("--no-extras", action="store_true", help="skip the extra workload lines and cpu_baseline")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch_under_torchrun(args))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; launch one rank per GPU "
              "(python bench.py --gpus N starts them itself)", file=sys.stderr)
        sys.exit(2)
    if args.impl == "reference":
        out = reference_arm(args, world, rank)
        if out is not None:
            print(json.dumps(out), flush=True)
        return
    world, rank, local = setup_dist(args)
    import __graft_entry__
    __graft_entry__.build()
    if args.workload == "cg":
        out = bench_cg(args, world, rank, local)
        if not args.no_extras and world == 1:
            lbm = bench_lbm_run(args.n, 20, 3, 1, local)
            out["also"] = {"lbm_d3q19": lbm, "c1": bench_c1(local),
                           "sparse_c4": bench_sparse_run(args.n, 20, 3, 1, local),
                           "fem_c5": bench_fem_run(384, 20, 3, 1, local),
                           "skeleton_f1": bench_skeleton(local),
                           "lbm_sparse_f2": bench_lbm_sparse_run(args.n, 20, 3, local),
                           "lbm_aa_f3": bench_lbm_aa_run(args.n, 20, 4, local),
                           "lbm_layouts_f3": bench_lbm_layouts(args.n, 10, local),
                           "karman_f4": bench_karman(local),
                           "fem_sparse_f4": bench_fem_sparse_run(384, 20, local)}
            out["cpu_baseline"] = cpu_baseline_cg(args.n)
            out["also"]["lbm_d3q19"]["cpu_baseline"] = cpu_baseline_lbm()
        elif not args.no_extras:
            # N > 1: the scaling lines of SURVEY §8(d) — C2 weak (n^3 per GPU),
            # C3 D3Q19 weak (n^3 per GPU), C4 and C5 strong — each with its
            # per-rank dominant-kernel roofline and communication times
            wa = argparse.Namespace(**vars(args))
            wa.steps = min(args.steps, 50)
            out["also"] = {"c2_weak": bench_cg(wa, world, rank, local, weak=True, with_e2e=False),
                           "lbm_d3q19_weak": bench_lbm_run(args.n, 20, 3, world, local),
                           "sparse_c4_strong": bench_sparse_run(args.n, 20, 3, world, local),
                           "fem_c5_strong": bench_fem_run(384, 20, 3, world, local)}
    elif args.workload in ("sparse", "fem"):
        fn = bench_sparse_run if args.workload == "sparse" else bench_fem_run
        r = fn(args.n if args.workload == "sparse" else min(args.n, 384), args.steps, args.warmup, world, local)
        out = {"metric": METRIC, "higher_is_better": True, "vs_baseline": None, "data": "synthetic",
               "warmup": args.warmup, **r}
    else:
        r = bench_lbm_run(args.n, args.steps, args.warmup, world, local, occ=args.occ if args.occ in
                          ("none", "standard") else "standard")
        out = {"metric": METRIC, "higher_is_better": True, "vs_baseline": None, "data": "synthetic", **r}
        if world == 1 and not args.no_extras:
            out["cpu_baseline"] = cpu_baseline_lbm()
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
