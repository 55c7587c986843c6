"""R2 / R3 replicas (Fig. 8) on ONE B200:
C2 CG time per iteration for G = 1..8 virtual partitions under the four OCC
modes (R2: 320^3), and the size sweep 128^3..512^3 at G = 8 (R3).  With
virtual partitions on one GPU every halo is a device-local fused store, so
this measures what the OCC schedules cost in kernel splits and launches —
the communication side needs the 8-GPU box.  R1 (Fig. 7 analogue): the
D3Q19 cavity at 192^3..512^3, one partition vs 8 virtual partitions under
No-OCC and Standard OCC.
  python tools/occ_sweep.py [--out gpurun_out/occ_sweep.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

ITERS = 32
OCC = {"none": nb.OCC_NONE, "standard": nb.OCC_STANDARD, "extended": nb.OCC_EXTENDED, "two_way": nb.OCC_TWO_WAY}


def cg_ms(n, parts, occ):
    with nb.Grid((n, n, n), nparts=parts, devices=[0] * parts) as g:
        b, x = nb.Field(g), nb.Field(g)
        b.fill(nb.FILL_POISSON_RHS)
        x.fill_const(0.0)
        cg = nb.CG(x, b, max_iter=10 ** 9, occ=occ)
        cg.prepare(ITERS)
        cg.iterate(ITERS)
        g.sync()
        s = torch.cuda.ExternalStream(g.stream())
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        cg.iterate(ITERS)
        e1.record(s)
        torch.cuda.synchronize()
        cg.finish()
        cg.close()
        b.close(), x.close()
        return e0.elapsed_time(e1) / ITERS


r2 = []
for parts in (1, 2, 4, 8):
    row = {"G": parts}
    for name, occ in OCC.items():
        row[name] = cg_ms(320, parts, occ)
    r2.append(row)
    print("R2 320^3", row, flush=True)
r3 = []
for n in (128, 192, 256, 320, 384, 448, 512):
    row = {"n": n}
    for name, occ in OCC.items():
        row[name] = cg_ms(n, 8, occ)
    row["mlups_two_way"] = n ** 3 / row["two_way"] / 1e3
    r3.append(row)
    print("R3 G=8", row, flush=True)


def lbm_ms(n, parts, occ, steps=8):
    """R1 (Fig. 7 analogue): D3Q19 cavity, n^3 global, ms per step."""
    with nb.Grid((n, n, n), nparts=parts, devices=[0] * parts) as g:
        f0, f1 = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        nb.nb_lbm_init(f0, 1.0, (0.0, 0.0, 0.0))
        om = 1.0 / (3.0 * 0.05 * n / 100.0 + 0.5)
        a, b = nb.nb_lbm_step(f0, f1, om, 2, occ=occ)
        g.sync()
        s = torch.cuda.ExternalStream(g.stream())
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        a, b = nb.nb_lbm_step(a, b, om, steps, occ=occ)
        e1.record(s)
        torch.cuda.synchronize()
        a.close(), b.close()
        return e0.elapsed_time(e1) / steps


r1 = []
if "--no-lbm" not in sys.argv:
    for n in (192, 256, 320, 384, 448, 512):
        row = {"n": n, "G1_standard": lbm_ms(n, 1, nb.OCC_STANDARD)}
        for name in ("none", "standard"):
            row["G8_" + name] = lbm_ms(n, 8, OCC[name])
        row["mlups_G8_standard"] = n ** 3 / row["G8_standard"] / 1e3
        r1.append(row)
        print("R1 LBM", row, flush=True)
out = {"iters": ITERS, "R2_320": r2, "R3_G8": r3, "R1_lbm": r1,
       "note": "ms per CG iteration (CUDA-graph chunks, device events) / per LBM step; virtual partitions on one B200"}
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as fh:
        json.dump(out, fh, indent=1)
