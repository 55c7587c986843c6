"""CUPTI kernel timeline (torch.profiler) of a few CG iterations / LBM steps:
per-kernel device durations and the idle gaps between consecutive kernels.
  python tools/timeline.py [n] [iters] [cg|lbm] [--out gpurun_out/timeline.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 8
what = sys.argv[3] if len(sys.argv) > 3 else "cg"
parts = int(sys.argv[4]) if len(sys.argv) > 4 and not sys.argv[4].startswith("--") else 1
hmode = int(sys.argv[5]) if len(sys.argv) > 5 and not sys.argv[5].startswith("--") else 0
if what == "sparse":
    import synth  # noqa: E402
    g = nb.Grid((n, n, n), nparts=parts, devices=[0] * parts, active=synth.sphere_mask(n))
else:
    g = nb.Grid((n, n, n), nparts=parts, devices=[0] * parts)
g.set_halo_mode(hmode)
if what in ("sparse", "fem"):  # C4 / C5 CG under Two-way OCC
    card = 3 if what == "fem" else 1
    b, x = nb.Field(g, card=card), nb.Field(g, card=card)
    if what == "fem":
        nb.nb_fem27_rhs(b, 1.0)
    else:
        b.fill_uniform(seed=4)
    x.fill_const(0.0)
    cg = nb.CG(x, b, op=nb.OP_FEM27 if what == "fem" else nb.OP_LAPLACE7)
    cg.iterate(4)
    g.sync()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        cg.iterate(iters)
        g.sync()
    cg.finish()
    cg.close()
elif what == "cg":
    b, x = nb.Field(g), nb.Field(g)
    b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0)
    cg = nb.CG(x, b)
    cg.iterate(16)
    g.sync()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        cg.iterate(iters)
        g.sync()
    cg.finish()
    cg.close()
else:
    fa, fb = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(fa, 1.0, (0, 0, 0))
    fa, fb = nb.nb_lbm_step(fa, fb, 0.7886, 2)
    g.sync()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        fa, fb = nb.nb_lbm_step(fa, fb, 0.7886, iters)
        g.sync()
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
ks = sorted([(e.time_range.start, e.time_range.end, e.name) for e in evs])
streams = {}  # kernel name -> set of device streams (the halo stream shows up separately)
# halo copies vs kernels: fraction of copy time overlapped by a running kernel
def is_copy(nm):
    return "Memcpy" in nm or "memcpy" in nm or "k_halo_copy" in nm


copies = [(s, e) for s, e, nm in ks if is_copy(nm)]
kern = [(s, e) for s, e, nm in ks if not is_copy(nm)]
cov = 0.0
for cs_, ce_ in copies:
    segs = sorted((max(cs_, s), min(ce_, e)) for s, e in kern if s < ce_ and e > cs_)
    t, cur = 0.0, cs_
    for s, e in segs:
        s = max(s, cur)
        if e > s:
            t += e - s
            cur = e
    cov += t
copy_t = sum(e - s for s, e in copies)
rows = []
for i, (s, e, name) in enumerate(ks):
    gap = s - ks[i - 1][1] if i else 0.0
    rows.append({"name": name[:50], "start_us": s - ks[0][0], "dur_us": e - s, "gap_us": gap})
tot = ks[-1][1] - ks[0][0]
# busy = union of device activity (kernels and copies may overlap)
busy, cur = 0.0, None
for s_, e_, _ in ks:
    if cur is None or s_ > cur[1]:
        if cur:
            busy += cur[1] - cur[0]
        cur = [s_, e_]
    else:
        cur[1] = max(cur[1], e_)
busy += cur[1] - cur[0] if cur else 0.0
summary = {"what": what, "n": n, "parts": parts, "halo_mode": hmode, "iters": iters, "span_us": tot,
           "busy_us": busy, "idle_us": tot - busy, "kernels": len(rows), "halo_copies": len(copies),
           "halo_copy_us": copy_t, "halo_copy_overlapped_frac": (cov / copy_t) if copy_t else None}
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as fh:
        json.dump({"summary": summary, "kernels": rows}, fh, indent=1)
print(json.dumps(summary), flush=True)
if "--quiet" not in sys.argv:
    for r in rows[:24]:
        print(f"{r['name']:50s} dur {r['dur_us']:9.1f} us  gap {r['gap_us']:7.1f} us")
