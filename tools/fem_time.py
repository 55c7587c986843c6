"""FEM (C5) timing probe: K u (nb_fem27_apply) and CG iterations at n^3
nodes, CUDA-event timed, plus the per-kernel split of a CG iteration.
Select a library build with NB_LIB=... (e.g. an NB_VARIANT build).
  python tools/fem_time.py [n] [iters]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 384
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 20
g = nb.Grid((n, n, n))
stream = torch.cuda.ExternalStream(g.stream())
u, y = nb.Field(g, card=3), nb.Field(g, card=3)
u.fill_uniform(seed=5)
u.halo_update()


def timed(fn, reps):
    with torch.cuda.stream(stream):
        fn()
        g.sync()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            fn()
        e1.record(stream)
        e1.synchronize()
    return e0.elapsed_time(e1) / reps


apply_ms = timed(lambda: nb.nb_fem27_apply(u, y, 1.0, 0.3), iters)
b, x = nb.Field(g, card=3), nb.Field(g, card=3)
nb.nb_fem27_rhs(b, 1.0)
x.fill_const(0.0)
cg = nb.CG(x, b, op=nb.OP_FEM27)
cg.iterate(3)
cg.prepare(iters)
g.sync()
with torch.cuda.stream(stream):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    cg.iterate(iters)
    e1.record(stream)
    e1.synchronize()
cg_ms = e0.elapsed_time(e1) / iters
cg.finish()
cg.close()
x.fill_const(0.0)
cg = nb.CG(x, b, op=nb.OP_FEM27)
g.profile(True)
cg.iterate(5)
names = ["k_fem_map", "k_fem_surface", "k_fem_faces", "k_fem_cg_q", "k_fem_cg_a", "k_fem_r"]
split = {}
for nm in names:
    k, ms = g.profile_read(nm)
    if k:
        split[nm] = ms / 5  # per CG iteration (k launches over 5 iterations)
g.profile(False)
cg.finish()
cg.close()
nodes = n ** 3
print(json.dumps({"lib": os.environ.get("NB_LIB", "libnb.so").split("/")[-1], "n": n,
                  "apply_ms": apply_ms, "apply_tflops": 306 * nodes / apply_ms / 1e9,
                  "cg_ms_per_iter": cg_ms, "kernel_ms_per_iter": split}))
