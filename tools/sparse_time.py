"""C4 sparse CG timing probe: ms per iteration (graph replay, CUDA events)
and the per-kernel split, plus a digest of x (bitwise comparison of build
variants; select one with NB_LIB=...).  python tools/sparse_time.py [n] [iters]"""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402
import synth  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 20
mask = synth.sphere_mask(n)
g = nb.Grid((n, n, n), nparts=1, devices=[0], active=mask)
stream = torch.cuda.ExternalStream(g.stream())
b, x = nb.Field(g), nb.Field(g)
b.fill_uniform(seed=4)
x.fill_const(0.0)
cg = nb.CG(x, b)
cg.iterate(3)
cg.prepare(iters)
g.sync()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(stream)
cg.iterate(iters)
e1.record(stream)
e1.synchronize()
ms = e0.elapsed_time(e1) / iters
g.profile(True)
cg.iterate(5)
split = {}
for nm in ("k_sp_cg_map", "k_sp_cg_q", "k_sp_cg_mq", "k_sp_cg_r", "k_sp_cg_a", "k_sp_cg_b", "k_finalize"):
    k, t = g.profile_read(nm)
    if k:
        split[nm] = t / 5
g.profile(False)
cg.finish()
dig = hashlib.sha1(x.download().tobytes()).hexdigest()
print(json.dumps({"lib": os.environ.get("NB_LIB", "libnb.so").split("/")[-1], "ms_per_iter": ms,
                  "mlups": int(mask.sum()) / ms / 1e3, "split": split, "digest": dig}))
