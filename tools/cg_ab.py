"""Interleaved A/B of the C2 CG iteration time (512^3, graph replay, CUDA
events): default vs an environment switch read per call (e.g. NB_NO_FOLD=1).
  python tools/cg_ab.py [n] [iters] [ENV=VALUE ...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

args = [a for a in sys.argv[1:] if "=" not in a]
envs = [a.split("=", 1) for a in sys.argv[1:] if "=" in a]
n = int(args[0]) if args else 512
iters = int(args[1]) if len(args) > 1 else 100
parts = int(os.environ.get("AB_PARTS", "1"))
g = nb.Grid((n, n, n), nparts=parts, devices=[0] * parts)
g.set_halo_mode(int(os.environ.get("AB_HALO", "0")))  # 1: halo copies on the halo stream
s = torch.cuda.ExternalStream(g.stream())
b, x = nb.Field(g), nb.Field(g)
b.fill(nb.FILL_POISSON_RHS)


def run(variant):
    for k, v in envs:
        if variant:
            os.environ[k] = v
        else:
            os.environ.pop(k, None)
    x.fill_const(0.0)
    cg = nb.CG(x, b, max_iter=10 ** 9)
    cg.prepare(iters)
    cg.iterate(10)
    cg.prepare(iters)
    g.sync()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    cg.iterate(iters)
    e1.record(s)
    torch.cuda.synchronize()
    r = cg.finish()
    cg.close()
    return e0.elapsed_time(e1) / iters, r.rr


res = {"A": [], "B": []}
for rep in range(3):
    for v, key in ((0, "A"), (1, "B")):
        ms, rr = run(v)
        res[key].append(ms)
        print(json.dumps({"variant": key, "env": envs if v else [], "ms_per_iter": ms, "rr": rr}), flush=True)
print(json.dumps({"A_min": min(res["A"]), "B_min": min(res["B"]), "n": n, "parts": parts}))
