"""A/B of the sparse FEM operator: shared-memory box (default) vs the gather
pass (NB_SPF_GATHER=1): per-kernel times of one CG iteration (profiled,
eager) and the CG iteration time (graph), 384^3 full cube and the C4-style
sphere, plus a bitwise check of the iterates.  Usage: python tools/sparse_fem_box_ab.py [N]"""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

N = int(sys.argv[1]) if len(sys.argv) > 1 else 384
KS = ("k_sp_fem_cg_a", "k_sp_fem_q", "k_sp_fem_dot", "k_sp_cg_map", "k_sp_cg_r", "k_finalize")
MODES = {"box": {}, "tiledot": {"NB_SPF_TILEDOT": "1"}, "fused": {"NB_SPF_FUSED": "1"},
         "gather": {"NB_SPF_GATHER": "1"}}


def run(mask, mode, iters=10):
    for k in ("NB_SPF_FUSED", "NB_SPF_GATHER", "NB_SPF_TILEDOT"):
        os.environ.pop(k, None)
    os.environ.update(MODES[mode])
    g = nb.Grid((N, N, N), active=mask)
    b, x = nb.Field(g, card=3), nb.Field(g, card=3)
    nb.nb_fem27_rhs(b, 1.0)
    x.fill_const(0.0)
    cg = nb.CG(x, b, op=nb.OP_FEM27)
    cg.iterate(3)
    cg.prepare(iters)
    g.sync()
    s = torch.cuda.ExternalStream(g.stream())
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    cg.iterate(iters)
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / iters
    g.profile(True)
    cg.iterate(2)
    prof = {k: g.profile_read(k)[1] / 2 for k in KS}
    g.profile(False)
    cg.finish()
    dig = hashlib.sha1(x.download().tobytes()).hexdigest()[:12]
    cg.close(), b.close(), x.close(), g.close()
    return {"ms_per_iter": ms, "kernel_ms": prof, "x_digest": dig}


out = {"N": N}
for name, mask in (("full", np.ones((N, N, N), np.uint8)), ("sphere", synth.sphere_mask(N))):
    act = int(mask.sum())
    r = {"active": act}
    for mode in MODES:
        r[mode] = run(mask, mode)
    r["same_bits_segment_dot"] = len({r[m]["x_digest"] for m in ("box", "fused", "gather")}) == 1
    out[name] = r
    print(name, json.dumps(r), flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/sparse_fem_box_ab.json", "w"), indent=1)
