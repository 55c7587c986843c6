"""OCC on the sparse (C4) and FEM (C5) CG schedules on ONE B200: ms per
iteration at G = 1, 2, 4, 8 virtual partitions under No-OCC and Two-way OCC,
with the fused (stream-ordered) halo and with the halo on its own stream
(NB_HALO_STREAM: the copies overlap the interior work, as the peer / NCCL
transports do across GPUs).
  python tools/occ_sparse_fem.py [--out gpurun_out/occ_sparse_fem.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402
import synth  # noqa: E402

ITERS = 16


def cg_ms(what, n, parts, occ, halo):
    active = synth.sphere_mask(n) if what == "sparse" else None
    with nb.Grid((n, n, n), nparts=parts, devices=[0] * parts, active=active) as g:
        g.set_halo_mode(halo)
        card = 3 if what == "fem" else 1
        b, x = nb.Field(g, card=card), nb.Field(g, card=card)
        if what == "fem":
            nb.nb_fem27_rhs(b, 1.0)
        else:
            b.fill_uniform(seed=4)
        x.fill_const(0.0)
        cg = nb.CG(x, b, max_iter=10 ** 9, occ=occ, op=nb.OP_FEM27 if what == "fem" else nb.OP_LAPLACE7)
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


rows = []
for what, n in (("sparse", 512), ("fem", 384)):
    for parts in (1, 2, 4, 8):
        row = {"what": what, "n": n, "G": parts}
        for oname, occ in (("none", nb.OCC_NONE), ("two_way", nb.OCC_TWO_WAY)):
            for hname, halo in (("fused", nb.HALO_FUSED), ("stream", nb.HALO_STREAM)):
                row[f"{oname}_{hname}"] = cg_ms(what, n, parts, occ, halo)
        rows.append(row)
        print(json.dumps(row), flush=True)
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as fh:
        json.dump({"ms_per_iter": rows, "iters": ITERS}, fh, indent=1)
