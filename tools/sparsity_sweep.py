"""Fig. 9 analogue (the linear-elastic FEM "on dense and
sparse" grids): a solid cube of volume fraction phi inside
an N^3 box, solved (a) on the element-sparse grid (only the cube's nodes
stored) and (b) on the dense grid over the whole box (the dense data
structure cannot skip cells).  Device time per CG iteration for
phi = 1.0 ... 0.1; the crossover is where the sparse grid starts to win.
Workloads: fem (the paper's, C5 physics: 3 fp64 dof per node, Dirichlet
z = 0, pressure on the exposed top faces) and poisson (7-point CG).
  python tools/sparsity_sweep.py [N] [fem|poisson|both] [--out gpurun_out/sparsity_sweep.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
if "--out" in sys.argv:
    args = [a for a in args if a != sys.argv[sys.argv.index("--out") + 1]]
N = int(args[0]) if args else 384
WHAT = args[1] if len(args) > 1 else "both"
ITERS = 20


def cg_ms(grid, fem):
    card = 3 if fem else 1
    b, x = nb.Field(grid, card=card), nb.Field(grid, card=card)
    if fem:
        nb.nb_fem27_rhs(b, 1.0)
    else:
        b.fill_uniform(seed=4)
    x.fill_const(0.0)
    cg = nb.CG(x, b, max_iter=10 ** 9, op=nb.OP_FEM27 if fem else nb.OP_LAPLACE7)
    cg.prepare(ITERS)
    cg.iterate(ITERS)
    grid.sync()
    s = torch.cuda.ExternalStream(grid.stream())
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    cg.iterate(ITERS)
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / ITERS
    cg.finish()
    cg.close()
    b.close(), x.close()
    return ms


out = {"N": N, "iters": ITERS}
for kind in (("fem", "poisson") if WHAT == "both" else (WHAT,)):
    fem = kind == "fem"
    rows = []
    with nb.Grid((N, N, N)) as g:
        dense_ms = cg_ms(g, fem)
    for phi in (1.0, 0.9, 0.8, 0.7, 0.6, 0.5, 0.4, 0.3, 0.2, 0.1):
        side = max(2, int(round(N * phi ** (1.0 / 3.0))))
        lo = (N - side) // 2
        m = np.zeros((N, N, N), np.uint8)
        # the cube stands on the z = 0 plane (the FEM's Dirichlet support)
        m[0:side, lo:lo + side, lo:lo + side] = 1
        act = int(m.sum(dtype=np.int64))
        with nb.Grid((N, N, N), active=m) as g:
            sp = cg_ms(g, fem)
        rows.append({"phi": act / N ** 3, "active": act, "sparse_ms_per_iter": sp, "dense_ms_per_iter": dense_ms,
                     "sparse_over_dense": sp / dense_ms})
        print(f"{kind} phi {act / N ** 3:5.3f}  sparse {sp:7.3f} ms  dense {dense_ms:7.3f} ms  ratio "
              f"{sp / dense_ms:5.2f}", flush=True)
    cross = next((r["phi"] for r in rows if r["sparse_over_dense"] < 1.0), None)
    out[kind] = {"rows": rows, "crossover_phi": cross}
out["note"] = ("dense = the same CG over the whole box (Poisson: 64 B/cell/iter; FEM: the fused 216 B/node "
               "schedule); sparse = the element-sparse grid of the cube (Poisson: 96 B/active cell/iter incl. the "
               "16 B neighbour table; FEM: 3-pass schedule, 27-neighbourhood table 40 B/node)")
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as fh:
        json.dump(out, fh, indent=1)
