"""Fig. 9 analogue: Poisson CG on a solid
cube of volume fraction phi inside an N^3 box, run (a) on the element-sparse
grid (only the cube's cells stored, connectivity table) and (b) on the dense
grid over the whole box (the dense data structure cannot skip cells).
Device time per CG iteration for phi = 1.0 ... 0.1; the crossover is where
the sparse grid starts to win.
  python tools/sparsity_sweep.py [N] [--out gpurun_out/sparsity_sweep.json]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 and not sys.argv[1].startswith("--") else 384
ITERS = 20


def cg_ms(grid, active_cells):
    b, x = nb.Field(grid), nb.Field(grid)
    b.fill_uniform(seed=4)
    x.fill_const(0.0)
    cg = nb.CG(x, b, max_iter=10 ** 9)
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


rows = []
with nb.Grid((N, N, N)) as g:
    dense_ms = cg_ms(g, N ** 3)
for phi in (1.0, 0.9, 0.8, 0.7, 0.6, 0.5, 0.4, 0.3, 0.2, 0.1):
    side = max(2, int(round(N * phi ** (1.0 / 3.0))))
    lo = (N - side) // 2
    m = np.zeros((N, N, N), np.uint8)
    m[lo:lo + side, lo:lo + side, lo:lo + side] = 1
    act = int(m.sum(dtype=np.int64))
    with nb.Grid((N, N, N), active=m) as g:
        sp = cg_ms(g, act)
    rows.append({"phi": act / N ** 3, "active": act, "sparse_ms_per_iter": sp, "dense_ms_per_iter": dense_ms,
                 "sparse_over_dense": sp / dense_ms})
    print(f"phi {act / N ** 3:5.3f}  sparse {sp:7.3f} ms  dense {dense_ms:7.3f} ms  ratio {sp / dense_ms:5.2f}",
          flush=True)
out = {"N": N, "iters": ITERS, "rows": rows,
       "note": "dense = the same Poisson CG over the whole box (64 B/cell/iter); sparse = element-sparse grid "
               "of the cube (104 B/active cell/iter incl. 24 B connectivity)"}
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as fh:
        json.dump(out, fh, indent=1)
