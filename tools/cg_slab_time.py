"""ms per CG iteration on one GPU for an nx x ny x nz slab (a proxy for one
rank's share of a z-partitioned strong-scaling run), CUDA events over a
graph-replayed run.  python tools/cg_slab_time.py nx ny nz [iters]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

nx, ny, nz = (int(a) for a in sys.argv[1:4])
iters = int(sys.argv[4]) if len(sys.argv) > 4 else 64
g = nb.Grid((nx, ny, nz))
b, x = nb.Field(g), nb.Field(g)
b.fill_uniform(seed=2)
x.fill_const(0.0)
cg = nb.CG(x, b, max_iter=10 ** 9)
cg.iterate(16)
cg.prepare(iters)
g.sync()
s = torch.cuda.ExternalStream(g.stream())
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s)
cg.iterate(iters)
e1.record(s)
e1.synchronize()
ms = e0.elapsed_time(e1) / iters
print(f"{nx}x{ny}x{nz} zc={os.environ.get('NB_CG_ZC', 'auto')} ms/iter {ms:.4f} MLUPS {nx * ny * nz / ms / 1e3:.0f}")
cg.finish()
