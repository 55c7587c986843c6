"""Per-chunk timing of C2 CG at 512^3 over a long run (power / clock drift
check): CUDA events around every 16-iteration chunk on the grid stream."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
chunks = int(sys.argv[2]) if len(sys.argv) > 2 else 24
g = nb.Grid((n, n, n))
b, x = nb.Field(g), nb.Field(g)
b.fill(nb.FILL_POISSON_RHS)
x.fill_const(0.0)
cg = nb.CG(x, b, max_iter=10 ** 9)
cg.prepare(16)
cg.iterate(16)
g.sync()
s = torch.cuda.ExternalStream(g.stream())
evs = [torch.cuda.Event(enable_timing=True) for _ in range(chunks + 1)]
evs[0].record(s)
for i in range(chunks):
    cg.iterate(16)
    evs[i + 1].record(s)
g.sync()
ms = [evs[i].elapsed_time(evs[i + 1]) / 16 for i in range(chunks)]
print("ms/iter per chunk:", " ".join(f"{m:.3f}" for m in ms))
cg.finish()
cg.close()
b.close(), x.close()
g.close()
