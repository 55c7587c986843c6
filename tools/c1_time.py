"""C1 (64^3 fp64, 10 map-stencil-reduce iterations) per-call time, as
bench.py measures it (CUDA events on the grid stream over 50 synchronous
calls).  python tools/c1_time.py [n]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
g = nb.Grid((n, n, n))
stream = torch.cuda.ExternalStream(g.stream())
x, y = nb.Field(g), nb.Field(g)
x.fill_int(seed=1)
y.fill_const(0.0)
for _ in range(20):
    nb.nb_map_stencil_reduce(x, y, 0.125, 10, nb.OCC_TWO_WAY)
g.sync()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
t0 = time.perf_counter()
e0.record(stream)
for _ in range(50):
    nb.nb_map_stencil_reduce(x, y, 0.125, 10, nb.OCC_TWO_WAY)
e1.record(stream)
torch.cuda.synchronize()
print(f"C1 {n}^3 fin_each={os.environ.get('NB_C1_FIN_EACH', '0')} ms/call dev {e0.elapsed_time(e1) / 50:.4f} "
      f"wall {(time.perf_counter() - t0) / 50 * 1e3:.4f}")
x.close(), y.close()
g.close()
