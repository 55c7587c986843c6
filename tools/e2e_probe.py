"""Where the C2 e2e time goes: CUDA-event times of each public-API piece of
bench.py's e2e call (uploads, CG create, prepare, iterate, finish, download)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 200
cells = n ** 3
g = nb.Grid((n, n, n))
stream = torch.cuda.ExternalStream(g.stream())
b, x = nb.Field(g), nb.Field(g)
bh = torch.rand(cells, dtype=torch.float64).pin_memory()
xh = torch.zeros(cells, dtype=torch.float64).pin_memory()
pieces = {}


def run(record):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(8)]
    t = [0.0] * 8
    ev[0].record(stream); t[0] = time.perf_counter()
    b.upload_async(bh.data_ptr())
    ev[1].record(stream); t[1] = time.perf_counter()
    x.upload_async(xh.data_ptr())
    ev[2].record(stream); t[2] = time.perf_counter()
    s = nb.CG(x, b)
    ev[3].record(stream); t[3] = time.perf_counter()
    s.prepare(steps)
    ev[4].record(stream); t[4] = time.perf_counter()
    s.iterate(steps)
    ev[5].record(stream); t[5] = time.perf_counter()
    s.finish()
    s.close()
    ev[6].record(stream); t[6] = time.perf_counter()
    x.download(xh)
    ev[7].record(stream); t[7] = time.perf_counter()
    torch.cuda.synchronize()
    if record:
        names = ["upload_b", "upload_x", "cg_create", "prepare", "iterate", "finish", "download_x"]
        for i, nm in enumerate(names):
            pieces[nm] = {"gpu_ms": ev[i].elapsed_time(ev[i + 1]), "host_ms": (t[i + 1] - t[i]) * 1e3}
        pieces["total_gpu_ms"] = ev[0].elapsed_time(ev[7])


run(False)
run(True)
print(pieces)
