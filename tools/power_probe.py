"""Board power / clocks while a workload runs back to back for a few seconds
(C2 CG 512^3, or C3 LBM 512^3): nvidia-smi sampled every 50 ms alongside
per-chunk CUDA-event times.  Diagnostic for the sw_power_cap drift."""
import os
import subprocess
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

work = sys.argv[1] if len(sys.argv) > 1 else "cg"
chunks = int(sys.argv[2]) if len(sys.argv) > 2 else 40
rows = []


def sampler(stop):
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.mem,power.draw,clocks_event_reasons.active",
                          "--format=csv,noheader,nounits", "-lms", "50"], stdout=subprocess.PIPE, text=True)
    while not stop.is_set():
        line = p.stdout.readline()
        if line:
            rows.append((time.time(), line.strip()))
    p.terminate()


n = 512
g = nb.Grid((n, n, n))
if work == "cg":
    b, x = nb.Field(g), nb.Field(g)
    b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0)
    cg = nb.CG(x, b, max_iter=10 ** 9)
    cg.prepare(16)
    step, per = (lambda: cg.iterate(16)), 16
else:
    f0, f1 = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(f0, 1.0, (0.0, 0.0, 0.0))
    st = [f0, f1]

    def step():
        st[0], st[1] = nb.nb_lbm_step(st[0], st[1], 0.7886, 4)
    per = 4
step()
g.sync()
stop = threading.Event()
th = threading.Thread(target=sampler, args=(stop,), daemon=True)
th.start()
time.sleep(0.5)
s = torch.cuda.ExternalStream(g.stream())
evs = [torch.cuda.Event(enable_timing=True) for _ in range(chunks + 1)]
t0 = time.time()
evs[0].record(s)
for i in range(chunks):
    step()
    evs[i + 1].record(s)
g.sync()
t1 = time.time()
time.sleep(0.3)
stop.set()
ms = [evs[i].elapsed_time(evs[i + 1]) / per for i in range(chunks)]
print(work, "ms/step per chunk:", " ".join(f"{m:.3f}" for m in ms))
print("samples during run:")
for t, r in rows:
    if t0 - 0.1 <= t <= t1 + 0.1:
        print(f"  {t - t0:6.3f}s  {r}")
