"""Sustained HBM copy bandwidth: torch copy_ of 1 Gi bf16 elements (the
MEASURED_PEAKS.json recipe) back to back for a few seconds, CUDA events per
chunk, nvidia-smi clocks / power sampled alongside.  Shows whether a plain
streaming copy also slows once the board reaches its power cap (context for
the C2 drift)."""
import json
import subprocess
import sys
import threading
import time

import torch

secs = float(sys.argv[1]) if len(sys.argv) > 1 else 3.0
n = 1 << 30
a = torch.empty(n, dtype=torch.bfloat16, device="cuda").fill_(1)
b = torch.empty_like(a)
rows = []


def sampler(stop):
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw,clocks_event_reasons.active",
                          "--format=csv,noheader,nounits", "-lms", "50"], stdout=subprocess.PIPE, text=True)
    while not stop.is_set():
        line = p.stdout.readline()
        if line:
            rows.append(line.strip())
    p.terminate()


for _ in range(3):
    b.copy_(a)
torch.cuda.synchronize()
stop = threading.Event()
threading.Thread(target=sampler, args=(stop,), daemon=True).start()
time.sleep(0.3)
per = 10
chunks = []
t0 = time.time()
while time.time() - t0 < secs:
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(per):
        b.copy_(a)
    e1.record()
    e1.synchronize()
    chunks.append(2 * n * 2 * per / (e0.elapsed_time(e1) * 1e-3) / 1e9)
stop.set()
clk = [int(r.split(",")[0]) for r in rows[len(rows) // 3:]]
print(json.dumps({"copy_gbs_first_chunk": chunks[0], "copy_gbs_best": max(chunks),
                  "copy_gbs_last_third_median": sorted(chunks[2 * len(chunks) // 3:])[len(chunks[2 * len(chunks) // 3:]) // 2],
                  "chunks": [round(c, 1) for c in chunks], "sm_mhz_median_late": sorted(clk)[len(clk) // 2] if clk else None,
                  "samples": rows}))
