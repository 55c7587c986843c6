"""Long-run drift of the C2 CG kernels: per-kernel event times (profiling
mode, eager launches) chunk by chunk, with the SM clock sampled alongside."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n, chunks = 512, int(sys.argv[1]) if len(sys.argv) > 1 else 20
g = nb.Grid((n, n, n))
b, x = nb.Field(g), nb.Field(g)
b.fill(nb.FILL_POISSON_RHS)
x.fill_const(0.0)
cg = nb.CG(x, b, max_iter=10 ** 9)
cg.iterate(4)
g.sync()
for i in range(chunks):
    g.profile(True)
    cg.iterate(16)
    g.sync()
    a = g.profile_read("k_msr_cgA")
    bb = g.profile_read("k_cg_B")
    f = g.profile_read("k_finalize")
    clk = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm,power.draw,clocks_throttle_reasons.active",
                          "--format=csv,noheader"], capture_output=True, text=True).stdout.strip()
    print(f"chunk {i:2d}  A {a[1] / a[0]:.3f}  B {bb[1] / bb[0]:.3f}  fin {f[1] / f[0]:.4f} ms   [{clk}]", flush=True)
g.profile(False)
cg.finish()
cg.close()
b.close(), x.close()
g.close()
