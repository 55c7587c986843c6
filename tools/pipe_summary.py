"""Per-launch pipe utilisation from an ncu raw page (--page raw --csv):
time, DRAM bytes, LSU data-pipe wavefronts (all / shared-memory part),
FP64 pipe, issue activity, resident warps, grid.  Shows which on-chip limit
a kernel sits against when it is below the HBM roofline.
  python tools/pipe_summary.py <raw.csv> [title]"""
import csv
import sys

K = [("gpu__time_duration.sum", "us", 1.0),
     ("dram__bytes_read.sum", "rd_GB", None), ("dram__bytes_write.sum", "wr_GB", None),
     ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", "lsu%", 1.0),
     ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed", "smem%", 1.0),
     ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_elapsed", "fp64%", 1.0),
     ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue%", 1.0),
     ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps%", 1.0),
     ("launch__grid_size", "grid", 1.0)]
SCALE = {"byte": 1e-9, "Kbyte": 1e-6, "Mbyte": 1e-3, "Gbyte": 1.0, "B": 1e-9, "KB": 1e-6, "MB": 1e-3, "GB": 1.0}
rows = list(csv.reader(open(sys.argv[1])))
h, u = rows[0], rows[1]
print(f"# {sys.argv[2] if len(sys.argv) > 2 else sys.argv[1]}")
print(f"{'kernel':44s} " + " ".join(f"{n:>7s}" for _, n, _ in K))
for r in rows[2:]:
    out = []
    for key, name, sc in K:
        if key not in h:
            out.append(f"{'-':>7s}")
            continue
        i = h.index(key)
        v = float(r[i].replace(",", "") or 0)
        if sc is None:
            v *= SCALE.get(u[i], 1.0)
        if name == "us" and u[i] in ("msecond", "ms"):
            v *= 1e3
        if name == "us" and u[i] in ("nsecond", "ns"):
            v *= 1e-3
        out.append(f"{v:7.3f}" if name.endswith("GB") else f"{v:7.1f}")
    print(f"{r[h.index('Kernel Name')][:44]:44s} " + " ".join(out))
