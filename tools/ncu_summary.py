"""Summarise an ncu --set full report: per kernel launch, duration, DRAM
bytes, throughputs, occupancy, top stall reasons.  Usage:
  python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--json out.json]"""
import csv
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "ms",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "l1tex__throughput.avg.pct_of_peak_sustained_active": "l1_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occ_pct",
    "launch__registers_per_thread": "regs",
    "smsp__inst_executed.sum": "inst",
    "launch__grid_size": "grid",
}


def load(rep):
    if rep.endswith(".csv"):  # raw page exported on the GPU box (ncu -i rep --page raw --csv)
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    stall_cols = [i for i, h in enumerate(hdr) if h.startswith("smsp__average_warp_latency_issue_stalled_")
                  or h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio")]
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")][:80]}
        for k, v in KEYS.items():
            if k in hdr:
                i = hdr.index(k)
                val = float(r[i].replace(",", "")) if r[i] else 0.0
                u = units[i]
                if v in ("dram_read", "dram_write"):
                    val *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
                            "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
                if v == "ms":
                    val *= {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1, "ms": 1,
                            "second": 1e3, "s": 1e3}.get(u, 1)
                d[v] = val
        stalls = []
        for i in stall_cols:
            try:
                stalls.append((float(r[i]), hdr[i].replace("smsp__average_warps_issue_stalled_", "")
                               .replace("_per_issue_active.ratio", "")))
            except ValueError:
                pass
        d["top_stalls"] = [f"{n}={v:.2f}" for v, n in sorted(stalls, reverse=True)[:4]]
        res.append(d)
    return res


if __name__ == "__main__":
    res = load(sys.argv[1])
    for d in res:
        gb = (d.get("dram_read", 0) + d.get("dram_write", 0)) / 1e9
        print(f"{d['kernel'][:60]:60s} {d.get('ms', 0):7.3f} ms  dram {gb:6.3f} GB "
              f"({gb / max(d.get('ms', 1e-9), 1e-9):6.2f} TB/s, {d.get('dram_pct', 0):5.1f}%)  "
              f"L1 {d.get('l1_pct', 0):5.1f}% L2 {d.get('l2_pct', 0):5.1f}% occ {d.get('occ_pct', 0):5.1f}% "
              f"regs {d.get('regs', 0):.0f}  {' '.join(d['top_stalls'])}")
    if "--json" in sys.argv:
        json.dump(res, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)
