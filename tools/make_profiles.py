"""Turn a round's gpurun_out/ ncu artefacts into the committed summaries
under profiles/ (launch shares, per-kernel ncu metrics, ncu_traffic.json).
  python tools/make_profiles.py r1"""
import collections
import csv
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import ncu_summary  # noqa: E402

R = sys.argv[1] if len(sys.argv) > 1 else "r1"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles")
GO = os.path.join(ROOT, "gpurun_out")
os.makedirs(OUT, exist_ok=True)

# kernel label (the name bench.py / nb_profile_read use) from the ncu name
LABELS = [("k_sp_runs<4>", "k_sp_cg_q"), ("k_sp_runs<2>", "k_sp_cg_init"), ("k_sp_fem<1>", "k_sp_fem_q"),
          ("k_sp_fem<0>", "k_sp_fem_apply"), ("k_sp_fem<2>", "k_sp_fem_init"), ("k_cgA_tma", "k_msr_cgA"), ("k_cgB_tma", "k_cg_B"), ("k_msr_fast<1, 1>", "k_msr_cgA"),
          ("k_msr_fast<0", "k_msr_c1"), ("MsrOp<1, 1, 1>", "k_msr_cgA"), ("MsrOp<0,", "k_msr_c1"),
          ("CgBOp", "k_cg_B"), ("CgInitOp", "k_cg_init"), ("Lap7Op", "k_laplace7"), ("k_map_u", "k_map_u"),
          ("k_lbm_d3q19", "k_lbm_d3q19"), ("k_finalize", "k_finalize"), ("k_sp<3>", "k_sp_cg_map"),
          ("k_sp<4>", "k_sp_cg_q"), ("k_sp<5>", "k_sp_cg_r"), ("k_sp<2>", "k_sp_cg_init"),
          ("k_fem_tma<1", "k_fem_cg_q"), ("k_fem_tma<2", "k_fem_cg_init"), ("k_fem_tma<3", "k_fem_cg_a"),
          ("k_fem_tma<0", "k_fem_apply"), ("k_fem_faces", "k_fem_faces"),
          ("k_fem_surface", "k_fem_surface"), ("k_fem_xface", "k_fem_xface"), ("k_fem<1>", "k_fem_cg_q"), ("k_fem<2>", "k_fem_cg_init"),
          ("k_fem_map", "k_fem_map"), ("k_fem_r(", "k_fem_r"), ("k_fem_rhs", "k_fem_rhs"),
          ("k_halo_copy", "k_halo_copy"), ("k_peer_ops", "k_peer_ops")]


def label(name):
    for pat, lab in LABELS:
        if pat in name:
            return lab
    return name.split("(")[0]


# 1. launch shares of the bench command
lines = []
lc = os.path.join(GO, f"launches_{R}.csv")
if os.path.exists(lc):
    rows = [r for r in csv.reader(open(lc)) if len(r) > 10 and r[0] != "ID"]
    cnt, tot = collections.Counter(), collections.Counter()
    for r in rows:
        n = label(r[4])
        cnt[n] += 1
        tot[n] += float(r[-1]) / 1e3  # ns -> us
    s = sum(tot.values())
    lines.append(f"# ncu launch list of `python bench.py --steps 3 --warmup 3 --no-extras` ({R})")
    lines.append("# gpu__time_duration.sum, --clock-control none; cold-cache serialised: compare SHARES")
    lines.append(f"{'kernel':24s} {'launches':>8s} {'total_us':>12s} {'avg_us':>10s} {'share':>7s}")
    for n in sorted(tot, key=tot.get, reverse=True):
        lines.append(f"{n:24s} {cnt[n]:8d} {tot[n]:12.1f} {tot[n] / cnt[n]:10.1f} {tot[n] / s:7.1%}")
    open(os.path.join(OUT, f"{R}_launch_shares.txt"), "w").write("\n".join(lines) + "\n")

# 2. ncu --set full summaries + traffic per launch
traffic = {}
tp = os.path.join(OUT, "ncu_traffic.json")
if os.path.exists(tp):
    traffic = json.load(open(tp))
for rep in sorted(os.listdir(GO)):
    if not (rep.startswith(f"prof_{R}_") and rep.endswith((".ncu-rep", ".raw.csv"))):
        continue
    if rep.endswith(".ncu-rep") and os.path.exists(os.path.join(GO, rep.replace(".ncu-rep", ".raw.csv"))):
        continue
    res = ncu_summary.load(os.path.join(GO, rep))
    out = [f"# ncu --set full --clock-control none summary of {rep} ({R})",
           f"{'kernel':18s} {'ms':>8s} {'dram_GB':>8s} {'TB/s':>6s} {'L1%':>5s} {'L2%':>5s} {'occ%':>5s} "
           f"{'regs':>4s}  top stalls (cycles per issued instruction)"]
    per = collections.defaultdict(list)
    for d in res:
        lab = label(d["kernel"])
        gb = (d.get("dram_read", 0) + d.get("dram_write", 0)) / 1e9
        out.append(f"{lab:18s} {d.get('ms', 0):8.3f} {gb:8.3f} {gb / max(d.get('ms', 1e-9), 1e-9):6.2f} "
                   f"{d.get('l1_pct', 0):5.1f} {d.get('l2_pct', 0):5.1f} {d.get('occ_pct', 0):5.1f} "
                   f"{d.get('regs', 0):4.0f}  {' '.join(d['top_stalls'])}")
        per[lab].append(d.get("dram_read", 0) + d.get("dram_write", 0))
    for lab, v in per.items():
        traffic[lab] = max(v)  # the steady-state launch (x update active) is the largest
    open(os.path.join(OUT, rep.replace(".ncu-rep", ".txt").replace(".raw.csv", ".txt")), "w").write("\n".join(out) + "\n")
json.dump(traffic, open(tp, "w"), indent=1, sort_keys=True)
print("\n".join(lines))
print(json.dumps(traffic, indent=1))
