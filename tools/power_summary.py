"""Summarise gpurun_out/power_{cg,lbm}.log and copy_sustained.json (written by
tools/gpu/final_r1.sh) into profiles/power_<round>.json."""
import json
import os
import sys

R = sys.argv[1] if len(sys.argv) > 1 else "r1"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GO = os.path.join(ROOT, "gpurun_out")
out = {}
for w in ("cg", "lbm"):
    L = open(os.path.join(GO, f"power_{w}.log")).read().splitlines()
    v = [float(x) for x in L[0].split(":")[1].split()]
    rows = []
    for s in (l.strip() for l in L[2:] if l.strip()):
        t, rest = s.split("s", 1)
        f = [x.strip() for x in rest.split(",")]
        rows.append({"t_s": float(t), "sm_mhz": int(f[0]), "mem_mhz": int(f[1]), "power_w": float(f[2]), "reasons": f[3]})
    late = [r for r in rows if r["t_s"] > 0.8 * rows[-1]["t_s"]]
    out[w] = {"ms_per_step_per_chunk": v, "first3_mean": sum(v[:3]) / 3, "last20_mean": sum(v[-20:]) / 20,
              "late_sm_mhz_median": sorted(r["sm_mhz"] for r in late)[len(late) // 2] if late else None,
              "late_power_w_max": max(r["power_w"] for r in late) if late else None, "samples": rows}
c = json.load(open(os.path.join(GO, "copy_sustained.json")))
pw = [float(s.split(",")[1]) for s in c["samples"]]
out["copy"] = {"gbs_first_chunk": c["copy_gbs_first_chunk"], "gbs_best": c["copy_gbs_best"],
               "gbs_last_third_median": c["copy_gbs_last_third_median"], "sm_mhz_median_late": c["sm_mhz_median_late"],
               "power_w_max": max(pw), "reasons_seen": sorted(set(s.split(",")[2].strip() for s in c["samples"]))}
out["how"] = ("tools/power_probe.py (C2 CG 512^3 in 16-iteration graph chunks / C3 LBM 512^3 in 4-step chunks, CUDA "
              "events per chunk) and tools/copy_sustained.py (torch copy_ of 1 Gi bf16, the MEASURED_PEAKS recipe, back "
              "to back for 3 s); nvidia-smi sampled every 50 ms (power.draw is averaged by the driver, so it lags the "
              "clock response)")
json.dump(out, open(os.path.join(ROOT, "profiles", f"power_{R}.json"), "w"), indent=1)
print({k: {kk: vv for kk, vv in v.items() if kk not in ("samples", "ms_per_step_per_chunk")} if isinstance(v, dict) else v
       for k, v in out.items() if k != "how"})
