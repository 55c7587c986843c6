"""Per-opcode executed-instruction mix from an ncu source page export
(ncu -i X.ncu-rep --page source --csv --print-source sass): one kernel
section, counts per unit (e.g. per node).
  python tools/sass_counts.py file.csv <section-index> <units> [--hot out.txt]"""
import collections
import csv
import sys

path, idx, units = sys.argv[1], int(sys.argv[2]), float(sys.argv[3])
lines = open(path).read().split("\n")
starts = [i for i, l in enumerate(lines) if l.startswith('"Kernel Name"')] + [len(lines)]
sec = lines[starts[idx]:starts[idx + 1]]
print(sec[0][:150])
rows = list(csv.reader(sec[1:]))
hdr, rows = rows[0], rows[1:]
iA, iS = hdr.index("Address"), hdr.index("Source")
iW, iSm = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
cnt, stl = collections.Counter(), collections.Counter()
hot = []
for r in rows:
    if len(r) <= iW or not r[iS].strip():
        continue
    op = r[iS].split()
    o = (op[1] if op[0].startswith("@") else op[0]).split(".")[0]
    w, sm = int(r[iW] or 0), int(r[iSm] or 0)
    cnt[o] += w
    stl[o] += sm
    if w * 32 / units > 0.05:
        hot.append(f"{r[iA][-5:]} {w * 32 / units:7.2f} {sm:6d}  {r[iS][:100]}")
S = max(1, sum(stl.values()))
print(f"warp-instructions x 32 per unit: {sum(cnt.values()) * 32 / units:.1f}")
for o, w in cnt.most_common(25):
    print(f"  {o:10s} {w * 32 / units:8.2f}  stall% {100 * stl[o] / S:5.1f}")
if "--hot" in sys.argv:
    open(sys.argv[sys.argv.index("--hot") + 1], "w").write("\n".join(hot))
