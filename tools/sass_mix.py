"""Dynamic instruction mix of one kernel launch from an ncu source page
(--page source --csv --print-source sass): executed warp instructions per
cell by opcode, and the warp-stall samples attributed to each opcode.
  python tools/sass_mix.py <sass.csv> <cells> [title]"""
import collections
import csv
import sys

path, cells = sys.argv[1], float(sys.argv[2])
title = sys.argv[3] if len(sys.argv) > 3 else path
rows = list(csv.reader(open(path)))
hdr = rows[1]
iS, iE = hdr.index("Source"), hdr.index("Instructions Executed")
iW = hdr.index("Warp Stall Sampling (All Samples)")
name = rows[0][1] if len(rows[0]) > 1 else "?"
mix, stall = collections.Counter(), collections.Counter()
for r in rows[2:]:
    op = r[iS].strip().split()
    if not op:
        continue
    o = op[1] if op[0].startswith("@") and len(op) > 1 else op[0]
    o = o.split(".")[0]
    mix[o] += int(r[iE] or 0)
    stall[o] += int(r[iW] or 0)
tot = sum(mix.values())
tstall = max(sum(stall.values()), 1)
print(f"# {title}: {name[:100]}")
print(f"# executed instructions per cell (thread view): {tot * 32 / cells:.1f}")
print(f"{'opcode':10s} {'per cell':>9s} {'stall %':>8s}")
for o, c in mix.most_common(20):
    print(f"{o:10s} {c * 32 / cells:9.2f} {100.0 * stall[o] / tstall:8.1f}")
