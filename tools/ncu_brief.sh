# brief ncu readout of a report: duration, pipes, stall samples, per-opcode mix
# usage: tools/ncu_brief.sh report.ncu-rep nodes
R=$1; N=${2:-56623104}
ncu -i $R --page details 2>/dev/null | grep -E '^  [a-z_]|Duration|DRAM Throughput|Issue Slots Busy|Executed Ipc A|Warp Cycles Per Issued|Achieved Occ|Registers Per' | head -12
ncu -i $R --page raw --csv 2>/dev/null | python3 -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h=rows[0]; v=rows[2]
want=('l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed','l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed','sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active','dram__bytes_read.sum','dram__bytes_write.sum')
st=[(k.replace('smsp__pcsamp_warps_issue_stalled_',''),float(x or 0)) for k,x in zip(h,v) if k.startswith('smsp__pcsamp_warps_issue_stalled') and 'not_issued' not in k]
for k,x in zip(h,v):
    if k in want: print(k,x)
tot=sum(x for _,x in st)
print('stalls:', ', '.join('%s %.0f%%'%(k,100*x/tot) for k,x in sorted(st,key=lambda t:-t[1])[:8]))
"
ncu -i $R --page source --csv --print-source sass 2>/dev/null > /tmp/_sass.csv
python3 - $N <<'PY'
import csv,sys
from collections import Counter
N=float(sys.argv[1])
rows=list(csv.reader(open('/tmp/_sass.csv'))); h=rows[1]; data=rows[2:]
ix={k:i for i,k in enumerate(h)}
f=lambda r,k: float(r[ix[k]] or 0) if r[ix[k]] not in ('','-') else 0.0
ti=sum(f(r,'Instructions Executed') for r in data)
print('instr/node %.0f'%(ti*32/N))
c=Counter(); s=Counter(); ts=sum(f(r,'Warp Stall Sampling (All Samples)') for r in data)
for r in data:
    t=r[ix['Source']].split()
    if not t: continue
    op=(t[1] if t[0].startswith('@') else t[0]).split('.')[0]
    c[op]+=f(r,'Instructions Executed'); s[op]+=f(r,'Warp Stall Sampling (All Samples)')
print(' '.join('%s:%.0f(%.0f%%)'%(o,n*32/N,100*s[o]/ts) for o,n in c.most_common(12)))
PY
