import os, sys, time, json
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth
n=512; steps=int(sys.argv[1]) if len(sys.argv) > 1 else 20; cells=n**3
g = nb.Grid((n,n,n), devices=[0])
stream = torch.cuda.ExternalStream(g.stream())
b, x = nb.Field(g), nb.Field(g)
bh = torch.from_numpy(synth.poisson_poly_rhs((n,n,n)).reshape(-1)).pin_memory()
xh = torch.zeros(cells, dtype=torch.float64).pin_memory()
def e2e(log):
    t=[time.perf_counter()]
    b.upload_async(bh.data_ptr()); t.append(time.perf_counter())
    x.upload_async(xh.data_ptr()); t.append(time.perf_counter())
    s = nb.CG(x, b, occ=nb.OCC_TWO_WAY); t.append(time.perf_counter())
    s.prepare(steps); t.append(time.perf_counter())
    s.iterate(steps); t.append(time.perf_counter())
    s.finish(); t.append(time.perf_counter())
    s.close(); t.append(time.perf_counter())
    x.download(xh); t.append(time.perf_counter())
    if log: print([round((t[i+1]-t[i])*1e3,2) for i in range(len(t)-1)], flush=True)
for k in range(4):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream); e2e(True); e1.record(stream); torch.cuda.synchronize()
    print('gpu span ms', e0.elapsed_time(e1))
