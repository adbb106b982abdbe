"""Attribution timing in the bench context: alone, after rank, after detect + rank.  python tools/attr_ctx_probe.py [lib]"""
import sys, os
sys.path.insert(0, '/root/repo')
import torch, numpy as np
if len(sys.argv) > 1:
    from paper_conf_sc_senvs23_b200 import binding
    binding.load_library(sys.argv[1])
import bench, paper_conf_sc_senvs23_b200 as g
from gen.device import DeviceTrace
s, tr = bench.build_workload('C4', 'trace')
words = DeviceTrace(tr).packed()
torch.cuda.set_stream(torch.cuda.Stream())
st = torch.cuda.current_stream()
ctx = g.Context(n_reasons=19, hist_row=19)
ctx.load_sass(s.text)
hist = torch.empty(ctx.n_instr * 19, dtype=torch.int32, device='cuda')
ninv = torch.zeros(1, dtype=torch.int64, device='cuda')
ctx.detect()
out = torch.empty(ctx.sites_device()[2] * g.RANKED_DTYPE.itemsize, dtype=torch.uint8, device='cuda')
def run(mode, iters=20):
    ts = []
    for i in range(iters + 3):
        if mode in ('full',):
            ctx.detect()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        if mode != 'nozero':
            ninv.zero_()
        ctx.attribute_samples(words, hist, ninv)
        e1.record(st)
        if mode in ('full', 'rank'):
            ctx.rank_sites(hist, out=out)
        torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1))
    return np.mean(ts), np.min(ts)
for m in ('alone', 'nozero', 'rank', 'full', 'alone'):
    print(m, run(m))
