"""Times gs_attribute_samples with a pinned HOST sample buffer (H2D inside the call) on the bench
workload.   python tools/time_e2e.py [--lib PATH] [--iters N]"""
import argparse, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
ap = argparse.ArgumentParser(); ap.add_argument("--lib"); ap.add_argument("--iters", type=int, default=5)
a = ap.parse_args()
import torch
from paper_conf_sc_senvs23_b200 import binding
if a.lib:
    binding.load_library(a.lib)
import bench
from gen.device import DeviceTrace
s, tr = bench.build_workload("C4", "trace")
words = DeviceTrace(tr).packed()
host = torch.empty(words.numel(), dtype=torch.int32, pin_memory=True)
host.copy_(words)
ctx = binding.Context(hist_row=19)
ctx.load_sass(s.text)
hist = torch.empty(ctx.n_instr * 19, dtype=torch.int32, device="cuda")
ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
ctx.attribute_samples(host, hist, ninv)
torch.cuda.synchronize()
t = time.perf_counter()
for _ in range(a.iters):
    ctx.attribute_samples(host, hist, ninv)
torch.cuda.synchronize()
dt = (time.perf_counter() - t) / a.iters
print(f"lib={a.lib}: {dt * 1e3:.2f} ms, {4 * tr.N / dt / 1e9:.1f} GB/s H2D, {tr.N / dt / 1e9:.2f} G samples/s, ok={torch.equal(hist.view(-1, 19).sum(1).cpu(), torch.from_numpy(tr.table[:, :19].sum(1)).int())}")
