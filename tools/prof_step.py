"""Profiling driver: sets up the bench workload and runs a few steps (for ncu / nsys-less runs).

    python tools/prof_step.py [--config C4] [--order trace] [--mode 0] [--steps 3] [--only hist|detect|rank|all]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_senvs23_b200 as g  # noqa: E402
from gen.device import DeviceTrace  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--order", default="trace")
ap.add_argument("--mode", type=int, default=0)
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--only", default="all")
ap.add_argument("--lib", default=None)
a = ap.parse_args()
if a.lib:
    from paper_conf_sc_senvs23_b200 import binding
    binding.load_library(a.lib)
s, tr = bench.build_workload(a.config, a.order)
words = DeviceTrace(tr).packed()
ctx = g.Context(hist_mode=a.mode, hist_row=19)   # compact rows, as bench.py
ctx.load_sass(s.text)
hist = torch.empty(ctx.n_instr * 19, dtype=torch.int32, device="cuda")
ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
ctx.detect()
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
for _ in range(a.steps):
    if a.only in ("all", "detect"):
        ctx.detect()
    if a.only in ("all", "hist"):
        ctx.attribute_samples(words, hist, ninv)
    if a.only in ("all", "rank"):
        ctx.rank_sites(hist, k=None)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("ok", ctx.last_hist_mode())
