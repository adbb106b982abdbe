"""Times gs_attribute_samples alone on the bench workload (CUDA events), optionally with another
build of the library (diagnostic variants).   python tools/time_hist.py [--lib PATH] [--bits 16] [--mode 0]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
ap = argparse.ArgumentParser()
ap.add_argument("--lib", default=None)
ap.add_argument("--bits", type=int, default=0)
ap.add_argument("--mode", type=int, default=0)
ap.add_argument("--order", default="trace")
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--row", type=int, default=19, help="histogram row width (19 compact, as bench.py, or 32)")
ap.add_argument("--synthetic", action="store_true", help="2^30 words on kernel 0 only: 80%% on a hot 10%% of its bins, 20%% uniform (the atoms_occ2 stream)")
ap.add_argument("--accumulate", action="store_true", help="no histogram zeroing (timing only)")
ap.add_argument("--check", action="store_true", help="compare the histogram with the count table")
a = ap.parse_args()
import torch  # noqa: E402

from paper_conf_sc_senvs23_b200 import binding  # noqa: E402
if a.lib:
    binding.load_library(a.lib)
import bench  # noqa: E402
from gen.device import DeviceTrace  # noqa: E402

s, tr = bench.build_workload("C4", a.order)
if a.synthetic:
    nb = int(s.n_instr[0]) * 19
    g = torch.Generator(device="cuda").manual_seed(1)
    N = 1 << 30
    words = torch.empty(N, dtype=torch.int64, device="cuda")
    CH = 1 << 27
    for c0 in range(0, N, CH):
        h = torch.randint(0, 10, (CH,), device="cuda", generator=g)
        u = torch.randint(0, 1 << 31, (CH,), device="cuda", generator=g)
        words[c0:c0 + CH] = torch.where(h < 8, nb // 3 + u % (nb // 10), u % nb)
    words = words.to(torch.int32)
    tr.N = N
else:
    words = DeviceTrace(tr).packed()
ctx = binding.Context(hist_mode=a.mode, hist_counter_bits=a.bits, hist_row=a.row)
ctx.load_sass(s.text)
hist = torch.empty(ctx.n_instr * a.row, dtype=torch.int32, device="cuda")
ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
for _ in range(3):
    ctx.attribute_samples(words, hist, ninv)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(a.iters):
    ctx.attribute_samples(words, hist, ninv, accumulate=a.accumulate)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / a.iters
print(f"lib={a.lib or 'default'} bits={a.bits} mode={a.mode} order={a.order}: {ms:.3f} ms, "
      f"{tr.N / ms / 1e6:.1f} G samples/s, frac {(4 * tr.N + 4 * a.row * ctx.n_instr) / ms / 1e6 / 6549.8:.3f} "
      f"n_invalid {int(ninv.item())}")
if a.check and not a.synthetic:
    import numpy as np
    want = tr.table[:, :a.row].reshape(-1) if a.row <= tr.table.shape[1] else None
    got = hist.cpu().numpy().astype(np.int64)
    print("check:", "OK" if np.array_equal(got, want) else f"MISMATCH ({int((got != want).sum())} bins)")
