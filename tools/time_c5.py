"""Times the attribution pass on configs[4] (C5: 200M samples, 90% on 10 PCs) in both orders.
    python tools/time_c5.py [--lib PATH] [--iters 20]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
ap = argparse.ArgumentParser()
ap.add_argument("--lib", default=None)
ap.add_argument("--iters", type=int, default=20)
a = ap.parse_args()
import torch  # noqa: E402

from paper_conf_sc_senvs23_b200 import binding  # noqa: E402
if a.lib:
    binding.load_library(a.lib)
import bench  # noqa: E402
import paper_conf_sc_senvs23_b200 as g  # noqa: E402

r = bench.extra_c5(g, bench.read_peaks()[0], a.iters, 3)
print(f"lib={a.lib or 'default'} C5 trace {r['trace']['attribute_ms']:.3f} ms, shuffled {r['shuffled']['attribute_ms']:.3f} ms")
