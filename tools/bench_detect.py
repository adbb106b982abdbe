"""Detection-only throughput on configs[2] (C3: 10,000 kernels, ~50M SASS instructions; the paper's
dry run): host parse + pack, then gs_detect over all kernels timed with CUDA events on a
non-default stream (graph replay), SASS instructions scanned per second. The oracle's detection is
timed on a bounded sample (--cpu-scale of the module).

    python tools/bench_detect.py [--scale 1.0] [--steps 10] [--cpu-scale 0.02]
"""
import argparse, json, os, subprocess, sys, tempfile, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=float, default=1.0)
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--cpu-scale", type=float, default=0.02)
ap.add_argument("--lib", default=None, help="another build of the library (diagnostic variants)")
a = ap.parse_args()
import torch
import paper_conf_sc_senvs23_b200 as g
if a.lib:
    from paper_conf_sc_senvs23_b200 import binding
    binding.load_library(a.lib)
from gen import sass as gsass
t = time.perf_counter()
s = gsass.config_sass("C3", scale=a.scale)
t_gen = time.perf_counter() - t
torch.cuda.set_stream(torch.cuda.Stream())
ctx = g.Context(hist_row=19)
t = time.perf_counter()
ctx.load_sass(s.text)
torch.cuda.synchronize()
t_load = time.perf_counter() - t
n_sites = 0
for _ in range(3):
    n_sites = ctx.detect()
torch.cuda.synchronize()
st = torch.cuda.current_stream()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for _ in range(a.steps):
    ctx.detect()
e1.record(st)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / a.steps
# oracle detection on a bounded sample of the same recipe
sc = gsass.config_sass("C3", scale=a.cpu_scale)
import oracle_run as orc
out, err = orc.run(sc.text, hist=False, timing=True)
det_s = [float(x.split("=")[1]) for x in err.split() if x.startswith("detect_s=")][0]
line = {"metric": "SASS instrs scanned/s (detection + def-use trace, C3)", "value": s.P / ms * 1e3,
        "unit": "instrs/s", "config": {"workload": "C3", "kernels": len(s.n_instr), "sass_instrs": s.P,
        "scale": a.scale}, "ms_per_detect": ms, "sites": n_sites, "host_parse_pack_s": t_load,
        "generate_s": t_gen,
        "cpu_baseline": {"value": sc.P / det_s, "unit": "instrs/s", "cores": 1, "kind": "oracle",
                         "sample": f"C3 recipe at scale {a.cpu_scale} ({sc.P} instrs), detection only"}}
print(json.dumps(line))
