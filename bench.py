#!/usr/bin/env python
"""Benchmark of the batched bottleneck-attribution hot path (SURVEY §8a rows a-2 .. a-12).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--order trace|shuffled]
    python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N   (N > 1, NCCL)
    python bench.py --impl reference      (the CPU oracle, timed on the host cores)

One step = one pass of the whole path over one batch: gs_detect (reaching defs, loop marks, traces,
rules, compaction) over this rank's kernels + gs_attribute_samples (histogram of this rank's
sample shard, compact R-bin rows) + [reduce-scatter of the histogram by the kernel-aligned slot
ranges of the detection shards] + gs_rank_sites_slice (join + rank of this rank's sites against
its summed slice, rows to a device buffer). Inputs (packed SASS records, packed samples) are resident in HBM before the
timed region. Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "PC stall samples attributed/s + SASS instrs scanned/s per GPU; % HBM peak; 1/2/4/8 GPU"
UNIT = "samples/s"
WORKLOADS = {
    # name: (sass config, samples)
    "C2": ("C2", 10_000_000),
    "C4": ("C4", 1 << 30),
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ----------------------------------------------------------------------------------- workload
def build_workload(name: str, order: str, seed: int = 1):
    from gen import samples as gsm
    from gen import sass as gsass
    cfg, n = WORKLOADS[name]
    s = gsass.config_sass(cfg)
    if name == "C4":
        tab = gsm.table_c4(s.cls, s.first_slot, s.n_instr, n, key=0x6E5C0004)
    else:
        tab = gsm.table_class_weighted(s.cls, n, key=0x6E5C0002)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order=order, seed=seed)
    return s, tr


def read_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampler for the timed region (B200_PROFILING.md clocks line)."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index: int):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.06)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=1)
        sm = [float(r[0]) for r in self.rows if len(r) >= 6 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 6 and r[1].replace(".", "").isdigit()]
        reasons = sorted({self.NAMES[i] for r in self.rows if len(r) >= 6 for i in range(4)
                          if r[2 + i].lower().startswith("active")})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


# ----------------------------------------------------------------------------------- oracle leg
def oracle_sample(tr, s, n_sample: int):
    """Bounded sample of the workload for the CPU oracle: the full SASS text + every stride-th
    sample of the trace (in stream order) as raw (kernel, pc, reason) triples."""
    stride = max(1, tr.N // n_sample)
    pos = np.arange(0, tr.N, stride, dtype=np.int64)[:n_sample]
    return tr.raw_at(pos), stride


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def run_oracle_step(s, raw, shards: int, td: str):
    """One oracle step on the bounded sample, timed as it runs (wall clock of the oracle
    processes): shards == 1 is the plain single-threaded oracle; shards > 1 runs independent
    kernel ranges (with their samples) in parallel and merges (tests/oracle_run.run_sharded)."""
    import oracle_run
    if shards == 1:
        sp, rp = os.path.join(td, "sass.txt"), os.path.join(td, "raw.bin")
        if not os.path.exists(sp):
            open(sp, "wb").write(s.text)
            raw.tofile(rp)
        exe = oracle_run.build_oracle()
        t0 = time.perf_counter()
        p = subprocess.run([exe, "--sass", sp, "--samples", rp, "--quiet", "--time"], capture_output=True, text=True)
        wall = time.perf_counter() - t0
        if p.returncode != 0:
            raise RuntimeError(p.stderr)
        t = {"wall": wall}
        for line in p.stderr.splitlines():
            if line.startswith("TIME"):
                for kv in line.split()[1:]:
                    k, v = kv.split("=")
                    t[k] = float(v)
        return t
    _, wall = oracle_run.run_sharded(s.text, raw, s.n_instr, shards, timing=True, tmpdir=td)
    return {"wall": wall}


def oracle_baseline(s, tr, n_sample: int, steps: int = 1, warmup: int = 0, one_core: bool = True):
    """cpu_baseline: the oracle as it stands on this box's host cores, on a bounded sample of the
    workload (the full SASS + n_sample samples); value = samples in the step / measured step time
    (no extrapolation). Returns (all-cores entry with the 1-core entry inside, median step s)."""
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    raw, stride = oracle_sample(tr, s, n_sample)
    ns = len(raw)
    cores = host_cores()
    sample = (f"full {len(s.n_instr)}-kernel SASS ({s.P} instrs: parse, detection, join, rank) + every {stride}-th "
              f"sample of the trace ({ns} of {tr.N}); value = {ns} samples / measured step time")
    out = {}
    with tempfile.TemporaryDirectory() as td1, tempfile.TemporaryDirectory() as tdn:
        for label, shards, td in (("one", 1, td1), ("all", cores, tdn)):
            if label == "one" and not one_core:
                continue
            ts = []
            for i in range(warmup + steps):
                t = run_oracle_step(s, raw, shards, td)
                if i >= warmup:
                    ts.append(t["wall"])
            med = float(np.median(ts))
            out[label] = {"value": ns / med, "unit": UNIT, "cores": shards, "kind": "oracle",
                          "sample": sample + ("" if shards == 1 else
                                              f"; {shards} single-threaded oracle processes on kernel ranges "
                                              f"balanced by instruction count, merged by integer sums"),
                          "ms_per_step": med * 1e3}
    best = dict(out["all"])
    if "one" in out:
        best["one_core"] = out["one"]
    return best, best["ms_per_step"] / 1e3


# ----------------------------------------------------------------------------------- reference arm
def reference_arm(args, world, rank):
    """The CPU oracle (there is no reference code: /root/reference holds only the paper): every
    step runs the all-cores oracle on the bounded sample and is timed as it runs."""
    if rank != 0:
        return
    s, tr = build_workload(args.config, args.order)
    cpu, step_s = oracle_baseline(s, tr, args.cpu_samples, steps=args.steps, warmup=args.warmup, one_core=False)
    value = cpu["value"]
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": step_s * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": workload_config(args, s, tr, world),
        "cpu_baseline": cpu,
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ----------------------------------------------------------------------------------- extra lines
def _time_events(fn, steps, warmup, stream):
    """mean ms of fn() over `steps` calls, CUDA events on `stream`, after `warmup` calls"""
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def extra_detect_c3(g, peak, steps, warmup):
    """configs[2] (C3: 10,000 kernels, ~50M SASS instructions; the paper's dry run):
    gs_load_sass host parse+pack+upload (wall) and gs_detect (CUDA events). Algorithmic bytes
    (SURVEY §8d): 16 B read per instruction + 16 B per site + 4 B per chain step written."""
    import torch
    from gen import sass as gsass
    s3 = gsass.config_sass("C3")
    ctx = g.Context(n_reasons=19)
    t0 = time.perf_counter()
    ctx.load_sass(s3.text)
    torch.cuda.synchronize()
    parse_s = time.perf_counter() - t0
    n_sites = ctx.detect()
    _, _, ns, nc = ctx.sites_device()
    ms = _time_events(ctx.detect, steps, warmup, torch.cuda.current_stream())
    alg = 16.0 * ctx.n_instr + 16.0 * ns + 4.0 * nc
    ach = alg / (ms * 1e-3) / 1e9
    return {"workload": "C3", "kernels": ctx.n_kernels, "sass_instrs": ctx.n_instr, "sites": int(n_sites),
            "chain_steps": int(nc), "detect_ms": ms, "instrs_per_s": ctx.n_instr / (ms * 1e-3),
            "host_parse_pack_upload_s": parse_s, "text_bytes": len(s3.text),
            "roofline": {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                         "algorithmic_bytes": alg}}


def extra_c5(g, peak, steps, warmup):
    """configs[4] (C5: 200M samples, 90% on 10 PCs, a 1M-PC module with 63/64/65-step chains):
    the attribution pass in both orders (trace: AUTO, shuffled: PARTITION, as the main line)."""
    import torch
    from gen import samples as gsm
    from gen import sass as gsass
    from gen.device import DeviceTrace
    s5 = gsass.config_sass("C5")
    hot = [int(f) + 40 for f in s5.first_slot[:10]]
    tab = gsm.table_c5(s5.cls, hot, 200_000_000, key=0x6E5C0005)
    out = {"workload": "C5", "samples": int(tab.sum()), "sass_instrs": int(sum(s5.n_instr))}
    R = 19
    for order, mode in (("trace", 0), ("shuffled", g.GS_HIST_PARTITION)):
        tr = gsm.Trace(tab, s5.first_slot, s5.n_instr, order=order, seed=2)
        words = DeviceTrace(tr, torch.cuda.current_device()).packed()
        ctx = g.Context(n_reasons=R, hist_mode=mode, hist_row=R)
        ctx.load_sass(s5.text)
        hist = torch.empty(ctx.n_instr * R, dtype=torch.int32, device="cuda")
        ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
        ms = _time_events(lambda: ctx.attribute_samples(words, hist, ninv), steps, warmup,
                          torch.cuda.current_stream())
        assert int(hist.to(torch.int64).sum().item()) == tr.N
        alg = 4.0 * tr.N + 4.0 * R * ctx.n_instr
        ach = alg / (ms * 1e-3) / 1e9
        out[order] = {"attribute_ms": ms, "samples_per_s": tr.N / (ms * 1e-3), "hist_mode": ctx.last_hist_mode(),
                      "roofline": {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                                   "algorithmic_bytes": alg}}
        del words, hist
    return out


def extra_pack_hist(g, ctx, words, hist, ninv, s, peak, steps, warmup):
    """N1 + N2 (SURVEY §8d timing protocol): raw 12-byte (kernel, pc offset, reason) records of the
    same trace through gs_pack_samples, then the histogram. The raw records are built on the device
    from the packed words (input preparation, not timed)."""
    import torch
    R = 19
    n = words.shape[0]
    first = torch.from_numpy(np.asarray(s.first_slot, dtype=np.int64)).cuda()
    raw = torch.empty((n, 3), dtype=torch.int32, device="cuda")
    chunk = 1 << 26
    for a in range(0, n, chunk):
        w = words[a:a + chunk].to(torch.int64)
        slot, reason = w // R, w % R
        k = torch.searchsorted(first, slot, right=True) - 1
        raw[a:a + chunk, 0] = k.to(torch.int32)
        raw[a:a + chunk, 1] = ((slot - first[k]) * 16).to(torch.int32)
        raw[a:a + chunk, 2] = reason.to(torch.int32)
        del w, slot, reason, k
    packed = torch.empty(n, dtype=torch.int32, device="cuda")
    pinv = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.current_stream()
    pack_ms = _time_events(lambda: ctx.pack_samples(raw, packed, pinv), steps, warmup, st)
    assert torch.equal(packed, words)

    def both():
        ctx.pack_samples(raw, packed, pinv)
        ctx.attribute_samples(packed, hist, ninv)
    both_ms = _time_events(both, steps, warmup, st)
    del raw, packed
    alg_pack = 16.0 * n            # 12 B read + 4 B written per record
    alg_both = alg_pack + 4.0 * n + 4.0 * R * ctx.n_instr
    return {"samples": n, "pack_ms": pack_ms, "pack_plus_hist_ms": both_ms,
            "samples_per_s": n / (both_ms * 1e-3),
            "pack_roofline": {"achieved": alg_pack / (pack_ms * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                              "frac": alg_pack / (pack_ms * 1e-3) / 1e9 / peak},
            "roofline": {"achieved": alg_both / (both_ms * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                         "frac": alg_both / (both_ms * 1e-3) / 1e9 / peak, "algorithmic_bytes": alg_both}}


def extra_cupti(g, s, peak, steps, warmup):
    """CUPTI ingest: the C4 count table as CUpti_PCSamplingPCData host records (one
    per PC, all-samples + not-issued counters per reason) through gs_attribute_cupti: host flattening
    into pinned memory, one H2D copy, the weighted device scatter-add. Wall clock per call (the host
    part dominates), records/s and the samples they represent per second."""
    import torch
    from gen import cupti
    from gen import samples as gsm
    tab = gsm.table_c4(s.cls, s.first_slot, s.n_instr, 1 << 30, key=0x6E5C0004)
    names = [ln.split(b"Function : ")[1].split()[0].decode() for ln in s.text.split(b"\n") if b"Function : " in ln]
    buf = cupti.FastBuffer(tab, names, s.first_slot)
    R = 19
    ctx = g.Context(n_reasons=R, hist_row=R)
    ctx.load_sass(s.text)
    ctx.cupti_stall_reasons(*buf.table_ptrs())
    hist = torch.empty(ctx.n_instr * R, dtype=torch.int32, device="cuda")
    ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
    ts = []
    for i in range(warmup + steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        _, _, sk, nrec = ctx.attribute_cupti(buf.ptr(), buf.n, buf.crc, hist, ninv)
        torch.cuda.synchronize()
        if i >= warmup:
            ts.append(time.perf_counter() - t0)
    assert int(hist.to(torch.int64).sum().item()) == buf.samples and sk == buf.skipped and int(ninv.item()) == 0
    sec = float(np.median(ts))
    return {"records": buf.n, "entries": int(nrec), "samples": buf.samples, "ms_per_call": sec * 1e3,
            "records_per_s": buf.n / sec, "entries_per_s": nrec / sec, "samples_per_s": buf.samples / sec,
            "host_threads": min(16, os.cpu_count() or 1)}


def workload_config(args, s, tr, world):
    return {"workload": args.config, "kernels": len(s.n_instr), "sass_instrs": s.P, "samples": tr.N,
            "order": args.order, "reasons": 19, "trace_depth": 64, "parallelism": f"dp{world}",
            "l2": "inputs (4 B/sample) exceed the 126 MB L2; no flush needed" if tr.N * 4 > 2 * 126e6 else
                  "L2 flushed (256 MB write) before every timed step"}


# ----------------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4", choices=sorted(WORKLOADS))
    ap.add_argument("--order", default="trace", choices=["trace", "shuffled"])
    ap.add_argument("--hist-mode", type=int, default=-1,
                    help="GS_HIST_* (default: AUTO for trace order, PARTITION for the unordered stream)")
    ap.add_argument("--hist-bits", type=int, default=0, choices=[0, 16, 32])
    ap.add_argument("--hist-row32", action="store_true", help="32-bin histogram rows instead of compact R-bin rows")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-samples", type=int, default=1 << 24,
                    help="samples in the oracle's bounded sample (with the full SASS) per step")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true", help="skip the C3 detection / C5 / pack+hist lines")
    ap.add_argument("--lib", default=None, help="another build of the library (same-box A/B of diagnostic variants)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return reference_arm(args, world, rank)

    import torch
    import torch.distributed as dist
    # GS_BENCH_DEVICE / GS_BENCH_BACKEND: functional checks of the multi-rank flow on one GPU
    # (all ranks on one device over gloo); the default is one GPU per rank over NCCL
    local = int(os.environ.get("GS_BENCH_DEVICE", local))
    torch.cuda.set_device(local)
    if world > 1:
        backend = os.environ.get("GS_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    import paper_conf_sc_senvs23_b200 as g
    from paper_conf_sc_senvs23_b200 import binding, build as gbuild, dist as gdist
    from gen.device import DeviceTrace
    gbuild.build()
    if args.lib:
        binding.load_library(args.lib)
    torch.cuda.set_stream(torch.cuda.Stream())   # a non-default stream: the library may replay CUDA graphs on it

    t_setup = time.perf_counter()
    s, tr = build_workload(args.config, args.order)
    a, b = gdist.sample_range(tr.N, rank, world)
    kb, ke = gdist.kernel_range(s.n_instr, rank, world)
    words = DeviceTrace(tr, local).packed(a, b)
    n_local = b - a
    R = 19
    row = 32 if args.hist_row32 else R     # compact rows: 4*R B per slot to zero, write and reduce
    hist_mode = args.hist_mode if args.hist_mode >= 0 else (g.GS_HIST_PARTITION if args.order == "shuffled" else 0)
    ctx = g.Context(device=local, n_reasons=R, hist_mode=hist_mode, hist_counter_bits=args.hist_bits,
                    hist_row=row)
    ctx.load_sass(s.text)
    P = ctx.n_instr
    hist = torch.empty(P * row, dtype=torch.int32, device="cuda")
    s0, s1 = gdist.slot_ranges(s.first_slot, s.n_instr, world)[rank]
    ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
    n_sites = ctx.detect(kb, ke)
    ranked_dev = torch.empty(max(1, n_sites) * binding.RANKED_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    log(f"[rank {rank}] setup {time.perf_counter() - t_setup:.1f}s: {len(s.n_instr)} kernels, {P} instrs, "
        f"{n_local} samples, {n_sites} sites")
    stream = torch.cuda.current_stream()
    hist_events = []
    pass_ms = []          # per timed step: GPU time of the attribution pass (library events around its kernels)
    phase_events = []     # per timed step: events at detect | attribute | merge | rank boundaries

    last_part = [None]   # this rank's summed histogram rows of the last step
    def step(record_hist=False):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(5)] if record_hist else None
        ninv.zero_()  # (the invalid-sample counter is added to)
        if ev:
            ev[0].record(stream)
        ctx.detect(kb, ke)
        if ev:
            ev[1].record(stream)
        ctx.attribute_samples(words, hist, ninv)
        if ev:
            ev[2].record(stream)
            hist_events.append((ev[1], ev[2]))
        part = gdist.reduce_scatter_hist(hist, row, gdist.slot_ranges(s.first_slot, s.n_instr, world))
        last_part[0] = part
        if ev:
            ev[3].record(stream)
        ctx.rank_sites(part, k=None, out=ranked_dev, slot_begin=s0, slot_end=s1)
        if ev:
            ev[4].record(stream)
            phase_events.append(ev)
            pass_ms.append(ctx.last_attribute_ms())  # the pass's own events (completed by rank's read-back)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = Clocks(local)
    clocks.start()
    time.sleep(0.15)
    l0 = binding.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStart()   # ncu --profile-from-start off: the timed steps only
    ev0.record(stream)
    for _ in range(args.steps):
        step(record_hist=True)
    ev1.record(stream)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()
    if world > 1:
        dist.barrier()
    launches = binding.launch_count() - l0
    clk = clocks.stop()
    ms = ev0.elapsed_time(ev1) / args.steps
    # the dominant kernel's duration: the pass's own events (the library records them on its stream
    # right before its first and after its last enqueue), not the attribute phase, whose events
    # also hold the host's launch gap after detect's read-back
    hist_ms = float(np.mean(pass_ms))
    call_ms = float(np.mean([e0.elapsed_time(e1) for e0, e1 in hist_events]))
    phases = {name: float(np.mean([ev[i].elapsed_time(ev[i + 1]) for ev in phase_events]))
              for i, name in enumerate(["detect", "attribute", "merge", "rank"])}
    t = torch.tensor([ms, hist_ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max, hist_ms_max = float(t[0]), float(t[1])
    mode = ctx.last_hist_mode()

    # correctness guard on the bench configuration (closed form: mass and invalid count; with a
    # reduce-scatter each rank holds the summed rows of its own slot range)
    mass = torch.tensor([int(last_part[0].to(torch.int64).sum().item())], dtype=torch.int64, device="cuda")
    if world > 1:
        dist.all_reduce(mass)
    assert int(mass.item()) == tr.N and int(ninv.item()) == 0, (int(mass.item()), tr.N, int(ninv.item()))

    # roofline of the dominant kernel (the attribution pass: histogram of this rank's samples)
    peak, peak_src = read_peaks()
    alg_bytes = 4.0 * n_local + 4.0 * R * P           # samples read + histogram (R bins per slot) written once
    achieved = alg_bytes / (hist_ms_max * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"traffic_{args.config}_{args.order}.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get("dram_bytes_per_launch")
        if traffic and world > 1:   # captured on the whole stream: this rank's launch holds n_local samples
            traffic = traffic * n_local / tr.N

    # extra lines (N = 1): N1 + N2 on this trace, configs[2] detection, configs[4] attribution
    extras = {}
    if world == 1 and not args.no_extras:
        try:
            extras["pack_hist"] = extra_pack_hist(g, ctx, words, hist, ninv, s, read_peaks()[0], 10, 3)
        except Exception as e:  # noqa: BLE001
            extras["pack_hist"] = {"failed": str(e)}
        torch.cuda.empty_cache()

    # e2e: same step through the C ABI with HOST buffers (pinned), copies inside the timed region
    host_words = torch.empty(n_local, dtype=torch.int32, pin_memory=True)
    host_words.copy_(words)
    torch.cuda.synchronize()
    del words
    e2e_times = []
    n_rows = 0
    for i in range(max(1, args.e2e_steps) + 1):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ctx.detect(kb, ke)
        ninv.zero_()
        ctx.attribute_samples(host_words, hist, ninv)     # H2D streamed inside the call
        part = gdist.reduce_scatter_hist(hist, row, gdist.slot_ranges(s.first_slot, s.n_instr, world))
        rows = ctx.rank_sites(part, k=None, slot_begin=s0, slot_end=s1)   # D2H of the ranked rows
        rows = gdist.gather_ranked(rows, None)
        torch.cuda.synchronize()
        if i:
            e2e_times.append(time.perf_counter() - t0)
        n_rows = len(rows)
    te = torch.tensor([float(np.mean(e2e_times))], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_s = float(te[0])

    if world == 1 and not args.no_extras:
        del host_words
        torch.cuda.empty_cache()
        for name, fn in (("detect_C3", extra_detect_c3), ("C5", extra_c5),
                         ("cupti_C4", lambda g_, pk, st, wu: extra_cupti(g_, s, pk, st, wu))):
            try:
                extras[name] = fn(g, read_peaks()[0], 10, 3)
            except Exception as e:  # noqa: BLE001
                extras[name] = {"failed": str(e)}
            torch.cuda.empty_cache()

    if rank != 0:
        dist.destroy_process_group()
        return
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        try:
            cpu, _ = oracle_baseline(s, tr, args.cpu_samples)
        except Exception as e:  # noqa: BLE001
            cpu = {"value": None, "unit": UNIT, "cores": host_cores(), "kind": "oracle", "sample": f"failed: {e}"}

    value = tr.N / (ms_max * 1e-3)
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": workload_config(args, s, tr, world),
        "instrs_per_s": s.P / (ms_max * 1e-3),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic, "kernel": "gs_attribute_samples (histogram pass)",
                     "hist_mode": ["auto", "global", "private", "window", "partition"][mode] if 0 <= mode < 5 else mode,
                     "kernel_ms": hist_ms_max, "call_ms": call_ms, "algorithmic_bytes": alg_bytes,
                     "peak_source": peak_src},
        "clocks": clk,
        "gpu_launches": int(launches),
        "e2e": {"value": tr.N / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 4 * n_local,
                "d2h_bytes_per_step": n_rows * binding.RANKED_DTYPE.itemsize + 8,
                "ms_per_step": e2e_s * 1e3},
        "cpu_baseline": cpu,
        "sites": n_sites,
        "phases_ms": phases,
        "extra": extras,
    }
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
