"""Summaries of ncu outputs for profiles/: launch list shares and key raw metrics of a capture.

    python tools/ncu_summary.py launches <launches.csv> [steps]
    python tools/ncu_summary.py kernel <report.ncu-rep>
"""
import collections
import csv
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed_op_shared_atom.sum",
        "smsp__inst_executed_op_global_red.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__cycles_active.avg", "gpc__cycles_elapsed.max"]


SETUP_KERNELS = ("k_expand", "at::", "at_cuda_detail", "curand", "distribution_elementwise")


def launches(path, steps=1):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    mi = h.index("Metric Name") if "Metric Name" in h else -1
    agg = collections.OrderedDict()
    skipped = collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        if mi >= 0 and r[mi] != "gpu__time_duration.sum":  # launch lists may carry other metrics
            continue
        if any(x in r[ki] for x in SETUP_KERNELS):  # input generation before the timed region
            skipped[r[ki].split("(")[0][-40:]] += 1
            continue
        scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}.get(r[ui], 1.0)
        name = r[ki].split("(")[0].replace("gs::<unnamed>::", "").replace("void ", "")[:70]
        agg.setdefault(name, []).append(float(r[vi].replace(",", "")) * scale)
    tot = sum(sum(v) for v in agg.values()) / steps
    print(f"{'us/step':>10} {'share':>6} {'n':>4}  kernel")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"{sum(v) / steps:10.1f} {100 * sum(v) / steps / tot:5.1f}% {len(v) // steps:4d}  {k}")
    print(f"{tot:10.1f} us per step (serialised, cold-cache ncu replay)")
    if skipped:
        print("  not counted (workload generation, outside the timed steps):",
              ", ".join(f"{k} x{v}" for k, v in skipped.items()))


def kernel(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(out.splitlines()))
    h, v = r[0], r[2] if len(r) > 2 else r[1]
    d = dict(zip(h, v))
    print("kernel:", d.get("Kernel Name", "?")[:100])
    for k in KEYS:
        print(f"  {k} = {d.get(k)}")
    st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(d[k].replace(",", "")) for k in d
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
          and d[k].replace(",", "").replace(".", "").isdigit()}
    tot = sum(st.values()) or 1
    print("  stall reasons (pc samples):", ", ".join(f"{k} {100 * v / tot:.1f}%" for k, v in
                                                  sorted(st.items(), key=lambda kv: -kv[1]) if v / tot > 0.01))


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 1)
    else:
        kernel(sys.argv[2])
