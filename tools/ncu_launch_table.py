"""Per-kernel averages of an ncu --csv launch list with several metrics (one row per kernel name).

    python tools/ncu_launch_table.py <launches.csv>
"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
agg = collections.OrderedDict()
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    n = r[ki].split("(")[0].split("::")[-1][:40]
    agg.setdefault(n, collections.defaultdict(list))[r[mi]].append(float(r[vi].replace(",", "")))
ms = sorted({m for d in agg.values() for m in d})
print(f"{'kernel':40s} " + " ".join(f"{m[:28]:>28s}" for m in ms))
for n, d in agg.items():
    print(f"{n:40s} " + " ".join(f"{sum(d[m]) / len(d[m]):28.1f}" if d[m] else " " * 28 for m in ms))
