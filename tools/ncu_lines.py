"""Per-source-line summary of an ncu capture taken with --import-source on (-lineinfo build):
warp-stall samples and warp instructions executed per CUDA line of one kernel.

    python tools/ncu_lines.py <report.ncu-rep> <kernel regex> [top]
"""
import csv
import io
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", "regex:" + kre, "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname = ""
lines = []
hdr = None
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    elif len(r) > 3 and r[0] == "Line No":
        hdr = r
    elif hdr and len(r) == len(hdr) and r[0] not in ("", "Line No") and r[2] == "-":
        si, ii = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
        try:
            lines.append((int(r[si]), int(r[ii]), fname, int(r[0]), r[1].strip()[:90]))
        except ValueError:
            pass
ts = sum(x[0] for x in lines) or 1
ti = sum(x[1] for x in lines) or 1
print(f"total samples {ts}, warp instructions {ti}")
print(f"{'samp%':>6} {'inst%':>6}  file:line  source")
for s, i, f, ln, src in sorted(lines, reverse=True)[:top]:
    print(f"{100*s/ts:6.1f} {100*i/ti:6.1f}  {f}:{ln}  {src}")
