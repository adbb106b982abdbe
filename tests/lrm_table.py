"""Test-side parser of nvdisasm's register life-range table (`nvdisasm -lrm narrow`): per function,
per instruction (text, live GPR count, defined GPRs, used GPRs, live GPRs). nvdisasm marks a
register column '^' (assigned), 'v' (used), 'x' (used and reassigned), ':' (live). This is the
external pin of the oracle's O16 register model (R36, R38). Test infrastructure only."""
from __future__ import annotations

import re


def parse(lines) -> list:
    funcs, cur, cols, hdr = [], None, None, []
    for t in lines:
        if re.match(r"\s*\.text\.(\S+):", t):
            cur = []
            funcs.append(cur)
            continue
        if "// |" not in t:
            continue
        tab = t[t.index("// |") + 3:].rstrip("\n")
        secs = tab.split("|")
        if len(secs) < 2:
            continue
        g = secs[1]  # the GPR section
        if "#" in g:  # the units row of the column header: map column -> register number
            rows = [h for h in hdr if re.fullmatch(r"[\s0-9]*", h) and re.search(r"\d", h)]
            start = g.index("#")
            cols = {}
            for ci, ch in enumerate(g):
                if ci > start and ch.isdigit():
                    digits = "".join((r[ci] if ci < len(r) and r[ci].isdigit() else "0") for r in rows) + ch
                    cols[ci] = int(digits)
            hdr = []
            continue
        if re.fullmatch(r"[\s0-9]*", g) and re.search(r"\d", g):  # hundreds / tens rows
            hdr.append(g)
            continue
        m = re.search(r"/\*([0-9a-f]{4,})\*/\s*(.*?);", t)
        if not m or cur is None or cols is None:
            continue
        cnt = re.match(r"\s*(\d*)", g).group(1)
        d, u, live = set(), set(), set()
        for ci, r in cols.items():
            ch = g[ci] if ci < len(g) else " "
            if ch in "^x":
                d.add(r)
            if ch in "vx":
                u.add(r)
            if ch != " ":
                live.add(r)
        cur.append((m.group(2).strip(), int(cnt or 0), d, u, live))
    return funcs
