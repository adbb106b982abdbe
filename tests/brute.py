"""Brute-force transcription of the detection rules (O2-O12) for TINY streams.

Test infrastructure, independent of oracle/gs_oracle.cpp: it never parses SASS text. Streams are
built as Python structures (``Ins``) and rendered to text for the oracle; this module evaluates
the rules on the structures directly, with O(n^3) rescans (every last-writer is recomputed by a
backward scan; no reaching-definition table, no grouping maps).

Grammar of the tiny streams (SURVEY §4 plan item 3): opcodes {MOV, IADD3, IMAD.WIDE, LDC.64,
LDG.E, LDG.E.64, LDG.E.CONSTANT, STG.E, STL, LDL, ATOMS.ADD, REDG.E.ADD, I2F, FFMA, BRA} over
registers R0..R5 and immediate offsets {0, 4, 8}.
"""
from __future__ import annotations

import random
from dataclasses import dataclass, field

PARAM_BASE = 0x380  # sm_100 (the rendered text carries "code for sm_100a")

# reason ids (ncu order, DESIGN.md §3 table R)
LG_THROTTLE, LONG_SB, TEX_THROTTLE = 5, 6, 16


@dataclass
class Ins:
    op: str                      # full opcode text, e.g. "LDG.E.64"
    dst: int | None = None       # GPR number written (None = no register dst)
    width: int = 1               # registers written
    srcs: list = field(default_factory=list)   # operand list after dst: ("R",n) ("C",off) ("I",v)
    base: int | None = None      # memory base register
    off: int = 0                 # memory immediate offset
    data: int | None = None      # stored register (STG/STL/ATOMS/REDG)
    target: int | None = None    # BRA target index

    def text(self, pc: int) -> str:
        def o(s):
            if s[0] == "R":
                return "RZ" if s[1] == 255 else f"R{s[1]}"
            if s[0] == "C":
                return f"c[0x0][{hex(s[1])}]"
            return hex(s[1])

        def mem(desc: bool, wide: bool):
            b = f"R{self.base}" + (".64" if wide else "")
            if self.off > 0:
                b += f"+{hex(self.off)}"
            elif self.off < 0:
                b += f"+-{hex(-self.off)}"
            return ("desc[UR4]" if desc else "") + f"[{b}]"

        fam = self.op.split(".")[0]
        if fam == "BRA":
            body = f"BRA {hex(self.target * 16)}"
        elif fam == "LDG":
            body = f"{self.op} R{self.dst}, {mem(True, True)}"
        elif fam == "STG":
            body = f"{self.op} {mem(True, True)}, R{self.data}"
        elif fam == "REDG":
            body = f"{self.op} {mem(True, True)}, R{self.data}"
        elif fam == "STL":
            body = f"{self.op} {mem(False, False)}, R{self.data}"
        elif fam == "LDL":
            body = f"{self.op} R{self.dst}, {mem(False, False)}"
        elif fam == "ATOMS":
            body = f"{self.op} RZ, {mem(False, False)}, R{self.data}"
        else:
            body = f"{self.op} R{self.dst}, " + ", ".join(o(s) for s in self.srcs)
        return f"        /*{pc:04x}*/                   {body} ;"


def render(kernels: list[list[Ins]], names=None) -> str:
    out = ["\tcode for sm_100a"]
    for k, ins in enumerate(kernels):
        out.append(f"\t\tFunction : {names[k] if names else f'tiny{k}'}")
        out += [x.text(16 * i) for i, x in enumerate(ins)]
    return "\n".join(out) + "\n"


# ----------------------------------------------------------------------------- random streams
def random_stream(rng: random.Random, n: int) -> list[Ins]:
    ins: list[Ins] = []
    R = lambda: rng.randrange(6)                     # R0..R5
    E = lambda: rng.choice([0, 2, 4])                 # even register for 64-bit pairs
    OFF = lambda: rng.choice([0, 4, 8])
    for i in range(n):
        c = rng.randrange(15)
        if c == 0:
            s = rng.choice([("R", R()), ("C", PARAM_BASE + 8 * rng.randrange(3)), ("I", 16)])
            ins.append(Ins("MOV", dst=R(), srcs=[s]))
        elif c == 1:
            mid = rng.choice([("R", R()), ("C", PARAM_BASE + 8 * rng.randrange(3)), ("I", 4)])
            ins.append(Ins("IADD3", dst=R(), srcs=[("R", R()), mid, ("R", 255)]))
        elif c == 2:
            ins.append(Ins("IMAD.WIDE", dst=E(), width=2, srcs=[("R", R()), ("I", 4), ("R", E())]))
        elif c == 3:
            ins.append(Ins("LDC.64", dst=E(), width=2, srcs=[("C", PARAM_BASE + 8 * rng.randrange(3))]))
        elif c in (4, 5, 6):
            op = ["LDG.E", "LDG.E.64", "LDG.E.CONSTANT"][c - 4]
            d = E() if op == "LDG.E.64" else R()
            ins.append(Ins(op, dst=d, width=2 if op == "LDG.E.64" else 1, base=E(), off=OFF()))
        elif c == 7:
            ins.append(Ins("STG.E", base=E(), off=OFF(), data=R()))
        elif c == 8:
            ins.append(Ins("STL", base=R(), off=OFF(), data=R()))
        elif c == 9:
            ins.append(Ins("LDL", dst=R(), base=R(), off=OFF()))
        elif c == 10:
            ins.append(Ins("ATOMS.ADD", base=R(), off=OFF(), data=R()))
        elif c == 11:
            ins.append(Ins("REDG.E.ADD.STRONG.GPU", base=E(), off=OFF(), data=R()))
        elif c == 12:
            ins.append(Ins("I2F", dst=R(), srcs=[("R", R())]))
        elif c == 13:
            ins.append(Ins("FFMA", dst=R(), srcs=[("R", R()), ("R", R()), ("R", R())]))
        else:
            ins.append(Ins("BRA", target=rng.randrange(n)))
    return ins


# ----------------------------------------------------------------------------- the rules
def writes(x: Ins, r: int) -> bool:
    return x.dst is not None and x.dst <= r < x.dst + x.width


def last_writer(ins, i, r):
    """O3 by brute force: scan backwards from i-1."""
    for j in range(i - 1, -1, -1):
        if writes(ins[j], r):
            return j
    return None


def reg_sources(x: Ins):
    s = [v for (k, v) in x.srcs if k == "R" and v != 255]
    if x.base is not None:
        s.append(x.base)
    if x.data is not None:
        s.append(x.data)
    return s


def fam(x: Ins) -> str:
    return x.op.split(".")[0]


def trace(ins, i, r0, D):
    """O5 by brute force.  Returns (term string, chain list)."""
    chain, pos, r = [], i, r0
    for _ in range(D):
        j = last_writer(ins, pos, r)
        if j is None:
            return f"ENTRY:R{r}", chain
        chain.append(j)
        pos = j
        x = ins[j]
        f = fam(x)
        if f == "LDC":
            off = x.srcs[0][1] + 4 * (r - x.dst)
            return (f"PARAM:{hex(off)}" if off >= PARAM_BASE else f"CONST:0x0:{hex(off)}"), chain
        if f in ("LDG", "LDL"):
            return f"MEMORY:{j}", chain
        # pointer operand
        if f == "IMAD" and "WIDE" in x.op:
            pick = x.srcs[2]
        elif f == "IADD3":
            cands = [s for s in x.srcs if s[0] == "C"] + [s for s in x.srcs if s[0] == "R" and s[1] != 255]
            pick = cands[0] if cands else ("I", 0)
        else:
            cands = [s for s in x.srcs if s[0] == "C" or (s[0] == "R" and s[1] != 255)]
            pick = cands[0] if cands else ("I", 0)
        if pick[0] == "C":
            off = pick[1]
            return (f"PARAM:{hex(off)}" if off >= PARAM_BASE else f"CONST:0x0:{hex(off)}"), chain
        if pick[0] != "R" or pick[1] == 255:
            return "IMM", chain
        r = pick[1]
    return "TRUNC", chain


def loop_depth(ins, i):
    return sum(1 for b, x in enumerate(ins) if fam(x) == "BRA" and x.target < b and x.target <= i <= b)


ARITH = {"IADD3", "IMAD", "FFMA"}  # the ARITH members that occur in tiny streams (IMAD.WIDE is IMAD)


def detect(kernels: list[list[Ins]], D=64, TA=1, TL=2):
    """Returns the canonical K and S lines (same layout as the oracle)."""
    klines, slines = [], []
    first = 0
    for k, ins in enumerate(kernels):
        n = len(ins)
        gatom = sum(1 for x in ins if fam(x) == "REDG")
        satom = sum(1 for x in ins if fam(x) == "ATOMS")
        conv = sum(1 for x in ins if fam(x) == "I2F")
        vec_already = sum(1 for x in ins if x.op == "LDG.E.64")
        # store roots
        store_roots, ustores = [], 0
        for i, x in enumerate(ins):
            if fam(x) in ("STG", "REDG"):
                t, _ = trace(ins, i, x.base, D)
                if t.startswith("PARAM") or t.startswith("ENTRY"):
                    store_roots.append(t)
                else:
                    ustores += 1
        klines.append(f"K {k} {n} {first} gatom={gatom} satom={satom} conv={conv} "
                      f"vec_already={vec_already} ustores={ustores} name=tiny{k}")
        first += n

        def same_key(i, j):
            a, b = ins[i], ins[j]
            return a.base == b.base and last_writer(ins, i, a.base) == last_writer(ins, j, b.base)

        for i, x in enumerate(ins):
            ld = loop_depth(ins, i)
            sites = []
            if fam(x) in ("LDG", "STG", "STL", "LDL", "REDG"):
                term, chain = trace(ins, i, x.base, D)
            else:
                term, chain = "NONE", []
            if fam(x) == "LDG":
                is32 = x.op in ("LDG.E", "LDG.E.CONSTANT")
                g32 = sorted({ins[j].off for j in range(n)
                              if ins[j].op in ("LDG.E", "LDG.E.CONSTANT") and same_key(i, j)})
                gall = [j for j in range(n) if fam(ins[j]) == "LDG" and same_key(i, j)]
                offs_all = {ins[j].off for j in gall}
                if is32 and len(g32) >= 2:
                    contig = int(all(g32[q + 1] - g32[q] == 4 for q in range(len(g32) - 1)))
                    sites.append(("VEC", f" n={len(g32)} min={g32[0]} max={g32[-1]} contig={contig}"))
                n_arith = 0
                for j in range(n):
                    y = ins[j]
                    if fam(y) in ARITH and any(last_writer(ins, j, s) == i for s in reg_sources(y)):
                        n_arith += 1
                if n_arith >= TA and (len(gall) >= TL or ld >= 1):
                    sites.append(("SHMEM", f" loads={len(gall)} arith={n_arith}"))
                ro = ("CONSTANT" not in x.op and (term.startswith("PARAM") or term.startswith("ENTRY"))
                      and term not in store_roots)
                if ro:
                    sites.append(("RO", ""))
                    if len(offs_all) >= 2:
                        sites.append(("TEX", f" n={len(offs_all)}"))
            if fam(x) in ("STL", "LDL"):
                if fam(x) == "STL":
                    c = last_writer(ins, i, x.data)
                    sites.append(("SPILL", f" data=R{x.data} cause={'E' if c is None else c}"))
                else:
                    sites.append(("SPILL", f" data=R{x.dst} cause=-"))
            if fam(x) == "REDG":
                sites.append(("GATOM", ""))
            if fam(x) == "I2F":
                sites.append(("CONV", ""))
            order = ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"]
            for rule, attrs in sorted(sites, key=lambda s: order.index(s[0])):
                ch = ",".join(map(str, chain)) if chain else "-"
                slines.append(f"S {k} {i} {rule} line=- ld={ld} term={term} d={len(chain)} chain={ch}{attrs}")
    return klines, slines


# ----------------------------------------------------------------------------- consumer join (R37)
def gpr_uses(x: Ins) -> set:
    """GPRs the instruction reads, register pairs expanded (O16 / R36 for this grammar): the
    64-bit memory bases rendered ``[Rb.64]`` (LDG, STG, REDG) and the addend of IMAD.WIDE are
    pairs; every other operand is one register."""
    u = set()
    for q, (k, v) in enumerate(x.srcs):
        if k == "R" and v != 255:
            u.add(v)
            if fam(x) == "IMAD" and q == 2:
                u.add(v + 1)
    if x.base is not None:
        u.add(x.base)
        if fam(x) in ("LDG", "STG", "REDG"):
            u.add(x.base + 1)
    if x.data is not None:
        u.add(x.data)
    return u


def consumers(ins, i):
    """Instructions j > i reading a register whose last writer before j is i (brute force)."""
    return [j for j in range(i + 1, len(ins))
            if any(last_writer(ins, j, r) == i for r in gpr_uses(ins[j]))]
