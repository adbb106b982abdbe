"""Test-side helpers to build/run the CPU oracle (oracle/gs_oracle.cpp) and parse its canonical
output. Test infrastructure only."""
from __future__ import annotations

import os
import subprocess
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")
ORACLE = os.path.join(ROOT, "oracle", "gs_oracle")
ORACLE_SRC = os.path.join(ROOT, "oracle", "gs_oracle.cpp")


def build_oracle(force: bool = False) -> str:
    if force or not os.path.exists(ORACLE) or os.path.getmtime(ORACLE) < os.path.getmtime(ORACLE_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-o", ORACLE, ORACLE_SRC])
    return ORACLE


def run(sass, samples: np.ndarray | None = None, D=64, R=19, TA=1, TL=2, k=-1, kbegin=0, kend=-1,
        detect=True, hist=True, timing=False, counts: np.ndarray | None = None, join: str = "pc",
        liveness: bool = False, hlines: bool = True, regsets: bool = False) -> str:
    """sass: path or text/bytes. samples: [N,3] uint32 raw triples. counts: [M,4] uint32
    pre-aggregated (kernel, pc, reason, count) records. join: pc | line | consumer. Returns canonical text."""
    build_oracle()
    tmp = []
    try:
        if isinstance(sass, (bytes, bytearray)) or (isinstance(sass, str) and "\n" in sass):
            f = tempfile.NamedTemporaryFile("wb", suffix=".sass", delete=False)
            f.write(sass if isinstance(sass, (bytes, bytearray)) else sass.encode())
            f.close()
            tmp.append(f.name)
            sass_path = f.name
        else:
            sass_path = sass
        cmd = [ORACLE, "--sass", sass_path, "--D", str(D), "--R", str(R), "--ta", str(TA), "--tl", str(TL),
               "--k", str(k), "--kbegin", str(kbegin), "--kend", str(kend)]
        if samples is not None:
            f = tempfile.NamedTemporaryFile("wb", suffix=".bin", delete=False)
            np.ascontiguousarray(samples, dtype=np.uint32).tofile(f)
            f.close()
            tmp.append(f.name)
            cmd += ["--samples", f.name]
        if counts is not None:
            f = tempfile.NamedTemporaryFile("wb", suffix=".bin", delete=False)
            np.ascontiguousarray(counts, dtype=np.uint32).tofile(f)
            f.close()
            tmp.append(f.name)
            cmd += ["--counts", f.name]
        if join != "pc":
            cmd += ["--join", join]
        if liveness:
            cmd.append("--liveness")
        if regsets:
            cmd.append("--regsets")
        if not hlines:
            cmd.append("--no-hlines")
        if not detect:
            cmd.append("--no-detect")
        if not hist:
            cmd.append("--no-hist")
        if timing:
            cmd.append("--time")
        p = subprocess.run(cmd, capture_output=True, text=True)
        if p.returncode != 0:
            raise RuntimeError(f"oracle failed rc={p.returncode}: {p.stderr}")
        return (p.stdout, p.stderr) if timing else p.stdout
    finally:
        for t in tmp:
            os.unlink(t)


class Canon:
    """Parsed canonical result."""

    def __init__(self, text: str):
        self.text = text
        self.K, self.S, self.R, self.H = [], [], [], {}
        self.N = None
        for line in text.splitlines():
            if line.startswith("K "):
                self.K.append(line)
            elif line.startswith("S "):
                self.S.append(line)
            elif line.startswith("R "):
                self.R.append(line)
            elif line.startswith("H "):
                _, s, r, c = line.split()
                self.H[(int(s), int(r))] = int(c)
            elif line.startswith("N "):
                self.N = dict(kv.split("=") for kv in line.split()[1:])

    def sites(self, rule=None, k=None):
        out = []
        for line in self.S:
            f = line.split()
            d = {"k": int(f[1]), "idx": int(f[2]), "rule": f[3]}
            for kv in f[4:]:
                a, b = kv.split("=", 1)
                d[a] = b
            if (rule is None or d["rule"] == rule) and (k is None or d["k"] == k):
                out.append(d)
        return out

    def kstats(self):
        out = []
        for line in self.K:
            f = line.split()
            d = {"k": int(f[1]), "n": int(f[2]), "first": int(f[3])}
            for kv in f[4:]:
                a, b = kv.split("=", 1)
                d[a] = b if a == "name" else int(b)
            out.append(d)
        return out


def golden(name: str) -> str:
    return os.path.join(GOLDEN, name)


def golden_text(name: str) -> str:
    """A fixture's text; `.xz` fixtures (the frozen torch SASS) are decompressed."""
    import lzma
    path = golden(name)
    if path.endswith(".xz"):
        with lzma.open(path, "rt") as f:
            return f.read()
    with open(path) as f:
        return f.read()


def regsets(text: str, **kw) -> dict:
    """(kernel, idx) -> (defs, uses, live) of the oracle's O16 register model (G lines)."""
    def ints(v):
        return set() if v == "-" else set(map(int, v.split(",")))
    out = {}
    for line in run(text, regsets=True, hist=False, **kw).splitlines():
        if line.startswith("G "):
            f = line.split()
            out[(int(f[1]), int(f[2]))] = (ints(f[3][4:]), ints(f[4][4:]), ints(f[5][5:]))
    return out


def sass_ops(path: str) -> dict:
    """idx -> full opcode token of a cuobjdump listing (test-side text lookup)."""
    import re
    ops = {}
    for line in open(path):
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(@\S+\s+)?(\S+)", line)
        if m:
            ops[int(m.group(1), 16) // 16] = m.group(3)
    return ops
