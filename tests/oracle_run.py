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
        liveness: bool = False, hlines: bool = True, regsets: bool = False, cupti: str | None = None,
        cupti_crc: int = 0) -> str:
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
        if cupti is not None:   # CUPTI PC-sampling records in their text form (gen/cupti.py)
            f = tempfile.NamedTemporaryFile("w", suffix=".cupti", delete=False)
            f.write(cupti)
            f.close()
            tmp.append(f.name)
            cmd += ["--cupti", f.name, "--cupti-crc", str(cupti_crc)]
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


# ------------------------------------------------------------------------------ sharded oracle
def split_kernels(text: bytes) -> list[bytes]:
    """cuobjdump text -> one text per kernel ("Function :" sections). The preamble (-res-usage
    block, first arch line) goes with every section, and each later section also gets the last
    "code for sm_NN" line before it. Test-side text slicing only: each section is parsed by the
    oracle itself."""
    def line_starts(needle):
        out, p = [], text.find(needle)
        while p >= 0:
            out.append(text.rfind(b"\n", 0, p) + 1)
            p = text.find(needle, p + len(needle))
        return out
    marks = line_starts(b"Function : ")
    if not marks:
        return [text]
    arches = line_starts(b"code for sm_")
    cuts = marks + [len(text)]
    pre = text[:marks[0]]
    out = [text[:cuts[1]]]
    a = 0
    for i in range(1, len(marks)):
        while a + 1 < len(arches) and arches[a + 1] < marks[i]:
            a += 1
        arch = b""
        if arches and arches[a] < marks[i]:
            e = text.find(b"\n", arches[a])
            arch = text[arches[a]:e + 1]
        out.append(pre + arch + text[cuts[i]:cuts[i + 1]])
    return out


def run_sharded(sass: bytes, raw: np.ndarray | None, n_instr, shards: int, D=64, R=19, timing=False,
                tmpdir: str | None = None):
    """The all-cores oracle baseline (SURVEY §8d "the same oracle functions over kernel / sample
    shards, merged by integer sums"): the module is cut into `shards` contiguous kernel ranges
    balanced by instruction count, each with the samples of its kernels, and each range is a
    complete, independent oracle run (histogram bins, kernel totals and sites are per kernel).
    Runs the processes in parallel and merges their canonical outputs: kernel and slot numbers
    shifted, N lines summed, R lines re-sorted by the total order (R20). The merged text equals the
    single-process output (tests/test_oracle_pins.py). Returns (text, seconds of the parallel part
    incl. the merge) when timing."""
    import time
    n_instr = np.asarray(n_instr, dtype=np.int64)
    K = len(n_instr)
    shards = max(1, min(shards, K))
    csum = np.concatenate([[0], np.cumsum(n_instr)])
    bounds = [0] + [int(np.searchsorted(csum, csum[-1] * p / shards)) for p in range(1, shards)] + [K]
    bounds = sorted(set(min(max(b, 0), K) for b in bounds))
    secs = split_kernels(sass) if not (tmpdir and os.path.exists(os.path.join(tmpdir, "shard0.sass"))) else [b""] * K
    assert len(secs) == K, (len(secs), K)
    build_oracle()
    td = tmpdir or tempfile.mkdtemp()
    jobs = []
    for p in range(len(bounds) - 1):
        kb, ke = bounds[p], bounds[p + 1]
        if kb == ke:
            continue
        sp = os.path.join(td, f"shard{p}.sass")
        reuse = tmpdir is not None and os.path.exists(sp)  # a caller's tmpdir keeps the inputs of repeated steps
        if not reuse:
            with open(sp, "wb") as f:
                f.write(b"".join(secs[kb:ke]))
        cmd = [ORACLE, "--sass", sp, "--D", str(D), "--R", str(R), "--no-hlines"]
        if raw is not None and reuse:
            cmd += ["--samples", os.path.join(td, f"shard{p}.bin")]
        elif raw is not None:
            kk = raw[:, 0].astype(np.int64)
            sel = (kk >= kb) & (kk < ke) if p else ((kk < ke) | (kk >= K))  # invalid kernels: shard 0
            part = raw[sel].copy()
            ok = part[:, 0] < K
            part[ok, 0] -= kb
            rp = os.path.join(td, f"shard{p}.bin")
            np.ascontiguousarray(part, dtype=np.uint32).tofile(rp)
            cmd += ["--samples", rp]
        jobs.append((kb, int(csum[kb]), cmd))
    t0 = time.perf_counter()
    procs = [subprocess.Popen(c, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True) for _, _, c in jobs]
    outs = [p.communicate() for p in procs]
    for p, (o, e) in zip(procs, outs):
        if p.returncode != 0:
            raise RuntimeError(f"oracle shard failed: {e}")
    head, klines, slines, rrows = None, [], [], []
    tot = {"total": 0, "valid": 0, "invalid": 0}
    have_n = False
    for (kb, sb, _), (o, _) in zip(jobs, outs):
        for line in o.splitlines():
            f = line.split()
            if line.startswith("#") or line.startswith("CFG"):
                head = head or []
                if line not in head:
                    head.append(line)
            elif f[0] == "K":
                f[1] = str(int(f[1]) + kb)
                f[3] = str(int(f[3]) + sb)
                klines.append(" ".join(f))
            elif f[0] == "S":
                f[1] = str(int(f[1]) + kb)
                slines.append(" ".join(f))
            elif f[0] == "N":
                have_n = True
                for kv in f[1:]:
                    a, b = kv.split("=")
                    tot[a] += int(b)
            elif f[0] == "R":
                k = int(f[2]) + kb
                rel = int(f[5].split("=")[1])
                totv = int(f[6].split("=")[1])
                rrows.append((-rel, -totv, k, int(f[3]), ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX",
                                                           "CONV"].index(f[4]), f[4:]))
    rrows.sort(key=lambda r: r[:5])
    lines = head + klines + slines
    if have_n:
        lines.append(f"N total={tot['total']} valid={tot['valid']} invalid={tot['invalid']}")
    lines += [f"R {q} {r[2]} {r[3]} " + " ".join(r[5]) for q, r in enumerate(rrows)]
    secs_par = time.perf_counter() - t0
    if tmpdir is None:
        import shutil
        shutil.rmtree(td, ignore_errors=True)
    text = "\n".join(lines) + "\n"
    return (text, secs_par) if timing else text
