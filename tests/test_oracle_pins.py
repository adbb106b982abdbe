"""Pins of the CPU oracle against facts fixed outside it.

Every expected value here comes from the paper's text (cited), from the C ABI of a kernel whose
source is in tests/golden/src (parameter offsets), from ptxas' own spill accounting, from a
closed-form count table, or from the independent brute force in tests/brute.py — never from the
oracle itself and never from the CUDA path.
"""
import random

import numpy as np
import pytest

import brute
import oracle_run as orc
from oracle_run import Canon, golden

pytestmark = pytest.mark.usefixtures("oracle_bin")


# --------------------------------------------------------------------------- Listing 1
def test_listing1_texture_and_vector_groups():
    c = Canon(orc.run(golden("listing1.sass")))
    vec = {s["idx"] for s in c.sites("VEC")}
    # "Loads to R0 and R9 fetch data from adjacent memory addresses R2 and R2+-0x8 ...
    #  The same holds for loads to R5 and R7."
    assert vec == {0, 1, 2, 3}
    groups = {s["idx"]: (s["term"], s["min"], s["max"], s["n"]) for s in c.sites("VEC")}
    assert groups[0] == groups[3] == ("ENTRY:R2", "-8", "0", "2")
    assert groups[1] == groups[2] == ("ENTRY:R4", "-8", "0", "2")
    # "If these registers are read-only, they are potential candidates for texture memory":
    # STG [R4], R9 writes through R4, so only the R2-based loads (R0, R9) are read-only.
    assert {s["idx"] for s in c.sites("RO")} == {0, 3}
    assert {s["idx"] for s in c.sites("TEX")} == {0, 3}
    assert c.sites("SHMEM") == []  # no arithmetic on the loaded values


# --------------------------------------------------------------------------- SGEMM
# sgemm_naive(int M, int N, int K, float alpha, const float* A, const float* B, float beta, float* C)
# C ABI parameter offsets from the param base: A +0x10, B +0x18, C +0x28.
@pytest.mark.parametrize("arch,base", [("sm_100a", 0x380), ("sm_70", 0x160)])
def test_sgemm_readonly_A_B_not_C(arch, base):
    c = Canon(orc.run(golden(f"sgemm_naive.{arch}.sass")))
    A, B, C = hex(base + 0x10), hex(base + 0x18), hex(base + 0x28)
    ops = orc.sass_ops(golden(f"sgemm_naive.{arch}.sass"))
    ldg = {i for i, op in ops.items() if op.startswith("LDG")}
    ro_terms = {s["term"] for s in c.sites("RO")}
    # "registers that are read-only throughout the lifetime of the kernel, and are not aliased"
    # (P:943-946): A and B, never C (C is loaded and stored).
    assert ro_terms == {f"PARAM:{A}", f"PARAM:{B}"}
    ro = {s["idx"] for s in c.sites("RO")}
    assert len(ldg - ro) == 1                           # exactly the C load is not read-only
    # shared-memory advice on the loop loads
    shm = c.sites("SHMEM")
    assert {s["term"] for s in shm} == {f"PARAM:{A}", f"PARAM:{B}"}
    assert any(s["ld"] == "1" for s in shm)


def test_sgemm_sm100_eight_adjacent_A_loads():
    """The unroll-by-8 A loads off R4 at -0x10..+0xc (SURVEY [probe 4]); the "reads seven
    adjacent addresses" shape of P:789-792, inside the loop closed by `@P1 BRA 0x220` at 0x4b0."""
    c = Canon(orc.run(golden("sgemm_naive.sm_100a.sass")))
    want = {0x260 // 16, 0x270 // 16, 0x280 // 16, 0x2a0 // 16, 0x350 // 16, 0x370 // 16, 0x3a0 // 16,
            0x3c0 // 16}
    big = [s for s in c.sites("VEC") if s["n"] == "8"]
    assert {s["idx"] for s in big} == want
    for s in big:
        assert (s["min"], s["max"], s["contig"], s["term"], s["ld"]) == ("-16", "12", "1", "PARAM:0x390", "1")
        assert s["chain"].split(",")[-1] == str(0x190 // 16)     # LDCU.64 UR4, c[0x0][0x390]
    # loop span [0x220, 0x4b0] only: the load at 0x870 (C) has loop depth 0
    assert all(s["ld"] == "1" for s in c.sites() if 0x22 <= s["idx"] <= 0x4b)
    assert all(s["ld"] == "0" for s in c.sites() if s["idx"] > 0x4b)


# --------------------------------------------------------------------------- Jacobi
# jacobi(const float* Told, float* Tnew, ...): Told at +0x0, Tnew at +0x8; six (float) casts.
@pytest.mark.parametrize("arch,base", [("sm_100a", 0x380), ("sm_70", 0x160)])
def test_jacobi_flags_and_six_conversions(arch, base):
    c = Canon(orc.run(golden(f"jacobi.{arch}.sass")))
    k = c.kstats()[0]
    assert k["conv"] == 6 and len(c.sites("CONV")) == 6          # "six I2F"
    told = f"PARAM:{hex(base)}"
    # recommended: texture/shared, vectorised loads, __restrict__, conversions
    for rule in ("TEX", "SHMEM", "VEC", "RO"):
        assert c.sites(rule), rule
        assert {s["term"] for s in c.sites(rule)} == {told}, rule


# --------------------------------------------------------------------------- Mixbench
def test_mixbench_sp_vectorise_dp_already_vectorised():
    for arch in ("sm_100a", "sm_70"):
        c = Canon(orc.run(golden(f"mixbench.{arch}.sass")))
        ks = {d["name"]: d for d in c.kstats()}
        dp = [d for n, d in ks.items() if "dp" in n][0]
        sp = [d for n, d in ks.items() if "sp" in n][0]
        # SP: one 32-bit load "also reads seven adjacent addresses"
        vec = c.sites("VEC", k=sp["k"])
        assert len(vec) == 8 and {(s["n"], s["contig"]) for s in vec} == {("8", "1")}
        assert {int(s["max"]) - int(s["min"]) for s in vec} == {28}
        # DP: "a 64-bit width vectorized read performed by the compiler"
        assert c.sites("VEC", k=dp["k"]) == [] and dp["vec_already"] == 8
        # shared-memory advice on the same loads
        assert len(c.sites("SHMEM", k=sp["k"])) == 8 and len(c.sites("SHMEM", k=dp["k"])) == 8


# --------------------------------------------------------------------------- spills
@pytest.mark.parametrize("cap", [24, 32, 40, 64])
def test_spill_sites_match_ptxas_bytes(cap):
    """ptxas -v "N bytes spill stores, M bytes spill loads" == sum of STL / LDL access widths."""
    path = golden(f"spill.r{cap}.sm_100a.sass")
    c = Canon(orc.run(path))
    ops = orc.sass_ops(path)
    st = ld = 0
    for s in c.sites("SPILL"):
        op = ops[s["idx"]]
        w = 16 if ".128" in op else 8 if ".64" in op else 4
        if op.startswith("STL"):
            st += w
        else:
            assert op.startswith("LDL")
            ld += w
    txt = open(golden(f"spill.r{cap}.ptxas.txt")).read()
    want = txt.split("stack frame,")[1].split("\n")[0]
    assert f"{st} bytes spill stores, {ld} bytes spill loads" in want
    assert len(c.sites("SPILL")) == sum(1 for op in ops.values() if op.startswith(("STL", "LDL")))


def test_fig2_spill_cause_is_last_writer():
    """Fig.2 narrative: the cause of a spill of register X is the last instruction
    that wrote X (an IADD); the lg_throttle stall is the largest at that instruction."""
    text = "\tcode for sm_100a\n\t\tFunction : fig2\n" + "\n".join(
        f"        /*{16 * i:04x}*/                   {b} ;" for i, b in enumerate([
            "LDC R1, c[0x0][0x37c]",
            "IADD3 R5, PT, PT, R2, R3, RZ",
            "FMUL R6, R7, R8",
            "STL [R1+0x4], R5",
            "IADD3 R5, PT, PT, R5, 0x1, RZ",
            "EXIT",
        ])) + "\n"
    # samples at the STL (pc 0x30): lg_throttle 7, long_scoreboard 2, wait 1
    raw = np.array([[0, 0x30, 5]] * 7 + [[0, 0x30, 6]] * 2 + [[0, 0x30, 17]], dtype=np.uint32)
    c = Canon(orc.run(text, samples=raw))
    sp = c.sites("SPILL")
    assert len(sp) == 1 and sp[0]["idx"] == 3 and sp[0]["cause"] == "1" and sp[0]["data"] == "R5"
    assert sp[0]["term"] == "CONST:0x0:0x37c"               # the stack pointer, not a parameter
    r = c.R[0].split()
    h = [int(x) for x in r[-1].split("=")[1].split(",")]
    assert int(np.argmax(h)) == 5                            # lg_throttle largest offender
    assert r[5:8] == ["rel=9", "tot=10", "ktot=10"]          # SPILL REL = {long_sb, lg_throttle}


# --------------------------------------------------------------------------- atomics, conversions
def test_atomics_probe():
    c = Canon(orc.run(golden("atomics.sm_100a.sass")))
    g = c.sites("GATOM")
    ops = orc.sass_ops(golden("atomics.sm_100a.sass"))
    # source: one global atomicAdd in the loop, one after it (compiled to REDG), one shared atomic
    assert [ops[s["idx"]].split(".")[0] for s in g] == ["REDG", "REDG"]
    assert [s["ld"] for s in g] == ["1", "0"]
    assert c.kstats()[0]["satom"] == 1 and c.kstats()[0]["gatom"] == 2
    # gcount is param 1 (+0x8), gtotal param 2 (+0x10)
    assert [s["term"] for s in g] == ["PARAM:0x388", "PARAM:0x390"]


def test_conversion_probe():
    c = Canon(orc.run(golden("conv.sm_100a.sass")))
    assert c.kstats()[0]["conv"] == 2                       # one int->float, one double->float
    ops = orc.sass_ops(golden("conv.sm_100a.sass"))
    assert sorted(ops[s["idx"]] for s in c.sites("CONV")) == ["F2F.F32.F64", "I2FP.F32.S32"]


# --------------------------------------------------------------------------- trace depth bound
def chain_text(L):
    body = ["LDC.64 R2, c[0x0][0x388]"]
    r = 2
    for i in range(L):
        nr = 4 if r == 2 else 2
        body.append(["IADD3 R%d, P0, PT, R%d, 0x10, RZ", "MOV R%d, R%d", "IMAD.WIDE R%d, R9, 0x4, R%d"][i % 3]
                    % (nr, r))
        r = nr
    body.append(f"LDG.E R7, desc[UR6][R{r}.64]")
    return "\tcode for sm_100a\n\t\tFunction : chain\n" + "\n".join(
        f"        /*{16 * i:04x}*/                   {b} ;" for i, b in enumerate(body)) + "\n"


@pytest.mark.parametrize("L,D,resolved", [(62, 64, True), (63, 64, True), (64, 64, False), (3, 4, True),
                                          (4, 4, False)])
def test_trace_depth_semantics(L, D, resolved):
    """A chain needing exactly D last-writer steps resolves; D+1 steps is TRUNCATED (DESIGN §3 O5)."""
    c = Canon(orc.run(chain_text(L), D=D))
    ro = c.sites("RO")
    if resolved:
        assert len(ro) == 1 and ro[0]["term"] == "PARAM:0x388" and ro[0]["d"] == str(L + 1)
    else:
        assert ro == []          # TRUNCATED roots are never read-only (DESIGN §3 O10)
    steps = L + 1
    assert (steps <= D) == resolved


def test_trace_truncated_chain_recorded():
    # an LDG pair on the 65-step chain: both are VEC sites carrying the truncated trace
    body = chain_text(64).splitlines()
    last = body[-1]
    reg = last.split("[R")[1].split(".")[0]
    body.append(f"        /*{int(last.split('/*')[1].split('*/')[0], 16) + 16:04x}*/                   "
                f"LDG.E R8, desc[UR6][R{reg}.64+0x4] ;")
    c = Canon(orc.run("\n".join(body) + "\n", D=64))
    v = c.sites("VEC")
    assert len(v) == 2 and all(s["term"] == "TRUNC" and s["d"] == "64" for s in v)


# --------------------------------------------------------------------------- brute force
def test_brute_force_random_streams():
    rng = random.Random(20231112)
    for _ in range(300):
        ks = [brute.random_stream(rng, rng.randint(1, 6)) for _ in range(rng.randint(1, 3))]
        D = rng.choice([1, 2, 3, 64])
        c = Canon(orc.run(brute.render(ks), D=D))
        kl, sl = brute.detect(ks, D=D)
        assert c.K == kl and c.S == sl, brute.render(ks)


# --------------------------------------------------------------------------- histogram, join, rank
def _sgemm_samples(order="trace", seed=3, n=50_000, n_bad=64):
    from gen import samples as gs
    path = golden("sgemm_naive.sm_100a.sass")
    n_instr = [len(orc.sass_ops(path))]
    cls = np.full(n_instr[0], gs.CLS_ALU, dtype=np.uint8)
    cls[::7] = gs.CLS_MEM
    tab = gs.table_class_weighted(cls, n, key=seed)
    tr = gs.Trace(tab, [0], n_instr, order=order, seed=seed)
    raw = tr.raw()
    bad = gs.invalid_raw(1, n_instr, n_bad, key=seed)
    return path, tab, gs.interleave(raw, bad, key=seed + 1), n_bad


def test_histogram_equals_count_table():
    path, tab, raw, n_bad = _sgemm_samples()
    c = Canon(orc.run(path, samples=raw))
    want = {(s, r): int(tab[s, r]) for s, r in zip(*np.nonzero(tab))}
    assert c.H == want
    assert c.N == {"total": str(len(raw)), "valid": str(int(tab.sum())), "invalid": str(n_bad)}


def test_histogram_permutation_and_shard_invariance():
    path, tab, raw, _ = _sgemm_samples(order="shuffled", seed=5)
    full = Canon(orc.run(path, samples=raw))
    rev = Canon(orc.run(path, samples=raw[::-1].copy()))
    assert rev.H == full.H and rev.R == full.R
    for shards in (2, 4, 8):
        acc = {}
        for part in np.array_split(raw, shards):
            for key, v in Canon(orc.run(path, samples=part, detect=False)).H.items():
                acc[key] = acc.get(key, 0) + v
        assert acc == full.H


def test_join_and_rank_closed_form():
    """rel/tot/ktot recomputed from the count table and the site list, ranked with Python's sort."""
    path, tab, raw, _ = _sgemm_samples(seed=9)
    c = Canon(orc.run(path, samples=raw))
    rel_sets = {"VEC": [6], "SPILL": [5, 6], "SHMEM": [6], "GATOM": [5], "RO": [6], "TEX": [6, 16],
                "CONV": list(range(32))}
    order = ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"]
    rows = []
    for s in c.sites():
        h = tab[s["idx"]]
        rows.append((-int(h[rel_sets[s["rule"]]].sum()), -int(h.sum()), s["k"], s["idx"], order.index(s["rule"])))
    rows.sort()
    got = [r.split() for r in c.R]
    assert len(got) == len(rows)
    ktot = int(tab.sum())
    for q, (g, w) in enumerate(zip(got, rows)):
        assert g[:5] == ["R", str(q), str(w[2]), str(w[3]), order[w[4]]]
        assert g[5:8] == [f"rel={-w[0]}", f"tot={-w[1]}", f"ktot={ktot}"]


def test_configs_generate_and_run():
    from gen import sass as gsass
    for cfg in ("C1", "C2"):
        s = gsass.config_sass(cfg)
        c = Canon(orc.run(s.text))
        assert len(c.K) == {"C1": 1, "C2": 3}[cfg]
        assert sum(k["n"] for k in c.kstats()) == s.P
        assert c.sites("SPILL") if cfg == "C1" else c.sites("VEC")


# --------------------------------------------------------------------------- nvdisasm text (O1)
LINEINFO = ["sgemm_naive", "jacobi", "mixbench", "atomics", "spill"]


def _strip_lines(lines):
    import re
    return [re.sub(r" line=\S+", "", x) for x in lines]


@pytest.mark.parametrize("name", LINEINFO)
def test_nvdisasm_and_cuobjdump_of_one_cubin_agree(name):
    """One cubin, two disassemblers: nvdisasm -g (".text.f:" function labels, `(.L_x_N) branch
    labels, //## line info) and cuobjdump -sass (hex branch targets) must give identical kernels
    and sites (only the line= attribute differs). Pins the label resolution (loop marks, R28)."""
    a = Canon(orc.run(golden(f"lineinfo/{name}.cuobjdump.sass")))
    b = Canon(orc.run(golden(f"lineinfo/{name}.nvdisasm.sass")))
    assert a.K == b.K and len(a.K) >= 1
    assert _strip_lines(a.S) == _strip_lines(b.S)
    assert all("line=-" in x for x in a.S)
    assert all("line=-" not in x for x in b.S)
    if name in ("sgemm_naive", "atomics", "spill"):
        assert any(s["ld"] != "0" for s in b.sites())   # loops found through labels


def test_nvdisasm_lines_are_the_source_lines():
    """jacobi.cu: the five Told[...] loads sit on the source lines that read Told, the six
    conversions on the lines with (float) casts (tests/golden/src/jacobi.cu)."""
    src = open(golden("src/jacobi.cu")).read().splitlines()
    told = {i + 1 for i, t in enumerate(src) if "Told[" in t}
    casts = {i + 1 for i, t in enumerate(src) if "(float)" in t}
    c = Canon(orc.run(golden("lineinfo/jacobi.nvdisasm.sass")))
    assert {int(s["line"]) for s in c.sites("RO")} == told and len(told) == 5
    conv = c.sites("CONV")
    assert len(conv) == 6 and {int(s["line"]) for s in conv} <= casts


def _nvdisasm_line_table(path):
    """independent test-side parse: instruction index -> (file, line) of an nvdisasm -g listing"""
    import re
    out, cur = [], None
    for t in open(path):
        m = re.match(r'\s*//## File "([^"]*)", line (\d+)', t)
        if m:
            cur = (m.group(1), int(m.group(2)))
            continue
        if re.match(r"\s*/\*[0-9a-f]{4,}\*/\s", t):
            out.append(cur)
    return out


def test_line_join_closed_form():
    """join=line (R33): a site's row is the sum of the count-table rows of every
    instruction on its source line; tot, rel and h follow from the table and an independent parse
    of the //## line markers."""
    from gen import samples as gs
    path = golden("lineinfo/jacobi.nvdisasm.sass")
    lines = _nvdisasm_line_table(path)
    n = len(lines)
    rng = np.random.default_rng(31)
    tab = np.zeros((n, 32), np.int64)
    tab[:, :19] = rng.integers(0, 50, (n, 19))
    raw = gs.Trace(tab, [0], [n], order="shuffled", seed=31).raw()
    pc = Canon(orc.run(path, samples=raw))
    ln = Canon(orc.run(path, samples=raw, join="line"))
    assert ln.H == pc.H and ln.S == pc.S
    rel_sets = {"VEC": [6], "SPILL": [5, 6], "SHMEM": [6], "GATOM": [5], "RO": [6], "TEX": [6, 16],
                "CONV": list(range(32))}
    got = {}
    for r in ln.R:
        f = r.split()
        kv = dict(x.split("=") for x in f[5:])
        got[(int(f[3]), f[4])] = kv
    assert len(got) == len(pc.R)
    for s in ln.sites():
        row = tab[[i for i in range(n) if lines[i] == lines[s["idx"]]]].sum(axis=0)
        kv = got[(s["idx"], s["rule"])]
        assert int(kv["tot"]) == int(row.sum())
        assert int(kv["rel"]) == int(row[rel_sets[s["rule"]]].sum())
        assert kv["h"] == ",".join(str(int(x)) for x in row[:19])
    # a line holding several instructions really aggregates
    assert any(int(got[(s["idx"], s["rule"])]["tot"]) > int(tab[s["idx"]].sum()) for s in ln.sites())
    # without line information join=line is join=pc
    plain = golden("lineinfo/jacobi.cuobjdump.sass")
    assert Canon(orc.run(plain, samples=raw, join="line")).R == Canon(orc.run(plain, samples=raw)).R


def _ranked_rows(c):
    got = {}
    for r in c.R:
        f = r.split()
        kv = dict(x.split("=") for x in f[5:])
        got[(int(f[2]), int(f[3]), f[4])] = kv
    return got


REL_SETS = {"VEC": [6], "SPILL": [5, 6], "SHMEM": [6], "GATOM": [5], "RO": [6], "TEX": [6, 16],
            "CONV": list(range(32))}


def test_consumer_join_brute_force():
    """join=consumer (R37): a site's row is its PC row plus the rows of the
    instructions that read a register it wrote (last writer = the site). Checked against an O(n^3)
    brute force on random tiny streams (tests/brute.py: backward rescans, its own register-use
    rules) with random count tables."""
    from gen import samples as gs
    rng = random.Random(37)
    nrng = np.random.default_rng(37)
    checked = 0
    for _ in range(150):
        ks = [brute.random_stream(rng, rng.randint(2, 7)) for _ in range(rng.randint(1, 2))]
        n_instr = [len(k) for k in ks]
        first = list(np.cumsum([0] + n_instr[:-1]))
        tab = np.zeros((sum(n_instr), 32), np.int64)
        tab[:, :19] = nrng.integers(0, 9, (sum(n_instr), 19))
        if tab.sum() == 0:
            continue
        raw = gs.Trace(tab, first, n_instr, order="shuffled", seed=rng.randrange(1000)).raw()
        text = brute.render(ks)
        pc = Canon(orc.run(text, samples=raw))
        cs = Canon(orc.run(text, samples=raw, join="consumer"))
        assert cs.H == pc.H and cs.S == pc.S and cs.K == pc.K
        got = _ranked_rows(cs)
        assert len(got) == len(pc.R)
        for s in cs.sites():
            k, i = s["k"], s["idx"]
            rows = [first[k] + i] + [first[k] + j for j in brute.consumers(ks[k], i)]
            row = tab[rows].sum(axis=0)
            kv = got[(k, i, s["rule"])]
            assert int(kv["tot"]) == int(row.sum()), text
            assert int(kv["rel"]) == int(row[REL_SETS[s["rule"]]].sum()), text
            assert kv["h"] == ",".join(str(int(x)) for x in row[:19]), text
            checked += 1
    assert checked > 100


def test_consumer_join_hand_example():
    """A hand-checked stream: the load's two readers are its consumers; the reader after the
    register is overwritten is not; a store has no consumers (its row alone)."""
    from gen import samples as gs
    ins = [
        brute.Ins("LDC.64", dst=2, width=2, srcs=[("C", 0x380)]),
        brute.Ins("LDG.E", dst=4, base=2, off=0),                        # 1: RO site
        brute.Ins("FFMA", dst=5, srcs=[("R", 4), ("R", 4), ("R", 0)]),   # 2: consumer of 1 (once)
        brute.Ins("I2F", dst=6, srcs=[("R", 4)]),                        # 3: consumer of 1; CONV site
        brute.Ins("MOV", dst=4, srcs=[("I", 16)]),                       # 4: overwrites R4
        brute.Ins("FFMA", dst=1, srcs=[("R", 4), ("R", 6), ("R", 5)]),   # 5: consumer of 4, 3, 2
        brute.Ins("LDC.64", dst=8, width=2, srcs=[("C", 0x388)]),
        brute.Ins("REDG.E.ADD.STRONG.GPU", base=8, off=0, data=1),       # 7: GATOM site, no dst
    ]
    assert brute.consumers(ins, 1) == [2, 3]
    assert brute.consumers(ins, 3) == [5]
    assert brute.consumers(ins, 7) == []
    n = len(ins)
    tab = np.zeros((n, 32), np.int64)
    for i in range(n):
        tab[i, 6] = 10 ** i          # long_scoreboard: one decimal digit per instruction
        tab[i, 13] = 1
    raw = gs.Trace(tab, [0], [n], order="shuffled", seed=5).raw()
    c = Canon(orc.run(brute.render([ins]), samples=raw, join="consumer"))
    assert {(s["idx"], s["rule"]) for s in c.sites()} == {(1, "RO"), (3, "CONV"), (7, "GATOM")}
    got = _ranked_rows(c)
    assert int(got[(0, 1, "RO")]["rel"]) == 10 + 100 + 1000
    assert int(got[(0, 1, "RO")]["tot"]) == 10 + 100 + 1000 + 3
    assert int(got[(0, 3, "CONV")]["tot"]) == 1000 + 100000 + 2
    assert int(got[(0, 7, "GATOM")]["tot"]) == 10 ** 7 + 1


def test_count_records_equal_expanded_samples():
    """Pre-aggregated (kernel, pc, reason, count) records (CUPTI PC-sampling shape, SURVEY §8f
    row 3) give exactly the histogram, totals and ranking of the same samples one by one,
    including invalid records (counted by their sample count)."""
    path = golden("sgemm_naive.sm_100a.sass")
    n = len(orc.sass_ops(path))
    rng = np.random.default_rng(7)
    m = 400
    rec = np.zeros((m, 4), np.uint32)
    rec[:, 0] = 0
    rec[:, 1] = rng.integers(0, n, m) * 16
    rec[:, 2] = rng.integers(0, 19, m)
    rec[:, 3] = rng.integers(0, 40, m)
    rec[:5, 1] += 4            # pc not 16-aligned -> invalid
    rec[5:8, 2] = 25           # reason >= R -> invalid
    rec[8:10, 0] = 3           # kernel out of range -> invalid
    raw = np.repeat(rec[:, :3], rec[:, 3].astype(np.int64), axis=0)
    a = Canon(orc.run(path, counts=rec))
    b = Canon(orc.run(path, samples=raw))
    assert a.H == b.H and a.N == b.N and a.R == b.R
    assert int(a.N["invalid"]) == int(rec[:10, 3].sum())
    # samples and records together add up
    c = Canon(orc.run(path, samples=raw, counts=rec))
    assert c.H == {k: 2 * v for k, v in b.H.items()}


# --------------------------------------------------------------------------- O16 register pressure
def _lrm_gpr(path):
    """nvdisasm -lrm count listing -> per function the 'GPR #' column per instruction (test-side parse)"""
    import re
    out, cur = [], None
    for t in open(path):
        m = re.match(r"\s*\.text\.(\S+):", t)
        if m:
            cur = []
            out.append(cur)
            continue
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/.*;\s*//\s*\|\s*(\d*)\s*\|", t)
        if m and cur is not None:
            cur.append(int(m.group(1) or 0))
    return out


LRM_FIXTURES = [(f"lineinfo/{k}.{d}.sass", f"lineinfo/{k}.lrm.txt") for k in LINEINFO
                for d in ("nvdisasm", "cuobjdump")] + \
    [(f"{k}.{a}.sass", f"{k}.{a}.lrm.txt") for k in ("sgemm_naive", "jacobi", "mixbench", "atomics", "conv")
     for a in ("sm_100a", "sm_70")] + \
    [(f"spill.r{c}.sm_100a.sass", f"spill.r{c}.sm_100a.lrm.txt") for c in (24, 32, 40, 64)] + \
    [(f"b200/{k}.sm_100a.sass", f"b200/{k}.sm_100a.lrm.txt") for k in ("wmma", "v8", "tmem")]


@pytest.mark.parametrize("sass,lrm", LRM_FIXTURES)
def test_register_pressure_equals_nvdisasm_life_ranges(sass, lrm):
    """O16 ("the number of additional registers needed by each SASS instruction"): the
    live-GPR count of every instruction equals nvdisasm's own life-range analysis of the same cubin
    (nvdisasm -lrm count, GPR column), from either disassembler's text; 'additional' is the
    difference to the previous instruction."""
    want = _lrm_gpr(golden(lrm))
    for text in (golden(sass),):
        got = {}
        for line in orc.run(text, liveness=True).splitlines():
            if line.startswith("L "):
                _, k, i, c, a = line.split()
                got.setdefault(int(k), []).append((int(c), int(a)))
        assert len(got) == len(want)
        for k, w in enumerate(want):
            g = got[k][:len(w)]   # nvdisasm -lrm omits the trailing NOP padding
            assert len(got[k]) >= len(w)
            assert [c for c, _ in g] == w, (sass, k)
            assert [a for _, a in g] == [w[0]] + [w[i] - w[i - 1] for i in range(1, len(w))]


# --------------------------------------------------------------------------- O16 on sm_100a forms (R38)
# nvdisasm -lrm narrow prints, per instruction, which GPRs it assigns, reads and keeps live. The
# oracle's register model must give the same three sets on every instruction: this pins the
# operand widths of the B200-native forms (R38): LDG/STG.E.ENL2.256 (two register quads), HMMA
# fragments, LDSM/STSM, LDTM/STTM (tcgen05), CS2R/LEPC pairs, IMAD.HI's 64-bit addend, conversion
# type roles, the call ABI (clobbers, callee-saved registers live at RET) and REG:N from -res-usage.
B200_NARROW = [(f"b200/{k}.sm_100a.sass", f"b200/{k}.sm_100a.narrow.txt") for k in ("wmma", "v8", "tmem")] + [
    ("torch/k1779_tcgen05_gemm.sass.xz", "torch/k1779_tcgen05_gemm.narrow.txt.xz"),
    ("torch/cubin1810.sass.xz", "torch/cubin1810.narrow.txt.xz"),
]


def _narrow(name):
    import lrm_table
    return lrm_table.parse(orc.golden_text(name).splitlines(keepends=True))


@pytest.mark.parametrize("sass,narrow", B200_NARROW)
def test_register_sets_equal_nvdisasm_table(sass, narrow):
    """Per instruction: oracle defs == nvdisasm '^'/'x' columns, uses == 'v'/'x', live == every
    marked column (the set whose size is the count of O16)."""
    want = _narrow(narrow)
    got = orc.regsets(orc.golden_text(sass))
    n = 0
    for k, fn in enumerate(want):
        for i, (txt, cnt, d, u, live) in enumerate(fn):
            gd, gu, gl = got[(k, i)]
            assert (gd, gu, gl) == (d, u, live), (sass, k, i, txt)
            assert len(gl) == cnt
            n += 1
    assert n == sum(len(f) for f in want) and n > 0


def test_real_torch_cubin_live_counts_equal_nvdisasm():
    """A real sm_100 cubin of the torch wheel (ELF 1810 of libtorch_cuda.so: 200 kernels, 38,585
    instructions, tests/golden/torch/make_torch_fixtures.sh): every L line equals nvdisasm -lrm count."""
    import tempfile
    with tempfile.NamedTemporaryFile("w", suffix=".txt", delete=False) as f:
        f.write(orc.golden_text("torch/cubin1810.lrm.txt.xz"))
    want = _lrm_gpr(f.name)
    got = {}
    for line in orc.run(orc.golden_text("torch/cubin1810.sass.xz"), liveness=True, hist=False).splitlines():
        if line.startswith("L "):
            _, k, i, c, a = line.split()
            got.setdefault(int(k), []).append(int(c))
    assert len(want) == len(got) == 200
    assert sum(len(w) for w in want) == 38585
    for k, w in enumerate(want):
        assert got[k][:len(w)] == w, k


def test_256bit_loads_are_already_vectorised():
    """a load that already moves a vector (LDG.E.64 in the paper's DP mixbench) is
    "already vectorised" and is not flagged. sm_100a's LDG.E.ENL2.256 fills two register quads
    (R38a): it counts as already vectorised, is never a VEC site, and its second quad is a
    destination (its last writer for later readers), not a source."""
    text = orc.golden_text("b200/v8.sm_100a.sass")
    c = Canon(orc.run(text))
    ops = orc.sass_ops(golden("b200/v8.sm_100a.sass"))
    ldg256 = [i for i, o in ops.items() if o.startswith("LDG") and o.endswith(".256")]
    assert len(ldg256) == 1
    assert c.kstats()[0]["vec_already"] == 1
    assert ldg256[0] not in {s["idx"] for s in c.sites("VEC")}
    # the two 32-bit loads off the second base form the only VEC group (offsets 0 and +4)
    vec = c.sites("VEC")
    assert len(vec) == 2 and {(s["min"], s["max"], s["n"], s["contig"]) for s in vec} == {("0", "4", "2", "1")}
    g = orc.regsets(text)
    i = ldg256[0]
    assert g[(0, i)][0] == set(range(4, 12))  # LDG.E.ENL2.256 R4, R8, [R6.64]: R4..R11 written
    assert g[(0, i)][1] == {6, 7}             # ... and only the address pair read


# --------------------------------------------------------------------------- all-cores oracle baseline
@pytest.mark.parametrize("name,shards", [("C2", 3), ("C2", 2), ("atomics.sm_70.sass", 2), ("b200/tmem.sm_100a.sass", 1)])
def test_sharded_oracle_equals_single_process(name, shards):
    """The all-cores oracle baseline runs independent kernel ranges in parallel and
    merges by integer sums and the total order R20: its canonical text equals the single-process
    oracle's (sm_70 param bases and -res-usage REG:N survive the split)."""
    from gen import samples as gsm
    from gen import sass as gsass
    if name == "C2":
        s = gsass.config_sass("C2")
        text, n_instr = s.text, s.n_instr
        tab = gsm.table_class_weighted(s.cls, 300_000, key=3)
        raw = gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=3).raw()
        raw = gsm.interleave(raw, gsm.invalid_raw(len(n_instr), n_instr, 100, key=3), key=4)
    else:
        text = open(golden(name), "rb").read()
        n_instr = [k["n"] for k in Canon(orc.run(text)).kstats()]
        raw = None
    want = orc.run(text, samples=raw, hlines=False) if raw is not None else orc.run(text, hist=False)
    assert orc.run_sharded(text, raw, n_instr, shards) == want


# --------------------------------------------------------------------------- CUPTI records (R39)
def _module_names(text: bytes):
    return [ln.split(b"Function : ")[1].split()[0].decode() for ln in text.split(b"\n") if b"Function : " in ln]


def test_cupti_records_equal_count_table():
    """CUPTI PC-sampling records (CUpti_PCSamplingPCData: per PC, samples per CUPTI stall-reason
    index; SURVEY [probe 8]) built from an exact count table: the oracle's histogram is
    the table; _not_issued counters (a subset of the same samples) are skipped; a foreign cubin,
    an unknown function, an unknown reason and a misaligned pc are invalid (R39)."""
    from gen import cupti
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 200_000, key=9)
    buf = cupti.Buffer(tab, _module_names(s.text), s.first_slot, s.n_instr, key=9)
    c = Canon(orc.run(s.text, cupti=buf.text, cupti_crc=buf.crc, detect=False))
    nz = np.nonzero(tab)
    assert {(int(a), int(b)): int(tab[a, b]) for a, b in zip(*nz)} == c.H
    assert c.N == {"total": str(int(tab.sum()) + buf.invalid_crc), "valid": str(int(tab.sum())),
                   "invalid": str(buf.invalid_crc)}
    assert f"C skipped={buf.skipped}" in c.text
    # any cubin (crc 0): the foreign-cubin records of known functions count too
    c0 = Canon(orc.run(s.text, cupti=buf.text, cupti_crc=0, detect=False))
    want = {(int(a), int(b)): int(tab[a, b]) for a, b in zip(*nz)}
    for slot, r, w in buf.foreign_crc_bins:
        want[(slot, r)] = want.get((slot, r), 0) + w
    assert c0.H == want and c0.N["invalid"] == str(buf.invalid_any)


def test_join_and_rank_closed_form_multi_kernel():
    """The same closed form on a module of several kernels (C2: three kernels; the cubin's five
    kernels): every R line's rel/tot/ktot come from the count table rows of the site's own slot and
    the sum over ITS kernel's slots (first_slot offsets), and the order is Python's sort of the
    R20 key — pins the kernel totals beyond the first kernel and the slot mapping of later kernels."""
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 500_000, key=21)
    raw = gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=21).raw()
    c = Canon(orc.run(s.text, samples=raw))
    first = np.asarray(s.first_slot, dtype=np.int64)
    n = np.asarray(s.n_instr, dtype=np.int64)
    ktot = [int(tab[first[k]:first[k] + n[k]].sum()) for k in range(len(n))]
    assert len(set(ktot)) == len(ktot) and len(ktot) == 3
    rel_sets = {"VEC": [6], "SPILL": [5, 6], "SHMEM": [6], "GATOM": [5], "RO": [6], "TEX": [6, 16],
                "CONV": list(range(32))}
    order = ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"]
    rows = []
    for st in c.sites():
        h = tab[first[st["k"]] + st["idx"]]
        rows.append((-int(h[rel_sets[st["rule"]]].sum()), -int(h.sum()), st["k"], st["idx"], order.index(st["rule"])))
    rows.sort()
    got = [r.split() for r in c.R]
    assert len(got) == len(rows) and {w[2] for w in rows} == {0, 1, 2}
    for q, (g, w) in enumerate(zip(got, rows)):
        assert g[:5] == ["R", str(q), str(w[2]), str(w[3]), order[w[4]]]
        assert g[5:8] == [f"rel={-w[0]}", f"tot={-w[1]}", f"ktot={ktot[w[2]]}"]
        h = tab[first[w[2]] + w[3]][:19]
        assert g[8] == "h=" + ",".join(str(int(x)) for x in h)
