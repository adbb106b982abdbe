"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, line by line.

Bit-exact bar (integer/index work): identical canonical K/S/H/N/R lines.
"""
import random

import numpy as np
import pytest

import brute
import oracle_run as orc
from oracle_run import Canon, golden

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("oracle_bin")]

FIXTURES = ["listing1.sass", "sgemm_naive.sm_100a.sass", "sgemm_naive.sm_70.sass", "jacobi.sm_100a.sass",
            "jacobi.sm_70.sass", "mixbench.sm_100a.sass", "mixbench.sm_70.sass", "atomics.sm_100a.sass",
            "atomics.sm_70.sass", "conv.sm_100a.sass", "spill.r24.sm_100a.sass", "spill.r32.sm_100a.sass",
            "spill.r40.sm_100a.sass", "spill.r64.sm_100a.sass"] + \
    [f"lineinfo/{k}.{d}.sass" for k in ("sgemm_naive", "jacobi", "mixbench", "atomics", "spill")
     for d in ("cuobjdump", "nvdisasm")] + \
    ["b200/wmma.sm_100a.sass", "b200/v8.sm_100a.sass", "b200/tmem.sm_100a.sass", "b200/abi_brx.nvdisasm.sass",
     "torch/k1779_tcgen05_gemm.sass.xz"]


@pytest.fixture(scope="module")
def gs():
    import torch
    import paper_conf_sc_senvs23_b200 as g
    from paper_conf_sc_senvs23_b200 import build
    build.build()
    assert torch.cuda.is_available()
    return g


def _ctx(gs, **kw):
    return gs.Context(**kw)


def _detect_lines(gs, text, D=64, kb=0, ke=None, **kw):
    from paper_conf_sc_senvs23_b200 import report
    ctx = _ctx(gs, trace_depth=D, **kw)
    ctx.load_sass(text)
    ctx.detect(kb, ke)
    return Canon(report.canonical(ctx, kb, ke)), ctx


def _read(name):
    if name.endswith(".xz"):
        return orc.golden_text(name).encode()
    return open(golden(name), "rb").read()


@pytest.mark.parametrize("name", FIXTURES)
def test_detect_parity_fixtures(gs, name):
    text = _read(name)
    g, _ = _detect_lines(gs, text)
    o = Canon(orc.run(text))
    assert g.K == o.K
    assert g.S == o.S


def test_detect_parity_brute_streams(gs):
    rng = random.Random(7)
    for _ in range(60):
        ks = [brute.random_stream(rng, rng.randint(1, 6)) for _ in range(rng.randint(1, 4))]
        D = rng.choice([1, 2, 3, 64])
        text = brute.render(ks)
        g, _ = _detect_lines(gs, text, D=D)
        o = Canon(orc.run(text, D=D))
        assert g.K == o.K and g.S == o.S, text


@pytest.mark.parametrize("cfg,scale", [("C1", 1), ("C2", 1), ("C3", 0.002), ("C4", 0.02), ("C5", 0.02)])
def test_detect_parity_configs(gs, cfg, scale):
    from gen import sass as gsass
    s = gsass.config_sass(cfg, scale=scale)
    g, _ = _detect_lines(gs, s.text)
    o = Canon(orc.run(s.text))
    assert g.K == o.K
    assert len(g.S) == len(o.S)
    assert g.S == o.S


def test_detect_kernel_range(gs):
    from gen import sass as gsass
    s = gsass.config_sass("C4", scale=0.03)   # 7 kernels
    for kb, ke in [(0, 3), (2, 7), (5, 5)]:
        g, _ = _detect_lines(gs, s.text, kb=kb, ke=ke)
        o = Canon(orc.run(s.text, kbegin=kb, kend=ke))
        assert g.K == o.K and g.S == o.S


def test_trace_depth_edges(gs):
    from gen import sass as gsass
    s = gsass.config_sass("C5", scale=0.01)   # contains the 63/64/65-step chains
    for D in (1, 2, 63, 64, 65, 255):
        g, _ = _detect_lines(gs, s.text, D=D)
        o = Canon(orc.run(s.text, D=D))
        assert g.S == o.S, D


# ------------------------------------------------------------------------------ full flow
def _flow(gs, text, raw, hist_mode=0, host_input=False, k=None, n_reasons=19, hist_row=32, join_mode=0):
    import torch
    from paper_conf_sc_senvs23_b200 import report
    ctx = _ctx(gs, hist_mode=hist_mode, n_reasons=n_reasons, hist_row=hist_row, join_mode=join_mode)
    ctx.load_sass(text)
    ctx.detect()
    raw_t = torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda()
    words, ninv = ctx.pack_samples(raw_t)
    if host_input:
        hist, ninv2 = ctx.attribute_samples(words.cpu().numpy())
    else:
        hist, ninv2 = ctx.attribute_samples(words)
    ranked = ctx.rank_sites(hist, k=k)
    torch.cuda.synchronize()
    n_invalid = int(ninv2.item())
    assert n_invalid == int(ninv.item())     # packing marks exactly the invalid samples
    return Canon(report.canonical(ctx, hist=hist, n_samples=len(raw), n_invalid=n_invalid, ranked=ranked)), ctx


def _samples(s, n, order, seed, n_bad=100):
    from gen import samples as gsm
    tab = gsm.table_class_weighted(s.cls, n, key=seed)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order=order, seed=seed)
    raw = tr.raw()
    bad = gsm.invalid_raw(len(s.n_instr), s.n_instr, n_bad, key=seed)
    return gsm.interleave(raw, bad, key=seed + 1), tab


@pytest.mark.parametrize("cfg,n,order,mode", [
    ("C1", 16384, "trace", 0), ("C1", 16384, "shuffled", 1), ("C1", 16384, "shuffled", 2),
    ("C2", 400_000, "trace", 0), ("C2", 400_000, "shuffled", 1), ("C2", 400_000, "shuffled", 2),
    ("C1", 16384, "trace", 3), ("C2", 400_000, "trace", 3), ("C2", 400_000, "shuffled", 3),
    ("C1", 16384, "shuffled", 4), ("C2", 400_000, "trace", 4), ("C2", 400_000, "shuffled", 4),
])
def test_full_flow_parity(gs, cfg, n, order, mode):
    from gen import sass as gsass
    s = gsass.config_sass(cfg)
    raw, tab = _samples(s, n, order, seed=11)
    g, ctx = _flow(gs, s.text, raw, hist_mode=mode)
    o = Canon(orc.run(s.text, samples=raw))
    assert g.H == o.H and g.N == o.N
    assert g.S == o.S and g.K == o.K
    assert g.R == o.R


@pytest.mark.parametrize("cfg,n,order,mode", [("C1", 16384, "shuffled", 0), ("C2", 400_000, "trace", 0),
                                              ("C2", 400_000, "shuffled", 1), ("C2", 400_000, "trace", 3),
                                              ("C2", 400_000, "shuffled", 4)])
def test_full_flow_parity_compact_rows(gs, cfg, n, order, mode):
    """gs_config.hist_row = R: histogram rows hold only the active reasons."""
    from gen import sass as gsass
    s = gsass.config_sass(cfg)
    raw, _ = _samples(s, n, order, seed=13)
    g, _ = _flow(gs, s.text, raw, hist_mode=mode, hist_row=19)
    o = Canon(orc.run(s.text, samples=raw))
    assert g.H == o.H and g.N == o.N and g.S == o.S and g.R == o.R


@pytest.mark.parametrize("row", [32, 19])
def test_rank_against_histogram_slice(gs, row):
    """gs_rank_sites_slice: a detection shard ranked against only its kernels' rows (the part a rank
    holds after the reduce-scatter) gives the rows the oracle gives for that shard; a slice that
    misses a detected kernel's slot is refused."""
    import torch
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import dist as gdist
    s = gsass.config_sass("C2")
    raw, _ = _samples(s, 300_000, "shuffled", seed=17, n_bad=0)
    ctx = _ctx(gs, hist_row=row)
    ctx.load_sass(s.text)
    raw_t = torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda()
    words, _ = ctx.pack_samples(raw_t)
    hist, _ = ctx.attribute_samples(words)
    for world in (2, 3):
        ranges = gdist.slot_ranges(s.first_slot, s.n_instr, world)
        for g_ in range(world):
            kb, ke = gdist.kernel_range(s.n_instr, g_, world)
            sb, se = ranges[g_]
            ctx.detect(kb, ke)
            part = hist[sb * row:se * row].clone()        # a separate allocation, like a received slice
            got = ctx.rank_sites(part, slot_begin=sb, slot_end=se)
            want = Canon(orc.run(s.text, samples=raw, kbegin=kb, kend=ke)).R
            from paper_conf_sc_senvs23_b200 import report
            lines = report.canonical(ctx, kb, ke, hist=hist, n_samples=len(raw), n_invalid=0, ranked=got)
            assert Canon(lines).R == want, (world, g_)
            if se > sb:
                with pytest.raises(gs.GsError, match="does not cover"):
                    ctx.rank_sites(hist[(sb + 1) * row:se * row], slot_begin=sb + 1, slot_end=se)


@pytest.mark.parametrize("name", ["jacobi", "sgemm_naive", "mixbench", "spill"])
@pytest.mark.parametrize("row", [32, 19])
def test_line_join_parity(gs, name, row):
    """GS_JOIN_LINE on nvdisasm -g text: each site joined with the sum of its source line's rows
    (R33), against the oracle's --join line; on cuobjdump text (no lines) it is the PC
    join."""
    from gen import samples as gsm
    for disasm in ("nvdisasm", "cuobjdump"):
        text = _read(f"lineinfo/{name}.{disasm}.sass")
        o_pc = Canon(orc.run(text))
        n = sum(int(k["n"]) for k in o_pc.kstats())
        first = [int(k["first"]) for k in o_pc.kstats()]
        nk = [int(k["n"]) for k in o_pc.kstats()]
        rng = np.random.default_rng(41)
        tab = np.zeros((n, 32), np.int64)
        tab[:, :19] = rng.integers(0, 30, (n, 19))
        raw = gsm.Trace(tab, first, nk, order="shuffled", seed=41).raw()
        g, _ = _flow(gs, text, raw, hist_row=row, join_mode=1)
        o = Canon(orc.run(text, samples=raw, join="line"))
        assert g.S == o.S and g.H == o.H and g.N == o.N
        assert g.R == o.R, (name, disasm)


@pytest.mark.parametrize("name", ["listing1.sass", "sgemm_naive.sm_100a.sass", "jacobi.sm_70.sass",
                                  "mixbench.sm_100a.sass", "spill.r24.sm_100a.sass", "conv.sm_100a.sass"])
@pytest.mark.parametrize("row", [32, 19])
def test_consumer_join_parity(gs, name, row):
    """GS_JOIN_CONSUMER (R37): each site joined with its PC row plus the rows of its direct
    consumers, against the oracle's --join consumer."""
    from gen import samples as gsm
    text = _read(name)
    o_pc = Canon(orc.run(text))
    first = [int(k["first"]) for k in o_pc.kstats()]
    nk = [int(k["n"]) for k in o_pc.kstats()]
    rng = np.random.default_rng(47)
    tab = np.zeros((sum(nk), 32), np.int64)
    tab[:, :19] = rng.integers(0, 30, (sum(nk), 19))
    raw = gsm.Trace(tab, first, nk, order="shuffled", seed=47).raw()
    g, _ = _flow(gs, text, raw, hist_row=row, join_mode=gs.GS_JOIN_CONSUMER)
    o = Canon(orc.run(text, samples=raw, join="consumer"))
    assert g.S == o.S and g.H == o.H and g.N == o.N
    assert g.R == o.R, name


def test_consumer_join_parity_streams_and_configs(gs):
    """GS_JOIN_CONSUMER on random tiny streams (pairs, overwrites, several kernels) and on the C2
    and scaled C4 configurations, including a detection shard ranked against its histogram slice."""
    import torch
    from gen import samples as gsm
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    rng = random.Random(53)
    for _ in range(25):
        ks = [brute.random_stream(rng, rng.randint(2, 7)) for _ in range(rng.randint(1, 3))]
        nk = [len(k) for k in ks]
        first = list(np.cumsum([0] + nk[:-1]))
        tab = np.zeros((sum(nk), 32), np.int64)
        tab[:, :19] = np.random.default_rng(rng.randrange(99)).integers(0, 5, (sum(nk), 19))
        if not tab.any():
            continue
        raw = gsm.Trace(tab, first, nk, order="shuffled", seed=3).raw()
        text = brute.render(ks)
        g, _ = _flow(gs, text, raw, join_mode=gs.GS_JOIN_CONSUMER)
        assert g.R == Canon(orc.run(text, samples=raw, join="consumer")).R, text
    for cfg, scale in (("C2", 1), ("C4", 0.02)):
        s = gsass.config_sass(cfg, scale=scale)
        raw, _ = _samples(s, 200_000, "shuffled", seed=59)
        g, _ = _flow(gs, s.text, raw, hist_row=19, join_mode=gs.GS_JOIN_CONSUMER)
        o = Canon(orc.run(s.text, samples=raw, join="consumer"))
        assert g.S == o.S and g.R == o.R, cfg
    s = gsass.config_sass("C2")
    raw, _ = _samples(s, 100_000, "shuffled", seed=61, n_bad=0)
    ctx = _ctx(gs, hist_row=19, join_mode=gs.GS_JOIN_CONSUMER)
    ctx.load_sass(s.text)
    raw_t = torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda()
    words, _ = ctx.pack_samples(raw_t)
    hist, _ = ctx.attribute_samples(words)
    for kb, ke in ((1, 2), (0, 3), (2, 3)):
        ctx.detect(kb, ke)
        sb, se = int(s.first_slot[kb]), int(s.first_slot[ke]) if ke < len(s.first_slot) else int(sum(s.n_instr))
        got = ctx.rank_sites(hist[sb * 19:se * 19].clone(), slot_begin=sb, slot_end=se)
        lines = report.canonical(ctx, kb, ke, hist=hist, n_samples=len(raw), n_invalid=0, ranked=got)
        want = Canon(orc.run(s.text, samples=raw, kbegin=kb, kend=ke, join="consumer")).R
        assert Canon(lines).R == want, (kb, ke)


def test_attribute_counts_parity(gs):
    """gs_attribute_counts: pre-aggregated (kernel, pc, reason, count) records (CUPTI PC-sampling
    shape) against the oracle's --counts, invalid records included; plus accumulate on top of
    per-sample attribution."""
    import torch
    from paper_conf_sc_senvs23_b200 import report
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    rng = np.random.default_rng(43)
    m = 50_000
    rec = np.zeros((m, 4), np.uint32)
    rec[:, 0] = rng.integers(0, len(s.n_instr), m)
    rec[:, 1] = (rng.integers(0, 1 << 20, m) % s.n_instr[rec[:, 0]]) * 16
    rec[:, 2] = rng.integers(0, 19, m)
    rec[:, 3] = rng.integers(0, 1000, m)
    rec[:7, 1] += 8
    rec[7:11, 2] = 19
    rec[11:13, 0] = len(s.n_instr)
    rec[13:15, 1] = s.n_instr[rec[13:15, 0]] * 16
    for row in (32, 19):
        ctx = _ctx(gs, hist_row=row)
        ctx.load_sass(s.text)
        ctx.detect()
        recs = torch.from_numpy(rec.view(np.int32).copy()).cuda()
        hist, ninv = ctx.attribute_counts(recs)
        ranked = ctx.rank_sites(hist)
        torch.cuda.synchronize()
        g = Canon(report.canonical(ctx, hist=hist, n_samples=int(rec[:, 3].sum()), n_invalid=int(ninv.item()),
                                   ranked=ranked))
        o = Canon(orc.run(s.text, counts=rec))
        assert g.H == o.H and g.N == o.N and g.R == o.R
        # samples + records accumulate into one histogram
        raw = rec[15:2000]
        raw = np.repeat(raw[:, :3], raw[:, 3].astype(np.int64), axis=0)
        words, _ = ctx.pack_samples(torch.from_numpy(raw.view(np.int32).copy()).cuda())
        hist2, _ = ctx.attribute_samples(words)
        hist2, _ = ctx.attribute_counts(recs, hist=hist2, accumulate=True)
        o2 = Canon(orc.run(s.text, samples=raw, counts=rec))
        h2 = hist2.cpu().numpy().reshape(-1, row)
        assert {(int(a), int(b)): int(h2[a, b]) for a, b in zip(*np.nonzero(h2))} == o2.H


def test_rank_repeated_calls(gs):
    """gs_rank_sites enqueues its sort with the key widths of the previous call and redoes it when
    the new maxima do not fit: small -> large -> small histograms on one context, each against the
    oracle."""
    import torch
    from paper_conf_sc_senvs23_b200 import report
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    ctx = _ctx(gs, hist_row=19)
    ctx.load_sass(s.text)
    ctx.detect()
    for n, seed in ((20_000, 51), (3_000_000, 52), (50_000, 53), (50_000, 54)):
        raw, _ = _samples(s, n, "shuffled", seed=seed, n_bad=0)
        words, _ = ctx.pack_samples(torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda())
        hist, _ = ctx.attribute_samples(words)
        for k in (None, 7):
            ranked = ctx.rank_sites(hist, k=k)
            g = Canon(report.canonical(ctx, hist=hist, n_samples=len(raw), n_invalid=0, ranked=ranked))
            o = Canon(orc.run(s.text, samples=raw, k=-1 if k is None else k))
            assert g.R == o.R, (n, k)


def test_detect_repeated_calls(gs):
    """gs_detect writes sites into the buffers of the previous call and rewrites after growing them
    when the totals do not fit: few -> many -> few sites on one context."""
    from gen import sass as gsass
    small = _read("listing1.sass")
    big = gsass.config_sass("C2").text
    ctx = _ctx(gs)
    for text in (small, big, small, big):
        ctx.load_sass(text)
        ctx.detect()
        from paper_conf_sc_senvs23_b200 import report
        g = Canon(report.canonical(ctx))
        o = Canon(orc.run(text))
        assert g.S == o.S and g.K == o.K
    # kernel ranges of growing size on one load
    ctx.load_sass(big)
    for kb, ke in ((0, 1), (0, 3), (1, 2), (0, 3)):
        ctx.detect(kb, ke)
        from paper_conf_sc_senvs23_b200 import report
        assert Canon(report.canonical(ctx, kb, ke)).S == Canon(orc.run(big, kbegin=kb, kend=ke)).S


def test_host_input_and_topk(gs):
    from gen import sass as gsass
    s = gsass.config_sass("C1")
    raw, _ = _samples(s, 20000, "shuffled", seed=3)
    g, _ = _flow(gs, s.text, raw, host_input=True, k=10)
    o = Canon(orc.run(s.text, samples=raw, k=10))
    assert g.H == o.H and g.R == o.R and len(g.R) == 10


def test_fewer_reasons(gs):
    from gen import sass as gsass
    s = gsass.config_sass("C1")
    raw, _ = _samples(s, 20000, "shuffled", seed=5)
    g, _ = _flow(gs, s.text, raw, n_reasons=7)
    o = Canon(orc.run(s.text, samples=raw, R=7))
    assert g.H == o.H and g.N == o.N and g.R == o.R


def test_empty_and_degenerate(gs):
    import torch
    ctx = _ctx(gs)
    assert ctx.load_sass(b"") == (0, 0)
    assert ctx.detect() == 0
    hist, ninv = ctx.attribute_samples(torch.zeros(0, dtype=torch.int32, device="cuda"))
    assert ctx.rank_sites(hist).shape == (0,)
    # a kernel without instructions between two others
    text = ("\tcode for sm_100a\n\t\tFunction : a\n        /*0000*/ LDG.E R0, desc[UR4][R2.64] ;\n"
            "\t\tFunction : empty\n\t\tFunction : c\n        /*0000*/ LDG.E R1, desc[UR4][R2.64+0x4] ;\n")
    g, _ = _detect_lines(gs, text)
    o = Canon(orc.run(text))
    assert g.K == o.K and g.S == o.S


def test_parse_error_reported(gs):
    ctx = _ctx(gs)
    with pytest.raises(gs.GsError, match="line 3"):
        ctx.load_sass("\t\tFunction : x\n        /*0000*/ NOP ;\n        /*0020*/ NOP ;\n")


# ------------------------------------------------------------------------------ register pressure
def _oracle_live(text, kb=0, ke=-1):
    out = {}
    for line in orc.run(text, liveness=True, kbegin=kb, kend=ke).splitlines():
        if line.startswith("L "):
            _, k, i, c, _a = line.split()
            out[(int(k), int(i))] = int(c)
    return out


def _gpu_live(gs, text, kb=0, ke=None):
    import torch
    ctx = _ctx(gs)
    ctx.load_sass(text)
    first, n = ctx.kernel_table()
    ke = ctx.n_kernels if ke is None else ke
    live = ctx.register_pressure(kb, ke, out=torch.full((max(1, ctx.n_instr),), -1, dtype=torch.int16,
                                                        device="cuda")).cpu().numpy()
    got = {(k, i): int(live[first[k] + i]) for k in range(kb, ke) for i in range(int(n[k]))}
    untouched = all(int(live[first[k] + i]) == -1 for k in range(ctx.n_kernels) if not kb <= k < ke
                    for i in range(int(n[k])))
    return got, untouched


LIVE_TEXTS = ["lineinfo/sgemm_naive.nvdisasm.sass", "lineinfo/mixbench.nvdisasm.sass", "lineinfo/atomics.cuobjdump.sass",
              "lineinfo/spill.nvdisasm.sass", "jacobi.sm_70.sass", "sgemm_naive.sm_70.sass", "conv.sm_100a.sass",
              "spill.r24.sm_100a.sass", "listing1.sass",
              # sm_100a register forms (R38): HMMA/LDSM/CS2R, 256-bit quads, tcgen05 LDTM/STTM with the
              # call ABI, BRX target lists, a CUTLASS tcgen05 GEMM kernel
              "b200/wmma.sm_100a.sass", "b200/v8.sm_100a.sass", "b200/tmem.sm_100a.sass",
              "b200/abi_brx.nvdisasm.sass", "torch/k1779_tcgen05_gemm.sass.xz"]


@pytest.mark.parametrize("name", LIVE_TEXTS)
def test_register_pressure_parity_fixtures(gs, name):
    """gs_register_pressure against the oracle's O16 (itself pinned to nvdisasm's life ranges)."""
    text = _read(name)
    got, _ = _gpu_live(gs, text)
    assert got == _oracle_live(text)


def test_register_pressure_parity_generated(gs):
    """Generated multi-kernel SASS (loops, spills, conversions) and random branchy streams; a
    kernel range leaves the other kernels untouched."""
    from gen import sass as gsass
    for cfg, scale in (("C1", 1.0), ("C2", 1.0), ("C3", 0.002), ("C5", 0.01)):
        s = gsass.config_sass(cfg, scale=scale) if cfg in ("C3", "C5") else gsass.config_sass(cfg)
        got, _ = _gpu_live(gs, s.text)
        assert got == _oracle_live(s.text), cfg
    s = gsass.config_sass("C2")
    got, untouched = _gpu_live(gs, s.text, 1, 2)
    assert untouched and got == _oracle_live(s.text, 1, 2)
    rng = random.Random(17)
    for _ in range(40):
        ks = [brute.random_stream(rng, rng.randint(1, 6)) for _ in range(rng.randint(1, 4))]
        text = brute.render(ks)
        got, _ = _gpu_live(gs, text)
        assert got == _oracle_live(text)


def test_rank_graph_replay(gs):
    """gs_rank_sites on a non-default stream replays its captured CUDA graph while the parameters
    repeat: repeated calls, new histogram contents in the same buffer (larger maxima: the key widths
    grow and the sort is redone) and a host output all equal a plain run on the default stream."""
    import torch
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    s = gsass.config_sass("C2")
    raw_a, _ = _samples(s, 50_000, "shuffled", seed=71, n_bad=0)
    raw_b, _ = _samples(s, 2_000_000, "shuffled", seed=73, n_bad=0)
    st = torch.cuda.Stream()

    def canon(ctx, hist, n, rows):
        return Canon(report.canonical(ctx, hist=hist, n_samples=n, n_invalid=0, ranked=rows)).R

    with torch.cuda.stream(st):
        ctx = _ctx(gs, hist_row=19)
        ctx.load_sass(s.text)
        ctx.detect()
        hist = torch.empty(ctx.n_instr * 19, dtype=torch.int32, device="cuda")
        ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
        ns = ctx.sites_device()[2]
        dev_rows = torch.empty(ns * gs.RANKED_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
        got = []
        for q, raw in enumerate((raw_a, raw_a, raw_a, raw_b, raw_b, raw_a)):
            w, _ = ctx.pack_samples(torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda())
            ctx.attribute_samples(w, hist, ninv)
            if q % 2:   # device output: the captured graph path
                n = ctx.rank_sites(hist, out=dev_rows)
                rows = dev_rows.cpu().numpy().view(gs.RANKED_DTYPE)[:n]
            else:       # host (pageable) output: plain launches
                rows = ctx.rank_sites(hist)
            got.append(canon(ctx, hist, len(raw), rows))
        st.synchronize()
    want_a = Canon(orc.run(s.text, samples=raw_a)).R
    want_b = Canon(orc.run(s.text, samples=raw_b)).R
    assert got[0] == got[1] == got[2] == got[5] == want_a
    assert got[3] == got[4] == want_b


def test_detect_graph_replay(gs):
    """gs_detect on a non-default stream (captured CUDA graph, replayed while the kernel range and
    buffers repeat): repeated and alternating kernel ranges equal the oracle's K/S lines."""
    import torch
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    s = gsass.config_sass("C4", scale=0.03)   # 7 kernels
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        ctx = _ctx(gs)
        ctx.load_sass(s.text)
        for kb, ke in [(0, 7), (0, 7), (2, 5), (2, 5), (0, 7), (5, 7), (5, 5), (5, 5), (6, 7)]:
            ctx.detect(kb, ke)
            g = Canon(report.canonical(ctx, kb, ke))
            o = Canon(orc.run(s.text, kbegin=kb, kend=ke))
            assert g.K == o.K and g.S == o.S, (kb, ke)


@pytest.mark.parametrize("order,mode", [("trace", 0), ("shuffled", 4)])
def test_c4_full_size_flow_parity(gs, order, mode):
    """The bench configuration itself (C4: 2^30 samples over 1,048,576 PCs, compact rows; trace
    order with AUTO = WINDOW, shuffled with PARTITION): detection, attribution and ranking on the GPU
    against the oracle fed the same histogram as pre-aggregated (kernel, pc, reason, count) records;
    every K, S and R line."""
    import torch
    import bench
    from gen.device import DeviceTrace
    from paper_conf_sc_senvs23_b200 import report
    s, tr = bench.build_workload("C4", order)
    tab = tr.table
    words = DeviceTrace(tr).packed()
    ctx = _ctx(gs, hist_row=19, hist_mode=mode)
    ctx.load_sass(s.text)
    ctx.detect()
    hist, ninv = ctx.attribute_samples(words)
    del words
    rows = ctx.rank_sites(hist)
    torch.cuda.synchronize()
    assert int(ninv.item()) == 0
    g = Canon(report.canonical(ctx))
    g_r = [f"R {q} {int(r['kernel'])} {int(r['idx'])} {gs.RULES[r['rule']]} rel={int(r['rel'])} "
           f"tot={int(r['tot'])} ktot={int(r['ktot'])} h={','.join(str(int(x)) for x in r['counts'][:19])}"
           for q, r in enumerate(rows)]
    slot, reason = np.nonzero(tab)
    k = np.searchsorted(s.first_slot, slot, side="right") - 1
    counts = np.stack([k, (slot - s.first_slot[k]) * 16, reason, tab[slot, reason]], axis=1).astype(np.uint32)
    o = Canon(orc.run(s.text, counts=counts, hlines=False))
    assert g.K == o.K and g.S == o.S
    assert len(g_r) == len(o.R) and g_r == o.R


def test_c3_full_size_detect_parity(gs):
    """configs[2] at full size (C3: 10,000 kernels, 50M SASS instructions, the paper's dry run):
    every K and S line (3.76M sites) equals the oracle's."""
    from gen import sass as gsass
    s = gsass.config_sass("C3")
    g, _ = _detect_lines(gs, s.text)
    o = Canon(orc.run(s.text, hist=False))
    assert g.K == o.K
    assert len(g.S) == len(o.S) and g.S == o.S


def test_real_torch_cubin_parity(gs):
    """A whole real sm_100 cubin of the torch wheel (ELF 1810 of libtorch_cuda.so, 200 kernels,
    38,585 instructions; tests/golden/torch): the GPU's K/S lines and live-register counts equal the
    oracle's, whose L lines equal nvdisasm -lrm count on every instruction (test_oracle_pins)."""
    text = _read("torch/cubin1810.sass.xz")
    g, _ = _detect_lines(gs, text)
    o = Canon(orc.run(text, hist=False))
    assert len(g.K) == 200 and g.K == o.K
    assert g.S == o.S
    got, _ = _gpu_live(gs, text)
    assert got == _oracle_live(text)


def test_reload_then_rank_graph(gs):
    """one context, modules of 3 -> many -> 3 -> 1 kernels, each detected and ranked
    through the captured rank graph (device output on a non-default stream): the kernel-total buffer
    grows with the kernel count and a reload never replays a stale graph."""
    import torch
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    mods = [gsass.config_sass("C2"), gsass.config_sass("C3", scale=0.004), gsass.config_sass("C2"),
            gsass.config_sass("C1")]
    assert len(mods[1].n_instr) > 30
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        ctx = _ctx(gs, hist_row=19)
        for q, s in enumerate(mods):
            raw, _ = _samples(s, 200_000, "shuffled", seed=91 + q, n_bad=0)
            ctx.load_sass(s.text)
            ctx.detect()
            hist = torch.empty(ctx.n_instr * 19, dtype=torch.int32, device="cuda")
            ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
            w, _ = ctx.pack_samples(torch.from_numpy(raw.view(np.int32).reshape(-1, 3).copy()).cuda())
            ctx.attribute_samples(w, hist, ninv)
            ns = ctx.sites_device()[2]
            dev_rows = torch.empty(max(ns, 1) * gs.RANKED_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
            for _ in range(2):  # capture, then replay
                n = ctx.rank_sites(hist, out=dev_rows)
                rows = dev_rows.cpu().numpy().view(gs.RANKED_DTYPE)[:n]
                got = Canon(report.canonical(ctx, hist=hist, n_samples=len(raw), n_invalid=0, ranked=rows)).R
                assert got == Canon(orc.run(s.text, samples=raw)).R, q
        st.synchronize()


@pytest.mark.parametrize("cfg,crc_filter,row", [("C2", True, 32), ("C2", False, 19), ("C1", True, 19)])
def test_cupti_ingest_parity(gs, cfg, crc_filter, row):
    """gs_cupti_stall_reasons + gs_attribute_cupti on CUPTI-shaped host
    records (CUpti_PCSamplingPCData with host name / stall-reason pointers): histogram, invalid
    and skipped weights, and the ranking equal the oracle reading the same records."""
    import torch
    from gen import cupti
    from gen import samples as gsm
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    s = gsass.config_sass(cfg)
    tab = gsm.table_class_weighted(s.cls, 300_000, key=13)
    names = [ln.split(b"Function : ")[1].split()[0].decode() for ln in s.text.split(b"\n") if b"Function : " in ln]
    buf = cupti.Buffer(tab, names, s.first_slot, s.n_instr, key=13)
    crc = buf.crc if crc_filter else 0
    ctx = _ctx(gs, hist_row=row)
    ctx.load_sass(s.text)
    ctx.detect()
    ctx.cupti_stall_reasons(*buf.table_ptrs())
    hist, ninv, skipped, nrec = ctx.attribute_cupti(buf.ptr(), buf.n, crc)
    rows = ctx.rank_sites(hist)
    torch.cuda.synchronize()
    n_inv = int(ninv.item())
    total = int(tab.sum()) + n_inv + (sum(w for _, _, w in buf.foreign_crc_bins) if not crc_filter else 0)
    g = Canon(report.canonical(ctx, hist=hist, n_samples=total, n_invalid=n_inv, ranked=rows))
    o = Canon(orc.run(s.text, cupti=buf.text, cupti_crc=crc))
    assert g.H == o.H and g.N == o.N and g.R == o.R and g.S == o.S
    assert f"C skipped={skipped}" in o.text and skipped == buf.skipped
    assert nrec == sum(int(buf.pcdata[i].stallReasonCount) for i in range(buf.n))


@pytest.mark.parametrize("cfg,scale", [("C2", 1.0), ("C4", 1.0), ("C3", 0.04)])
def test_cluster_sort_equals_cub_sort(gs, cfg, scale):
    """gs_rank_sites sorts up to 131,072 sites in one 16-CTA cluster (distributed shared memory);
    the same ranking through CUB's radix sort (GS_NO_CLUSTER_SORT=1; C3 at this scale has more
    sites than the cluster holds, so both take CUB) is identical row for row."""
    import os
    import torch
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass(cfg, scale=scale)
    tab = gsm.table_class_weighted(s.cls, 3_000_000, key=11)
    words = torch.from_numpy(gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=3).packed()
                             .view(np.int32)).cuda()
    out = []
    for no_cluster in (False, True):
        if no_cluster:
            os.environ["GS_NO_CLUSTER_SORT"] = "1"
        try:
            ctx = _ctx(gs, hist_row=19)
            ctx.load_sass(s.text)
            n_sites = ctx.detect()
            hist, _ = ctx.attribute_samples(words)
            rows = ctx.rank_sites(hist)
            torch.cuda.synchronize()
        finally:
            os.environ.pop("GS_NO_CLUSTER_SORT", None)
        out.append(rows.copy())
        ctx.close()
    assert len(out[0]) == n_sites and np.array_equal(out[0], out[1])


def test_async_detect_equals_sync(gs):
    """gs_detect with n_sites == NULL returns without synchronising; the next call that reads the
    results completes it (including the first call's buffer growth and rewrite). Sites, counters
    and the ranking equal the synchronous path's, also with work enqueued in between and with two
    asynchronous detections back to back."""
    import torch
    from gen import samples as gsm
    from gen import sass as gsass
    from paper_conf_sc_senvs23_b200 import report
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 2_000_000, key=21)
    words = torch.from_numpy(gsm.Trace(tab, s.first_slot, s.n_instr, order="trace", seed=5).packed()
                             .view(np.int32)).cuda()
    res = []
    for wait in (True, False):
        ctx = _ctx(gs, hist_row=19)
        ctx.load_sass(s.text)
        if wait:
            ctx.detect()
        else:
            assert ctx.detect(wait=False) is None       # first call: buffers grow inside the finish
            ctx.detect(0, max(1, ctx.n_kernels // 2), wait=False)
            ctx.detect(wait=False)                      # the previous one is finished first
        hist, _ = ctx.attribute_samples(words)          # enqueued behind the pending detection
        rows = ctx.rank_sites(hist)
        torch.cuda.synchronize()
        res.append((report.canonical(ctx, hist=hist, n_samples=int(tab.sum()), n_invalid=0, ranked=rows),
                    ctx.sites_device()[2]))
        ctx.close()
    assert res[0][1] == res[1][1] and res[0][0] == res[1][0]
