"""Histogram strategies on the GPU against closed forms at full bench sizes.

The expected histogram of a generated trace is its exact-count table (gen/samples.py), so the
whole H can be compared bin by bin even at 2^30 samples (SURVEY §8c O13 pin).
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

MODES = [0, 1, 2, 3, 4]   # AUTO, GLOBAL, PRIVATE, WINDOW, PARTITION


@pytest.fixture(scope="module")
def gs():
    import torch
    import paper_conf_sc_senvs23_b200 as g
    from paper_conf_sc_senvs23_b200 import build
    build.build()
    assert torch.cuda.is_available()
    return g


def _want(tab, row):
    """closed-form histogram in the layout of `row` bins per slot (32, or R = 19 compact)"""
    import torch
    return torch.from_numpy(np.ascontiguousarray(tab[:, :row]).astype(np.int32).reshape(-1)).cuda()


def _check(gs, s, tr, modes, words=None, rows=(32, 19)):
    import torch
    from gen.device import DeviceTrace
    if words is None:
        words = DeviceTrace(tr).packed()
    for row in rows:
        want = _want(tr.table, row)
        for mode in modes:
            for bits in ((16, 32) if mode in (0, 2, 3) else (0,)):
                ctx = gs.Context(hist_mode=mode, hist_counter_bits=bits, hist_row=row)
                ctx.load_sass(s.text)
                hist, ninv = ctx.attribute_samples(words)
                torch.cuda.synchronize()
                assert int(ninv.item()) == 0, (mode, bits, row)
                assert torch.equal(hist, want), (mode, bits, row, int((hist != want).sum().item()))
                ctx.close()


@pytest.mark.parametrize("order", ["trace", "shuffled"])
def test_c4_full_size_closed_form(gs, order):
    """C4 (2^30 samples over 1M PCs) in both orders, 32-bin and compact 19-bin rows."""
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C4")
    tab = gsm.table_c4(s.cls, s.first_slot, s.n_instr, 1 << 30, key=0x6E5C0004)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order=order, seed=1)
    _check(gs, s, tr, [0, 3, 4] if order == "trace" else [0, 1, 3, 4])


def test_c5_skew_closed_form(gs):
    """90% of 200M samples on 10 PCs: hot bins receive >> 2^16 increments per CTA, exercising the
    16-bit drain path of the shared-memory table."""
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C5")
    hot = [int(f) + 40 for f in s.first_slot[:10]]
    tab = gsm.table_c5(s.cls, hot, 200_000_000, key=0x6E5C0005)
    assert tab.max() > 1 << 20
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=2)
    _check(gs, s, tr, MODES)


def test_single_bin_drain(gs):
    """All samples on one bin: every CTA drains that 16-bit counter many times."""
    import torch
    from gen import sass as gsass
    s = gsass.config_sass("C1")
    n = 3_000_000
    words = torch.full((n,), 17 * 19 + 6, dtype=torch.int32, device="cuda")
    for mode, bits, row in [(m, b, r) for m in MODES for b in (16, 32) for r in (32, 19)]:
        ctx = gs.Context(hist_mode=mode, hist_counter_bits=bits, hist_row=row)
        ctx.load_sass(s.text)
        hist, ninv = ctx.attribute_samples(words)
        torch.cuda.synchronize()
        h = hist.view(-1, row)
        assert int(h[17, 6].item()) == n and int(h.sum().item()) == n and int(ninv.item()) == 0
        ctx.close()


@pytest.mark.parametrize("offset", [0, 1, 2, 3])
def test_unaligned_views_and_invalid_words(gs, offset):
    import torch
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 2_000_000, key=4)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=4)
    base = torch.from_numpy(tr.packed().view(np.int32)).cuda()
    bad = torch.tensor([-1, s.P * 19 + 1, s.P * 19, -16], dtype=torch.int32, device="cuda")
    buf = torch.cat([torch.zeros(offset, dtype=torch.int32, device="cuda"), bad, base, bad])
    view = buf[offset:]
    for mode, bits, row in [(m, b, r) for m in MODES for b in (16, 32) for r in (32, 19)]:
        want = _want(tab, row)
        ctx = gs.Context(hist_mode=mode, hist_counter_bits=bits, hist_row=row)
        ctx.load_sass(s.text)
        hist, ninv = ctx.attribute_samples(view)
        torch.cuda.synchronize()
        assert int(ninv.item()) == 8 and torch.equal(hist, want), mode
        # accumulate=True adds on top
        hist2, _ = ctx.attribute_samples(view, hist=hist.clone(), accumulate=True)
        assert torch.equal(hist2, 2 * want)
        ctx.close()


@pytest.mark.parametrize("n", [1, 3, 5, 4097, 100_003])
@pytest.mark.parametrize("nr", [19, 8])
def test_small_and_ragged_streams_all_modes(gs, n, nr):
    """Tiny and ragged sample counts (no whole 128-bit vector, partial tiles) with 8 or 19 active
    reasons: every strategy equals the bincount of the words (closed form), invalid words counted."""
    import torch
    from gen import sass as gsass
    s = gsass.config_sass("C2")
    rng = np.random.default_rng(n + nr)
    w = rng.integers(0, s.P * nr, n).astype(np.int64)
    w[::7] = s.P * nr + 5                      # invalid words
    bad = int((w >= s.P * nr).sum())
    want_c = np.bincount(w[w < s.P * nr], minlength=s.P * nr).astype(np.int32)
    words = torch.from_numpy(w.astype(np.int32)).cuda()
    for mode in MODES:
        for row in (32, nr):
            ctx = gs.Context(hist_mode=mode, n_reasons=nr, hist_row=row)
            ctx.load_sass(s.text)
            hist, ninv = ctx.attribute_samples(words)
            torch.cuda.synchronize()
            got = hist.view(-1, row)[:, :nr].reshape(-1).cpu().numpy()
            assert int(ninv.item()) == bad, (mode, row)
            assert np.array_equal(got, want_c), (mode, row, n)
            ctx.close()


def test_c5_trace_order_hot_words(gs):
    """C5 in trace order (90% of 200M samples on 10 PCs, grouped by kernel): tiles whose probes
    repeat a word count those hot words in registers and add them to H once per item (WINDOW); the
    histogram equals the count table in every strategy, both counter widths and row layouts."""
    from gen import samples as gsm
    from gen import sass as gsass
    s = gsass.config_sass("C5")
    hot = [int(f) + 40 for f in s.first_slot[:10]]
    tab = gsm.table_c5(s.cls, hot, 200_000_000, key=0x6E5C0005)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order="trace", seed=2)
    _check(gs, s, tr, [0, 3, 4])


def test_hot_words_with_invalid_and_foreign_words(gs):
    """Hot-word edge cases: a tile whose most frequent probe word is INVALID (never hot: it must
    still be counted as invalid), hot words of another kernel than the tile's window, and the
    word 0xFFFFFFFF itself frequent. Exact histogram and invalid count in every strategy."""
    import torch
    from gen import sass as gsass
    s = gsass.config_sass("C4", scale=0.02)
    P, R = int(sum(s.n_instr)), 19
    n = 6_000_000
    g = torch.Generator(device="cuda").manual_seed(5)
    idx = torch.arange(n, device="cuda")
    k0 = int(s.first_slot[1]) * R                       # kernel 1's first bin
    base = torch.randint(0, int(s.n_instr[0]) * R, (n,), device="cuda", generator=g)   # kernel 0
    words = torch.where(idx % 7 == 0, torch.full_like(base, k0 + 5), base)           # a foreign hot word
    words = torch.where(idx % 11 == 0, torch.full_like(base, P * R + 3), words)        # a frequent invalid word
    words = torch.where(idx % 13 == 0, torch.full_like(base, -1), words)               # 0xFFFFFFFF, frequent
    words = words.to(torch.int32)
    w64 = words.to(torch.int64) & 0xFFFFFFFF
    valid = w64 < P * R
    want_inv = int((~valid).sum().item())
    for row in (32, 19):
        want = torch.zeros(P * row, dtype=torch.int64, device="cuda")
        vw = w64[valid]
        want.index_add_(0, (vw // R) * row + vw % R, torch.ones_like(vw))
        for mode in (0, 3, 4):
            for bits in ((16, 32) if mode in (0, 3) else (0,)):
                ctx = gs.Context(hist_mode=mode, hist_counter_bits=bits, hist_row=row)
                ctx.load_sass(s.text)
                hist, ninv = ctx.attribute_samples(words)
                torch.cuda.synchronize()
                assert int(ninv.item()) == want_inv, (mode, bits, row)
                assert torch.equal(hist.to(torch.int64), want), (mode, bits, row)
                ctx.close()


def test_partition_wide_destinations_and_bucket_limit(gs):
    """PARTITION's 64-bit destination kernel (forced; the natural trigger is a copy of >= 2^32
    entries) and its fallback to WINDOW when P * R reaches 2^25 bins (1024 buckets of 2^15):
    both equal the bincount of the words."""
    import os
    import torch
    from gen import sass as gsass
    s = gsass.config_sass("C4")
    for nr in (19, 32):  # 19.9M bins (PARTITION) and 2^25 bins (falls back to WINDOW)
        rng = np.random.default_rng(nr)
        w = rng.integers(0, s.P * nr, 3_000_017).astype(np.int64)
        w[::101] = s.P * nr + 3
        bad = int((w >= s.P * nr).sum())
        want = torch.from_numpy(np.bincount(w[w < s.P * nr], minlength=s.P * nr).astype(np.int32)).cuda()
        words = torch.from_numpy(w.astype(np.int32)).cuda()
        for forced in (False, True):
            if forced:
                os.environ["GS_PART_WIDE"] = "1"
            try:
                ctx = gs.Context(hist_mode=4, n_reasons=nr, hist_row=nr)
                ctx.load_sass(s.text)
                hist, ninv = ctx.attribute_samples(words)
                torch.cuda.synchronize()
            finally:
                os.environ.pop("GS_PART_WIDE", None)
            assert int(ninv.item()) == bad, (nr, forced)
            assert torch.equal(hist, want), (nr, forced, int((hist != want).sum().item()))
            assert ctx.last_hist_mode() == (4 if nr == 19 else 3), (nr, ctx.last_hist_mode())
            ctx.close()
