"""Multi-GPU host logic on CPU: two gloo ranks shard kernels and samples exactly as bench.py does
with NCCL, all-reduce the int32 histogram and merge per-rank rankings; the result must equal the
single-process result (integer addition is associative; the rank order is a total order, R20).

The per-rank device work is stood in for by the CPU oracle (test infrastructure); the code under
test is paper_conf_sc_senvs23_b200.dist (ranges, all_reduce, gather + merge).
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rows_from_R(lines, RANKED_DTYPE):
    out = np.zeros(len(lines), RANKED_DTYPE)
    for q, line in enumerate(lines):
        f = line.split()
        out[q]["kernel"], out[q]["idx"] = int(f[2]), int(f[3])
        out[q]["rule"] = ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"].index(f[4])
        kv = dict(x.split("=") for x in f[5:])
        out[q]["rel"], out[q]["tot"], out[q]["ktot"] = int(kv["rel"]), int(kv["tot"]), int(kv["ktot"])
        h = [int(x) for x in kv["h"].split(",")]
        out[q]["counts"][:len(h)] = h
    return out


def _worker(rank, world, port, text, raw, P, n_instr, k, result_q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch
    import torch.distributed as dist
    import oracle_run as orc
    from oracle_run import Canon
    from paper_conf_sc_senvs23_b200 import dist as gdist
    from paper_conf_sc_senvs23_b200.binding import RANKED_DTYPE
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        a, b = gdist.sample_range(len(raw), rank, world)
        kb, ke = gdist.kernel_range(n_instr, rank, world)
        # local histogram of this rank's sample shard (stand-in for gs_attribute_samples)
        local = Canon(orc.run(text, samples=raw[a:b], detect=False))
        hist = torch.zeros(P * 32, dtype=torch.int32)
        for (slot, r), c in local.H.items():
            hist[slot * 32 + r] = c
        gdist.allreduce_hist(hist)
        # local ranking of this rank's kernels against the full histogram (stand-in for gs_rank_sites)
        mine = Canon(orc.run(text, samples=raw, kbegin=kb, kend=ke))
        rows = _rows_from_R(mine.R, RANKED_DTYPE)
        merged = gdist.gather_ranked(rows, k)
        if rank == 0:
            result_q.put((hist.numpy().copy(), merged, (kb, ke), (a, b)))
        else:
            result_q.put((None, None, (kb, ke), (a, b)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("k", [None, 25])
def test_two_rank_gloo_matches_single_process(k):
    import oracle_run as orc
    from oracle_run import Canon
    from gen import samples as gsm
    from gen import sass as gsass
    orc.build_oracle()
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 300_000, key=21)
    raw = gsm.Trace(tab, s.first_slot, s.n_instr, order="trace", seed=21).raw()
    full = Canon(orc.run(s.text, samples=raw, k=-1 if k is None else k))
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, s.text, raw, s.P, s.n_instr, k, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    hist, merged, _, _ = [r for r in res if r[0] is not None][0]
    # shards cover everything exactly once
    ranges = sorted(r[2] for r in res)
    assert ranges[0][0] == 0 and ranges[0][1] == ranges[1][0] and ranges[1][1] == len(s.n_instr)
    spans = sorted(r[3] for r in res)
    assert spans[0][0] == 0 and spans[0][1] == spans[1][0] and spans[1][1] == len(raw)
    # all-reduced histogram == single-process histogram
    want = np.zeros(s.P * 32, np.int64)
    for (slot, r), c in full.H.items():
        want[slot * 32 + r] = c
    assert np.array_equal(hist.astype(np.int64), want)
    # merged ranking == single-process ranking
    from paper_conf_sc_senvs23_b200.binding import RANKED_DTYPE
    want_rows = _rows_from_R(full.R, RANKED_DTYPE)
    assert len(merged) == len(want_rows)
    for f in ("kernel", "idx", "rule", "rel", "tot", "ktot"):
        assert np.array_equal(merged[f], want_rows[f]), f


def _rs_worker(rank, world, port, text, raw, P, first_slot, n_instr, row, result_q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch
    import torch.distributed as dist
    import oracle_run as orc
    from oracle_run import Canon
    from paper_conf_sc_senvs23_b200 import dist as gdist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        a, b = gdist.sample_range(len(raw), rank, world)
        local = Canon(orc.run(text, samples=raw[a:b], detect=False))
        hist = torch.zeros(P * row, dtype=torch.int32)
        for (slot, r), c in local.H.items():
            hist[slot * row + r] = c
        ranges = gdist.slot_ranges(first_slot, n_instr, world)
        part = gdist.reduce_scatter_hist(hist, row, ranges)
        result_q.put((rank, ranges[rank], part.numpy().copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,row", [(2, 19), (3, 32)])
def test_reduce_scatter_slices_equal_full_histogram(world, row):
    """Each rank's reduce-scattered slice (kernel-aligned slot range of its detection shard) equals
    the single-process histogram rows of that range; the slices tile [0, P)."""
    import oracle_run as orc
    from oracle_run import Canon
    from gen import samples as gsm
    from gen import sass as gsass
    orc.build_oracle()
    s = gsass.config_sass("C2")
    tab = gsm.table_class_weighted(s.cls, 200_000, key=23)
    raw = gsm.Trace(tab, s.first_slot, s.n_instr, order="shuffled", seed=23).raw()
    full = Canon(orc.run(s.text, samples=raw, detect=False))
    want = np.zeros((s.P, row), np.int64)
    for (slot, r), c in full.H.items():
        want[slot, r] = c
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rs_worker, args=(r, world, port, s.text, raw, s.P, s.first_slot, s.n_instr, row, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0][1][0] == 0 and res[-1][1][1] == s.P
    assert all(res[i][1][1] == res[i + 1][1][0] for i in range(world - 1))
    for _, (sb, se), part in res:
        assert np.array_equal(part.reshape(-1, row).astype(np.int64), want[sb:se])


def test_kernel_range_balance():
    from paper_conf_sc_senvs23_b200 import dist as gdist
    n = np.array([100, 5000, 7, 7, 3000, 2000, 1, 64] * 5)
    for world in (1, 2, 4, 8):
        cuts = [gdist.kernel_range(n, r, world) for r in range(world)]
        assert cuts[0][0] == 0 and cuts[-1][1] == len(n)
        assert all(cuts[i][1] == cuts[i + 1][0] for i in range(world - 1))
        load = [int(n[a:b].sum()) for a, b in cuts]
        assert sum(load) == int(n.sum())
        assert max(load) <= n.sum() / world + n.max()
    for world in (1, 3, 8):
        spans = [gdist.sample_range(1000003, r, world) for r in range(world)]
        assert spans[0][0] == 0 and spans[-1][1] == 1000003
        assert max(b - a for a, b in spans) - min(b - a for a, b in spans) <= 1


def test_merge_topk_total_order():
    from paper_conf_sc_senvs23_b200 import dist as gdist
    from paper_conf_sc_senvs23_b200.binding import RANKED_DTYPE
    rng = np.random.default_rng(3)
    rows = np.zeros(200, RANKED_DTYPE)
    rows["kernel"] = rng.integers(0, 4, 200)
    rows["idx"] = rng.integers(0, 50, 200)
    rows["rule"] = rng.integers(0, 7, 200)
    rows["rel"] = rng.integers(0, 5, 200)
    rows["tot"] = rng.integers(0, 5, 200)
    key = [gdist.rank_key(r) for r in rows]
    order = sorted(range(200), key=lambda i: key[i])
    parts = [rows[rows["kernel"] % 2 == g] for g in range(2)]
    parts = [p[sorted(range(len(p)), key=lambda i: gdist.rank_key(p[i]))] for p in parts]
    merged = gdist.merge_topk(parts, 17)
    assert [gdist.rank_key(r) for r in merged] == [key[i] for i in order[:17]]
