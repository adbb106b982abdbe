"""Multi-GPU orchestration: one process per GPU, torch.distributed for the plumbing.

  * samples are sharded contiguously: rank g owns positions [g*N/G, (g+1)*N/G);
  * kernels (detection) are sharded contiguously, balanced by instruction count;
  * the per-rank int32 histograms are combined with ONE all_reduce(SUM) (NCCL over NVLink) —
    integer addition is associative, so the result is bit-identical for any G;
  * every rank joins its own sites against the full histogram and ranks them; the exact global
    top-K is the merge of the local top-K lists under the total order (rel desc, tot desc,
    kernel, idx, rule) (R20), gathered with one all_gather.

The functions below are host logic only (ranges, merge); the device work is the library's.
"""
from __future__ import annotations

import numpy as np


def sample_range(n: int, rank: int, world: int) -> tuple[int, int]:
    return n * rank // world, n * (rank + 1) // world


def kernel_range(n_instr, rank: int, world: int) -> tuple[int, int]:
    """Contiguous kernel range whose instruction count is ~1/world of the total."""
    n_instr = np.asarray(n_instr, dtype=np.int64)
    pre = np.concatenate([[0], np.cumsum(n_instr)])
    total = int(pre[-1])

    def cut(g):
        if g <= 0:
            return 0
        if g >= world:
            return len(n_instr)
        return int(np.searchsorted(pre, total * g // world, side="left"))

    return cut(rank), cut(rank + 1)


def slot_ranges(first_slot, n_instr, world: int) -> list[tuple[int, int]]:
    """Slot range [s, e) of every rank's detection shard (kernel_range): contiguous, kernel-aligned,
    covering [0, P) exactly once."""
    first_slot = np.asarray(first_slot, dtype=np.int64)
    n_instr = np.asarray(n_instr, dtype=np.int64)
    P = int(first_slot[-1] + n_instr[-1]) if len(n_instr) else 0
    out = []
    for g in range(world):
        kb, ke = kernel_range(n_instr, g, world)
        s = int(first_slot[kb]) if kb < len(n_instr) else P
        e = int(first_slot[ke]) if ke < len(n_instr) else P
        out.append((s, e))
    return out


def reduce_scatter_hist(hist, row: int, ranges, group=None):
    """Sum the per-rank histograms (rows of `row` bins, one per slot) and leave on rank g the summed
    rows of slots ranges[g] = [s, e); returns that slice (NCCL: a new tensor; otherwise a view of
    `hist`). One collective: NCCL's
    reduce_scatter (uneven parts run as grouped ncclReduce calls); on other backends one reduce per
    part. Single process: the slice of the whole histogram."""
    import torch
    import torch.distributed as dist
    parts = [hist[s * row:e * row] for s, e in ranges]
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return parts[0] if len(parts) == 1 else hist
    me = dist.get_rank(group)
    if dist.get_backend(group) == "nccl":
        out = torch.empty_like(parts[me])  # a separate output: no aliasing of an input part
        if len({p.numel() for p in parts}) == 1 and hist.is_contiguous() and hist.numel() == out.numel() * len(parts):
            # equal slot ranges (e.g. C4: 256 equal kernels): the parts are hist itself, in rank
            # order, so the tensor form reads it in place (the list form copies the inputs first)
            dist.reduce_scatter_tensor(out, hist, op=dist.ReduceOp.SUM, group=group)
        else:
            dist.reduce_scatter(out, parts, op=dist.ReduceOp.SUM, group=group)
        return out
    if hist.is_cuda:  # gloo with device tensors (functional checks on one GPU): one all_reduce
        dist.all_reduce(hist, op=dist.ReduceOp.SUM, group=group)
        return parts[me]
    works = [dist.reduce(p, dst=g, op=dist.ReduceOp.SUM, group=group, async_op=True)
             for g, p in enumerate(parts) if p.numel()]
    for w in works:
        w.wait()
    return parts[me]


def rank_key(row) -> tuple:
    return (-int(row["rel"]), -int(row["tot"]), int(row["kernel"]), int(row["idx"]), int(row["rule"]))


def merge_topk(parts: list[np.ndarray], k: int | None) -> np.ndarray:
    """Exact global top-k from per-rank ranked lists (each already sorted by the total order)."""
    rows = np.concatenate([p for p in parts if len(p)]) if any(len(p) for p in parts) else parts[0][:0]
    if not len(rows):
        return rows
    # np.lexsort: the last key is the primary one
    order = np.lexsort((rows["rule"], rows["idx"], rows["kernel"], -rows["tot"].astype(np.int64),
                        -rows["rel"].astype(np.int64)))
    rows = rows[order]
    return rows if k is None else rows[:k]


def allreduce_hist(hist, group=None):
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(hist, op=dist.ReduceOp.SUM, group=group)
    return hist


def gather_ranked(local: np.ndarray, k: int | None, group=None) -> np.ndarray:
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return local if k is None else local[:k]
    parts = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, local if k is None else local[:k], group=group)
    return merge_topk(parts, k)
