"""Seeded synthetic PC-sampling traces (DESIGN.md §6 "input recipe").

Shared by the oracle harness (tests) and the bench. Holds NONE of the method's arithmetic: it
only decides how many samples fall on each (slot, reason) bin (the exact-count table) and in what
order they are emitted (a seeded Feistel bijection). The expected histogram is therefore the
count table itself, a closed form independent of both implementations (SURVEY §8c O13 pin).

Sample record formats
  raw    : little-endian uint32 triples (kernel id, pc offset in bytes, reason id)  — what a
           PC-sampling collector reports; the oracle and gs_pack_samples consume it.
  packed : uint32 word = slot * R + reason with slot = first_slot[kernel] + pc/16 and R the
           active reason count — the record gs_attribute_samples consumes.
"""
from __future__ import annotations

import numpy as np

# ncu 2025.2 smsp__pcsamp_warps_issue_stalled_* reasons, fixed ids (SURVEY [probe 9]).
REASONS = ["barrier", "branch_resolving", "dispatch_stall", "drain", "imc_miss", "lg_throttle",
           "long_scoreboard", "math_pipe_throttle", "membar", "mio_throttle", "misc",
           "no_instructions", "not_selected", "selected", "short_scoreboard", "sleeping",
           "tex_throttle", "wait", "warpgroup_arrive"]
R_ACTIVE = len(REASONS)   # 19
R_SLOTS = 32              # bins per PC row

# Per-instruction class written by the SASS generator (gen/sassgen.c, enum GsClass).
CLS_ALU, CLS_MEM, CLS_CONSUMER, CLS_SMEM, CLS_BRA, CLS_BAR, CLS_OTHER = range(7)

# Reason mix per class: integer weights summing to 64 (reason id -> weight). SURVEY §8d.
_MIX = {
    CLS_ALU: {17: 20, 13: 12, 12: 12, 7: 8, 2: 4, 11: 4, 14: 4},
    CLS_MEM: {5: 24, 6: 24, 17: 8, 13: 8},
    CLS_CONSUMER: {6: 44, 17: 8, 13: 6, 12: 6},
    CLS_SMEM: {14: 24, 9: 24, 17: 8, 13: 8},
    CLS_BRA: {1: 40, 17: 12, 13: 12},
    CLS_BAR: {0: 48, 17: 8, 13: 8},
    CLS_OTHER: {17: 32, 13: 16, 12: 16},
}
MIX = np.zeros((7, R_SLOTS), dtype=np.int64)
for _c, _m in _MIX.items():
    for _r, _w in _m.items():
        MIX[_c, _r] = _w
    assert MIX[_c].sum() == 64
DOMINANT = MIX.argmax(axis=1)

M32 = np.uint64(0xFFFFFFFF)


def mix32(x: np.ndarray) -> np.ndarray:
    """lowbias32 integer hash on uint64 arrays holding 32-bit values."""
    x = x.astype(np.uint64) & M32
    x ^= x >> np.uint64(16)
    x = (x * np.uint64(0x7FEB352D)) & M32
    x ^= x >> np.uint64(15)
    x = (x * np.uint64(0x846CA68B)) & M32
    x ^= x >> np.uint64(16)
    return x


def feistel(x: np.ndarray, n: int, key: int) -> np.ndarray:
    """Seeded bijection of [0, n): 4-round balanced Feistel on 2^(2h) >= n with cycle-walking."""
    if n <= 1:
        return np.zeros_like(np.asarray(x, dtype=np.uint64))
    h = max(1, (int(n - 1).bit_length() + 1) // 2)
    mask = np.uint64((1 << h) - 1)
    keys = [int(mix32(np.array([key * 4 + r + 0x9E3779B9]))[0]) for r in range(4)]

    def once(v):
        left, right = (v >> np.uint64(h)) & mask, v & mask
        for r in range(4):
            f = mix32(right ^ np.uint64(keys[r])) & mask
            left, right = right, left ^ f
        return (left << np.uint64(h)) | right

    y = once(np.asarray(x, dtype=np.uint64))
    bad = y >= np.uint64(n)
    while bad.any():
        y[bad] = once(y[bad])
        bad = y >= np.uint64(n)
    return y


def apportion(total: int, weights: np.ndarray, key: int) -> np.ndarray:
    """Integer split of `total` proportional to integer `weights` (largest-first by hashed order)."""
    w = weights.astype(np.int64)
    W = int(w.sum())
    if W == 0 or total == 0:
        return np.zeros_like(w)
    # total * w fits int64 for total < 2^31, w < 2^32
    c = (np.int64(total) * w) // np.int64(W)
    rem = total - int(c.sum())
    if rem:
        nz = np.nonzero(w)[0]
        order = nz[np.argsort(mix32(nz.astype(np.uint64) ^ np.uint64(key & 0xFFFFFFFF)), kind="stable")]
        c[order[:rem]] += 1
    return c


def split_reasons(slot_counts: np.ndarray, slot_class: np.ndarray) -> np.ndarray:
    """[P] counts -> [P, 32] counts by the class reason mix (floor; remainder to the dominant)."""
    m = MIX[slot_class]                                   # [P, 32]
    t = (slot_counts[:, None] * m) // 64
    rem = slot_counts - t.sum(axis=1)
    t[np.arange(len(slot_counts)), DOMINANT[slot_class]] += rem
    return t


def table_weighted(slot_class: np.ndarray, n_samples: int, slot_weight: np.ndarray, key: int,
                   cover: bool = True) -> np.ndarray:
    """Exact count table: every slot >= 1 sample if `cover`, the rest apportioned by weight."""
    P = len(slot_class)
    base = np.ones(P, dtype=np.int64) if cover else np.zeros(P, dtype=np.int64)
    c = base + apportion(n_samples - int(base.sum()), slot_weight, key)
    return split_reasons(c, slot_class)


def table_class_weighted(slot_class, n_samples, key, hot_classes=(CLS_MEM, CLS_CONSUMER), hot_frac=(3, 5)):
    """C1/C2 recipe: hot classes (LDG/LDL/STL issue + load consumers) carry hot_frac of the mass."""
    slot_class = np.asarray(slot_class)
    hot = np.isin(slot_class, hot_classes)
    P = len(slot_class)
    n_cover = P
    rest = n_samples - n_cover
    n_hot = rest * hot_frac[0] // hot_frac[1] if hot.any() else 0
    c = np.ones(P, dtype=np.int64)
    if hot.any():
        c += apportion(n_hot, hot.astype(np.int64), key)
    c += apportion(rest - n_hot, (~hot).astype(np.int64) if (~hot).any() else np.ones(P, np.int64), key ^ 1)
    return split_reasons(c, slot_class)


def table_c4(slot_class, first_slot, n_instr, n_samples, key):
    """C4 recipe: Zipf(s=1) kernel weights; 80% of a kernel on a contiguous hot span (10% of its
    PCs), 20% uniform over the kernel; every PC >= 1 sample."""
    slot_class = np.asarray(slot_class)
    P = len(slot_class)
    w = np.zeros(P, dtype=np.int64)
    for k, (f, n) in enumerate(zip(first_slot, n_instr)):
        zk = (1 << 24) // (k + 1)
        nh = max(1, n // 10)
        h0 = int(mix32(np.array([key ^ (k * 7919)]))[0]) % max(1, n - nh + 1)
        w[f:f + n] += zk * 20 // n
        w[f + h0:f + h0 + nh] += zk * 80 // nh
    return table_weighted(slot_class, n_samples, w, key)


def table_c5(slot_class, hot_slots, n_samples, key, hot_share=(9, 10)):
    """C5 recipe: hot_share of all samples on len(hot_slots) PCs (70% long_scoreboard there), the
    rest uniform over the remaining PCs."""
    slot_class = np.asarray(slot_class)
    P = len(slot_class)
    n_hot = n_samples * hot_share[0] // hot_share[1]
    t = np.zeros((P, R_SLOTS), dtype=np.int64)
    per = apportion(n_hot, np.ones(len(hot_slots), np.int64), key)
    for s, c in zip(hot_slots, per):
        lsb = c * 7 // 10
        t[s, 6] += lsb
        t[s, 5] += (c - lsb) // 2
        t[s, 17] += c - lsb - (c - lsb) // 2
    cold = np.ones(P, dtype=np.int64)
    cold[list(hot_slots)] = 0
    t += split_reasons(apportion(n_samples - n_hot, cold, key ^ 5), slot_class)
    return t


class Trace:
    """Deterministic sample stream for a count table. Sample p (0 <= p < N) is computable on its
    own, so any shard [a, b) can be produced independently."""

    def __init__(self, table: np.ndarray, first_slot, n_instr, order: str = "trace", seed: int = 1):
        self.table = np.asarray(table, dtype=np.int64)
        flat = self.table.reshape(-1)
        self.nz = np.nonzero(flat)[0].astype(np.int64)            # nonzero bins, slot-major
        self.cum = np.concatenate([[0], np.cumsum(flat[self.nz])]).astype(np.int64)
        self.N = int(self.cum[-1])
        self.first_slot = np.asarray(first_slot, dtype=np.int64)
        self.n_instr = np.asarray(n_instr, dtype=np.int64)
        P = len(self.table)
        kper = np.zeros(len(self.first_slot), dtype=np.int64)
        slot_tot = self.table.sum(axis=1)
        for k, (f, n) in enumerate(zip(self.first_slot, self.n_instr)):
            kper[k] = slot_tot[f:f + n].sum()
        self.kstart = np.concatenate([[0], np.cumsum(kper)]).astype(np.int64)
        assert P == int(self.n_instr.sum())
        self.order, self.seed = order, seed

    def sorted_index(self, p: np.ndarray) -> np.ndarray:
        p = np.asarray(p, dtype=np.int64)
        if self.order == "sorted":
            return p
        if self.order == "shuffled":
            return feistel(p.astype(np.uint64), self.N, self.seed).astype(np.int64)
        # trace order: grouped by kernel, shuffled within the kernel's block
        q = np.empty_like(p)
        if len(p) > 1 and np.all(p[1:] >= p[:-1]):      # sorted positions: split by kernel blocks
            cuts = np.searchsorted(p, self.kstart, side="left")
            for kk in range(len(self.kstart) - 1):
                a, b = int(cuts[kk]), int(cuts[kk + 1])
                if a == b:
                    continue
                n_k = int(self.kstart[kk + 1] - self.kstart[kk])
                q[a:b] = self.kstart[kk] + feistel((p[a:b] - self.kstart[kk]).astype(np.uint64), n_k,
                                                   self.seed * 1000003 + kk).astype(np.int64)
            return q
        k = np.searchsorted(self.kstart, p, side="right") - 1
        for kk in np.unique(k):
            m = k == kk
            n_k = int(self.kstart[kk + 1] - self.kstart[kk])
            q[m] = self.kstart[kk] + feistel((p[m] - self.kstart[kk]).astype(np.uint64), n_k,
                                             self.seed * 1000003 + int(kk)).astype(np.int64)
        return q

    def bins(self, a: int, b: int, step: int = 1) -> np.ndarray:
        return self.bins_at(np.arange(a, b, step, dtype=np.int64))

    def bins_at(self, positions: np.ndarray) -> np.ndarray:
        q = self.sorted_index(np.asarray(positions, dtype=np.int64))
        return self.nz[np.searchsorted(self.cum, q, side="right") - 1]

    def raw_at(self, positions: np.ndarray) -> np.ndarray:
        return self.bins_to_raw(self.bins_at(positions))

    def bins_to_raw(self, bins: np.ndarray) -> np.ndarray:
        bins = np.asarray(bins, dtype=np.int64)
        slot, reason = bins // R_SLOTS, bins % R_SLOTS
        k = np.searchsorted(self.first_slot, slot, side="right") - 1
        pc = (slot - self.first_slot[k]) * 16
        return np.stack([k, pc, reason], axis=1).astype(np.uint32)

    def raw(self, a: int = 0, b: int | None = None) -> np.ndarray:
        """[b-a, 3] uint32 raw triples (kernel, pc byte offset, reason)."""
        b = self.N if b is None else b
        return self.bins_to_raw(self.bins(a, b))

    def packed(self, a: int = 0, b: int | None = None, n_reasons: int = R_ACTIVE) -> np.ndarray:
        b = self.N if b is None else b
        bins = self.bins(a, b)
        return ((bins // R_SLOTS) * n_reasons + (bins % R_SLOTS)).astype(np.uint32)


def invalid_raw(n_kernels: int, n_instr, n: int, key: int, n_reasons: int = R_ACTIVE) -> np.ndarray:
    """`n` raw samples that violate each validity condition of O13 in turn."""
    n_instr = np.asarray(n_instr)
    out = np.zeros((n, 3), dtype=np.uint32)
    h = mix32(np.arange(n, dtype=np.uint64) ^ np.uint64(key))
    for i in range(n):
        k = int(h[i] % n_kernels)
        kind = i % 4
        if kind == 0:    # kernel out of range
            out[i] = (n_kernels + int(h[i] % 7), 0, 0)
        elif kind == 1:  # pc not 16-aligned
            out[i] = (k, 16 * int(h[i] % n_instr[k]) + 4, int(h[i] % n_reasons))
        elif kind == 2:  # pc past the kernel end
            out[i] = (k, 16 * (int(n_instr[k]) + int(h[i] % 5)), 0)
        else:            # reason not active
            out[i] = (k, 16 * int(h[i] % n_instr[k]), n_reasons + int(h[i] % (R_SLOTS - n_reasons)))
    return out


def interleave(valid: np.ndarray, invalid: np.ndarray, key: int) -> np.ndarray:
    """Insert invalid rows at seeded positions (order of the valid rows is kept)."""
    n = len(valid) + len(invalid)
    pos = np.sort(feistel(np.arange(len(invalid), dtype=np.uint64), n, key).astype(np.int64))
    out = np.empty((n, 3), dtype=np.uint32)
    mask = np.zeros(n, dtype=bool)
    mask[pos] = True
    out[mask] = invalid
    out[~mask] = valid
    return out
