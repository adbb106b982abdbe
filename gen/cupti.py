"""Synthetic CUPTI PC-sampling buffers (CUpti_PCSamplingPCData records, cupti_pcsampling.h of CUDA
12.9; SURVEY [probe 8]) built from an exact-count table — test / bench INPUT infrastructure, no
method arithmetic. The same records are handed to the library (ctypes structs with host pointers,
as CUPTI delivers them) and to the oracle (their text form), so both read "the same buffer".

The stall-reason table imitates cuptiPCSamplingGetStallReasons: CUPTI indices (here a seeded
permutation, not the ncu ids) with names "smsp__pcsamp_warps_issue_stalled_<reason>" and the
"_not_issued" variants; each record carries, per nonzero reason, the all-samples counter and a
not-issued counter (a subset of the same samples).
"""
from __future__ import annotations

import ctypes

import numpy as np

from .samples import R_ACTIVE, REASONS, mix32

PREFIX = "smsp__pcsamp_warps_issue_stalled_"
NAME_SIZE = 128  # CUPTI_STALL_REASON_STRING_SIZE


class StallReason(ctypes.Structure):  # CUpti_PCSamplingStallReason (packed, aligned 8)
    _pack_ = 1
    _fields_ = [("pcSamplingStallReasonIndex", ctypes.c_uint32), ("samples", ctypes.c_uint32)]


class PCData(ctypes.Structure):  # CUpti_PCSamplingPCData (packed, aligned 8: 60 -> 64 bytes)
    _pack_ = 1
    _fields_ = [("size", ctypes.c_size_t), ("cubinCrc", ctypes.c_uint64), ("pcOffset", ctypes.c_uint64),
                ("functionIndex", ctypes.c_uint32), ("pad", ctypes.c_uint32), ("functionName", ctypes.c_char_p),
                ("stallReasonCount", ctypes.c_size_t), ("stallReason", ctypes.POINTER(StallReason)),
                ("correlationId", ctypes.c_uint32), ("_tail", ctypes.c_uint32)]


assert ctypes.sizeof(StallReason) == 8 and ctypes.sizeof(PCData) == 64
PCDATA_SIZE = 60  # the `size` field a CUPTI 12.9 client sets: offsetof(correlationId) + 4


def stall_table(key: int = 7, extra_unknown: bool = True):
    """(indices, names) of a CUPTI stall-reason table: the 19 reasons and their _not_issued
    variants under seeded indices, plus one name the library does not know."""
    names = [PREFIX + r for r in REASONS] + [PREFIX + r + "_not_issued" for r in REASONS]
    if extra_unknown:
        names.append(PREFIX + "future_reason")
    perm = np.argsort(mix32(np.arange(len(names), dtype=np.uint64) * 2654435761 + key), kind="stable")
    idx = np.arange(len(names), dtype=np.uint32)[perm] * 3 + 5   # sparse, non-ncu numbering
    return idx.astype(np.uint32), names


class Buffer:
    """CUPTI records for a count table c[slot][reason] (reasons < 19) of the module (kernel names,
    first slots, sizes); plus `foreign` records of another cubin / unknown function, an unknown
    reason and a misaligned pc (all invalid). Keeps every ctypes object alive."""

    def __init__(self, table, names, first_slot, n_instr, crc: int = 0x1234ABCD5678EF01, key: int = 7,
                 n_foreign: int = 16):
        self.idx, self.names = stall_table(key)
        ix = {n: int(i) for i, n in zip(self.idx, self.names)}
        table = np.asarray(table)
        first_slot = np.asarray(first_slot, dtype=np.int64)
        n_instr = np.asarray(n_instr, dtype=np.int64)
        self.crc = crc
        self._names = [ctypes.c_char_p(n.encode()) for n in names]
        slots = np.nonzero(table[:, :R_ACTIVE].sum(axis=1))[0]
        kern = np.searchsorted(first_slot, slots, side="right") - 1
        recs, arrays, text = [], [], []
        text += [f"T {i} {n}" for i, n in zip(self.idx, self.names)]
        h = mix32(np.arange(len(slots) + 1, dtype=np.uint64) + key)
        for q, (s, k) in enumerate(zip(slots, kern)):
            rs = np.nonzero(table[s, :R_ACTIVE])[0]
            ents = []
            for r in rs:
                c = int(table[s, r])
                ents.append((ix[PREFIX + REASONS[r]], c))
                ents.append((ix[PREFIX + REASONS[r] + "_not_issued"], c * int(h[q] % 5) // 8))  # subset
            recs.append((crc, int(k), 16 * int(s - first_slot[k]), ents))
        rng = np.random.default_rng(key)
        for f in range(n_foreign):   # invalid records: foreign cubin, unknown function/reason, bad pc
            k = int(rng.integers(len(n_instr)))
            what = f % 4
            pc = 16 * int(rng.integers(n_instr[k]))
            ents = [(ix[PREFIX + REASONS[int(rng.integers(R_ACTIVE))]], int(rng.integers(1, 1000)))]
            if what == 0:
                recs.append((crc ^ 0xFF, k, pc, ents))
            elif what == 1:
                recs.append((crc, -1, pc, ents))
            elif what == 2:
                recs.append((crc, k, pc, [(ix[PREFIX + "future_reason"], int(rng.integers(1, 1000)))]))
            else:
                recs.append((crc, k, pc + 4, ents))
        # generator-side facts for the tests: not-issued weight, and the weight of the invalid
        # records for a crc filter (foreign crc invalid) or for any crc (foreign crc counted)
        self.skipped = sum(b for _, _, _, ents in recs for a, b in ents if self.names[list(self.idx).index(a)]
                           .endswith("_not_issued"))
        foreign = recs[len(recs) - n_foreign:]
        self.invalid_crc = sum(b for _, _, _, ents in foreign for _, b in ents)
        self.invalid_any = sum(b for q, (_, _, _, ents) in enumerate(foreign) if q % 4 != 0 for _, b in ents)
        self.foreign_crc_bins = [(int(first_slot[k]) + pc // 16, REASONS.index(self.names[list(self.idx).index(
            ents[0][0])][len(PREFIX):]), ents[0][1]) for q, (_, k, pc, ents) in enumerate(foreign) if q % 4 == 0]
        order = np.argsort(mix32(np.arange(len(recs), dtype=np.uint64) + key * 31), kind="stable")
        self.pcdata = (PCData * len(recs))()
        self._unknown = ctypes.c_char_p(b"_Z_not_in_this_module")
        for j, o in enumerate(order):
            crc_r, k, pc, ents = recs[o]
            arr = (StallReason * len(ents))(*[StallReason(a, b) for a, b in ents])
            arrays.append(arr)
            d = self.pcdata[j]
            d.size, d.cubinCrc, d.pcOffset = PCDATA_SIZE, crc_r, pc
            d.functionIndex = max(k, 0)
            d.functionName = self._names[k] if k >= 0 else self._unknown.value
            d.stallReasonCount = len(ents)
            d.stallReason = ctypes.cast(arr, ctypes.POINTER(StallReason))
            fname = names[k] if k >= 0 else self._unknown.value.decode()
            text.append(f"P {crc_r:#x} {fname} {pc} " + " ".join(f"{a}:{b}" for a, b in ents))
        self._arrays = arrays
        self.text = "\n".join(text) + "\n"
        self.n = len(recs)
        self._cnames = (ctypes.c_char_p * len(self.names))(*[n.encode() for n in self.names])

    def ptr(self) -> int:
        return ctypes.addressof(self.pcdata)

    def table_ptrs(self):
        """(n, pointer to uint32 indices, pointer to char* names) for gs_cupti_stall_reasons"""
        self._idx_arr = np.ascontiguousarray(self.idx, dtype=np.uint32)
        return len(self.names), self._idx_arr.ctypes.data, ctypes.addressof(self._cnames)


PCDATA_DTYPE = np.dtype({"names": ["size", "cubinCrc", "pcOffset", "functionIndex", "pad", "functionName",
                                   "stallReasonCount", "stallReason", "correlationId"],
                         "formats": [np.uint64, np.uint64, np.uint64, np.uint32, np.uint32, np.uint64, np.uint64,
                                     np.uint64, np.uint32],
                         "offsets": [0, 8, 16, 24, 28, 32, 40, 48, 56], "itemsize": 64})


class FastBuffer:
    """Bench-size CUPTI buffer (numpy, vectorised): one CUpti_PCSamplingPCData per PC with nonzero
    counts, all-samples and not-issued counters per nonzero reason, valid records only."""

    def __init__(self, table, names, first_slot, crc: int = 0x1234ABCD5678EF01, key: int = 7):
        self.idx, self.names = stall_table(key)
        ix = {n: int(i) for i, n in zip(self.idx, self.names)}
        all_ix = np.array([ix[PREFIX + r] for r in REASONS], dtype=np.uint32)
        ni_ix = np.array([ix[PREFIX + r + "_not_issued"] for r in REASONS], dtype=np.uint32)
        t = np.asarray(table)[:, :R_ACTIVE]
        first_slot = np.asarray(first_slot, dtype=np.int64)
        slots, reasons = np.nonzero(t)               # slot-major
        counts = t[slots, reasons].astype(np.uint64)
        n_ent = 2 * len(slots)
        ents = np.zeros((n_ent, 2), dtype=np.uint32)
        ents[0::2, 0] = all_ix[reasons]
        ents[0::2, 1] = counts
        ents[1::2, 0] = ni_ix[reasons]
        ents[1::2, 1] = counts // 4                  # not-issued: a subset of the same samples
        self.skipped = int((counts // 4).sum())
        self.samples = int(counts.sum())
        self.ents = ents
        pcs, start = np.unique(slots, return_index=True)
        per = np.diff(np.append(start, len(slots))) * 2
        kern = np.searchsorted(first_slot, pcs, side="right") - 1
        self._names = [ctypes.create_string_buffer(n.encode()) for n in names]
        name_addr = np.array([ctypes.addressof(b) for b in self._names], dtype=np.uint64)
        rec = np.zeros(len(pcs), dtype=PCDATA_DTYPE)
        rec["size"] = PCDATA_SIZE
        rec["cubinCrc"] = crc
        rec["pcOffset"] = 16 * (pcs - first_slot[kern])
        rec["functionIndex"] = kern
        rec["functionName"] = name_addr[kern]
        rec["stallReasonCount"] = per
        rec["stallReason"] = ents.ctypes.data + 16 * start.astype(np.uint64)  # 2 entries (8 B each) per bin
        self.rec = rec
        self.crc = crc
        self.n = len(rec)
        self.n_entries = n_ent
        self._cnames = (ctypes.c_char_p * len(self.names))(*[n.encode() for n in self.names])

    def ptr(self) -> int:
        return self.rec.ctypes.data

    def table_ptrs(self):
        self._idx_arr = np.ascontiguousarray(self.idx, dtype=np.uint32)
        return len(self.names), self._idx_arr.ctypes.data, ctypes.addressof(self._cnames)
