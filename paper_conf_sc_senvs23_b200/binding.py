"""Thin ctypes binding of libgpuscout_b200.so (include/gpuscout_b200.h).

Argument marshalling only: every step of the path runs in the library's CUDA kernels (or its
host-side SASS packer for gs_load_sass). PyTorch supplies device memory (tensor data_ptr) and
the stream (torch.cuda.current_stream().cuda_stream). There is no fallback: if the library is
missing or no CUDA device is present, the calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libgpuscout_b200.so")

GS_OK, GS_E_INVAL, GS_E_PARSE, GS_E_RANGE, GS_E_CUDA, GS_E_NOMEM, GS_E_STATE = 0, -1, -2, -3, -4, -5, -6
GS_HIST_AUTO, GS_HIST_GLOBAL, GS_HIST_PRIVATE, GS_HIST_WINDOW, GS_HIST_PARTITION = 0, 1, 2, 3, 4
GS_JOIN_PC, GS_JOIN_LINE, GS_JOIN_CONSUMER = 0, 1, 2
RULES = ["VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"]
TERMS = ["NONE", "PARAM", "CONST", "ENTRY", "SREG", "MEMORY", "IMM", "TRUNC"]

SITE_DTYPE = np.dtype([("kernel", "<u4"), ("idx", "<u4"), ("rule", "u1"), ("depth", "u1"), ("term_kind", "u1"),
                       ("loop_depth", "u1"), ("term_value", "<u4"), ("chain_off", "<u4"), ("a0", "<i4"),
                       ("a1", "<i4"), ("a2", "<i4")])
assert SITE_DTYPE.itemsize == 32
RANKED_DTYPE = np.dtype([("kernel", "<u4"), ("idx", "<u4"), ("rule", "<u4"), ("pad", "<u4"), ("rel", "<u8"),
                         ("tot", "<u8"), ("ktot", "<u8"), ("counts", "<u4", (32,))])
assert RANKED_DTYPE.itemsize == 168
KSTATS_DTYPE = np.dtype([("n_gatom", "<u4"), ("n_satom", "<u4"), ("n_conv", "<u4"), ("n_vec_already", "<u4"),
                         ("n_unresolved_stores", "<u4")])


class GsConfig(ctypes.Structure):
    _fields_ = [("trace_depth", ctypes.c_uint32), ("n_reasons", ctypes.c_uint32),
                ("shmem_min_arith", ctypes.c_uint32), ("shmem_min_loads", ctypes.c_uint32),
                ("hist_mode", ctypes.c_uint32), ("hist_counter_bits", ctypes.c_uint32),
                ("hist_row", ctypes.c_uint32), ("join_mode", ctypes.c_uint32)]


class GsError(RuntimeError):
    pass


_lib = None
EXPORTS = ["gs_create", "gs_destroy", "gs_last_error", "gs_version", "gs_load_sass", "gs_kernel_table",
           "gs_kernel_name", "gs_instr_lines", "gs_detect", "gs_sites", "gs_sites_host", "gs_kernel_stats_get", "gs_pack_samples",
           "gs_attribute_samples", "gs_attribute_counts", "gs_cupti_stall_reasons", "gs_attribute_cupti", "gs_register_pressure", "gs_rank_sites",
           "gs_rank_sites_slice", "gs_last_hist_mode", "gs_last_attribute_ms", "gs_launch_count"]


def launch_count() -> int:
    return int(load_library().gs_launch_count())


def load_library(path: str = LIB_PATH):
    """Loads (does not build) the shared library and declares every exported signature."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise GsError(f"{path} not built: run `python -m paper_conf_sc_senvs23_b200.build`")
    L = ctypes.CDLL(path)
    P, U32, U64, I32, SZ = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_size_t
    sig = {
        "gs_create": (I32, [ctypes.POINTER(P), I32, P, ctypes.POINTER(GsConfig)]),
        "gs_destroy": (None, [P]),
        "gs_last_error": (ctypes.c_char_p, [P]),
        "gs_version": (ctypes.c_char_p, []),
        "gs_load_sass": (I32, [P, ctypes.c_char_p, SZ, ctypes.POINTER(U32), ctypes.POINTER(U64)]),
        "gs_kernel_table": (I32, [P, P, P, SZ]),
        "gs_kernel_name": (ctypes.c_char_p, [P, U32]),
        "gs_instr_lines": (I32, [P, P, SZ]),
        "gs_detect": (I32, [P, U32, U32, ctypes.POINTER(U64)]),
        "gs_sites": (I32, [P, ctypes.POINTER(P), ctypes.POINTER(P), ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "gs_sites_host": (I32, [P, P, SZ, P, SZ]),
        "gs_kernel_stats_get": (I32, [P, P, SZ]),
        "gs_pack_samples": (I32, [P, P, U64, P, P]),
        "gs_attribute_samples": (I32, [P, P, U64, P, P, I32]),
        "gs_attribute_counts": (I32, [P, P, U64, P, P, I32]),
        "gs_cupti_stall_reasons": (I32, [P, SZ, P, P]),
        "gs_attribute_cupti": (I32, [P, P, SZ, U64, P, P, I32, ctypes.POINTER(ctypes.c_ulonglong),
                                     ctypes.POINTER(ctypes.c_ulonglong)]),
        "gs_register_pressure": (I32, [P, U32, U32, P]),
        "gs_rank_sites": (I32, [P, P, U64, P, ctypes.POINTER(U64)]),
        "gs_rank_sites_slice": (I32, [P, P, U64, U64, U64, P, ctypes.POINTER(U64)]),
        "gs_last_hist_mode": (I32, [P]),
        "gs_last_attribute_ms": (I32, [P, ctypes.POINTER(ctypes.c_float)]),
        "gs_launch_count": (U64, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _ptr(x) -> int | None:
    """tensor / numpy array / int -> address"""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    raise TypeError(type(x))


class Context:
    """One gs_ctx bound to a CUDA device and stream (default: torch's current stream)."""

    def __init__(self, device: int | None = None, stream=None, trace_depth: int = 64, n_reasons: int = 19,
                 shmem_min_arith: int = 1, shmem_min_loads: int = 2, hist_mode: int = GS_HIST_AUTO,
                 hist_counter_bits: int = 0, hist_row: int = 32, join_mode: int = GS_JOIN_PC):
        import torch
        if not torch.cuda.is_available():
            raise GsError("no CUDA device: the library has no CPU fallback")
        self.L = load_library()
        self.device = torch.cuda.current_device() if device is None else device
        if stream is None:
            stream = torch.cuda.current_stream(self.device)
        self.torch_stream = stream
        handle = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        cfg = GsConfig(trace_depth, n_reasons, shmem_min_arith, shmem_min_loads, hist_mode, hist_counter_bits,
                       hist_row, join_mode)
        self.n_reasons = n_reasons
        self.hist_row = hist_row or 32  # bins per histogram row: 32, or n_reasons (compact)
        self.trace_depth = trace_depth
        self.cfg = cfg
        h = ctypes.c_void_p()
        rc = self.L.gs_create(ctypes.byref(h), self.device, ctypes.c_void_p(handle), ctypes.byref(cfg))
        if rc != GS_OK:
            raise GsError(f"gs_create failed ({rc})")
        self.h = h
        self.n_kernels = 0
        self.n_instr = 0

    def close(self):
        if getattr(self, "h", None):
            self.L.gs_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc, what):
        if rc != GS_OK:
            msg = self.L.gs_last_error(self.h).decode(errors="replace")
            raise GsError(f"{what} failed ({rc}): {msg}")

    # ---- a-1
    def load_sass(self, text) -> tuple[int, int]:
        b = text.encode() if isinstance(text, str) else bytes(text)
        nk, ni = ctypes.c_uint32(), ctypes.c_uint64()
        self._check(self.L.gs_load_sass(self.h, b, len(b), ctypes.byref(nk), ctypes.byref(ni)), "gs_load_sass")
        self.n_kernels, self.n_instr = nk.value, ni.value
        return self.n_kernels, self.n_instr

    def kernel_table(self) -> tuple[np.ndarray, np.ndarray]:
        f = np.zeros(self.n_kernels, np.uint32)
        n = np.zeros(self.n_kernels, np.uint32)
        self._check(self.L.gs_kernel_table(self.h, f.ctypes.data, n.ctypes.data, self.n_kernels), "gs_kernel_table")
        return f, n

    def kernel_name(self, k: int) -> str:
        s = self.L.gs_kernel_name(self.h, k)
        return s.decode() if s else ""

    def instr_lines(self) -> np.ndarray:
        out = np.zeros(self.n_instr, np.int32)
        if self.n_instr:
            self._check(self.L.gs_instr_lines(self.h, out.ctypes.data, self.n_instr), "gs_instr_lines")
        return out

    # ---- a-2 .. a-7
    def detect(self, k_begin: int = 0, k_end: int | None = None, wait: bool = True) -> int | None:
        """gs_detect; wait=False enqueues it without synchronising (n_sites NULL): the site count
        and counters are resolved by the next call that reads them (sites, stats, rank)."""
        k_end = self.n_kernels if k_end is None else k_end
        if not wait:
            self._check(self.L.gs_detect(self.h, k_begin, k_end, None), "gs_detect")
            return None
        ns = ctypes.c_uint64()
        self._check(self.L.gs_detect(self.h, k_begin, k_end, ctypes.byref(ns)), "gs_detect")
        return ns.value

    def sites_device(self):
        """(device ptr of gs_site[n], device ptr of chain pool, n_sites, n_chain)"""
        ds, dc = ctypes.c_void_p(), ctypes.c_void_p()
        ns, nc = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self.L.gs_sites(self.h, ctypes.byref(ds), ctypes.byref(dc), ctypes.byref(ns), ctypes.byref(nc)),
                    "gs_sites")
        return ds.value, dc.value, ns.value, nc.value

    def sites(self) -> tuple[np.ndarray, np.ndarray]:
        """Host copies (numpy) of the sites and the chain pool."""
        _, _, ns, nc = self.sites_device()
        sites = np.zeros(ns, SITE_DTYPE)
        chain = np.zeros(nc, np.uint32)
        self._check(self.L.gs_sites_host(self.h, sites.ctypes.data if ns else None, ns,
                                         chain.ctypes.data if nc else None, nc), "gs_sites_host")
        return sites, chain

    def kernel_stats(self) -> np.ndarray:
        out = np.zeros(self.n_kernels, KSTATS_DTYPE)
        if self.n_kernels:
            self._check(self.L.gs_kernel_stats_get(self.h, out.ctypes.data, self.n_kernels), "gs_kernel_stats_get")
        return out

    # ---- a-8, a-9
    def pack_samples(self, raw, words=None, n_invalid=None):
        import torch
        n = raw.shape[0]
        if words is None:
            words = torch.empty(n, dtype=torch.int32, device=raw.device)
        if n_invalid is None:
            n_invalid = torch.zeros(1, dtype=torch.int64, device=raw.device)
        self._check(self.L.gs_pack_samples(self.h, raw.data_ptr(), n, words.data_ptr(), n_invalid.data_ptr()),
                    "gs_pack_samples")
        return words, n_invalid

    def attribute_samples(self, samples, hist=None, n_invalid=None, accumulate: bool = False):
        """samples: int32/uint32 tensor (cuda or cpu) or numpy array of packed words."""
        import torch
        dev = torch.device("cuda", self.device)
        if hist is None:
            hist = torch.empty(self.n_instr * self.hist_row, dtype=torch.int32, device=dev)
        if n_invalid is None:
            n_invalid = torch.zeros(1, dtype=torch.int64, device=dev)
        n = samples.shape[0] if hasattr(samples, "shape") else len(samples)
        self._check(self.L.gs_attribute_samples(self.h, _ptr(samples), n, hist.data_ptr(), n_invalid.data_ptr(),
                                                1 if accumulate else 0), "gs_attribute_samples")
        return hist, n_invalid

    def attribute_counts(self, recs, hist=None, n_invalid=None, accumulate: bool = False):
        """recs: device int32/uint32 tensor [M, 4] of pre-aggregated (kernel, pc, reason, count)."""
        import torch
        dev = torch.device("cuda", self.device)
        if hist is None:
            hist = torch.empty(self.n_instr * self.hist_row, dtype=torch.int32, device=dev)
        if n_invalid is None:
            n_invalid = torch.zeros(1, dtype=torch.int64, device=dev)
        self._check(self.L.gs_attribute_counts(self.h, recs.data_ptr(), recs.shape[0], hist.data_ptr(),
                                               n_invalid.data_ptr(), 1 if accumulate else 0), "gs_attribute_counts")
        return hist, n_invalid

    def cupti_stall_reasons(self, n: int, index_ptr: int, names_ptr: int):
        """the stall-reason table of cuptiPCSamplingGetStallReasons: n CUPTI indices (uint32 array
        address) and their names (char* array address)"""
        self._check(self.L.gs_cupti_stall_reasons(self.h, n, index_ptr, names_ptr), "gs_cupti_stall_reasons")

    def attribute_cupti(self, pc_data_ptr: int, n_pcs: int, cubin_crc: int = 0, hist=None, n_invalid=None,
                        accumulate: bool = False):
        """CUpti_PCSamplingPCData[n_pcs] at host address pc_data_ptr -> histogram. Returns
        (hist, n_invalid device tensor, skipped samples, flattened entries)."""
        import torch
        dev = torch.device("cuda", self.device)
        if hist is None:
            hist = torch.empty(self.n_instr * self.hist_row, dtype=torch.int32, device=dev)
        if n_invalid is None:
            n_invalid = torch.zeros(1, dtype=torch.int64, device=dev)
        sk, nr = ctypes.c_ulonglong(), ctypes.c_ulonglong()
        self._check(self.L.gs_attribute_cupti(self.h, pc_data_ptr, n_pcs, cubin_crc, hist.data_ptr(), n_invalid.data_ptr(),
                                              1 if accumulate else 0, ctypes.byref(sk), ctypes.byref(nr)),
                    "gs_attribute_cupti")
        return hist, n_invalid, sk.value, nr.value

    def register_pressure(self, k_begin: int = 0, k_end: int | None = None, out=None):
        """Live GPRs per instruction (int16 device tensor indexed by slot; kernels outside
        [k_begin, k_end) untouched). Additional registers of slot i: out[i] - out[i-1]."""
        import torch
        k_end = self.n_kernels if k_end is None else k_end
        if out is None:
            out = torch.zeros(max(1, self.n_instr), dtype=torch.int16, device=torch.device("cuda", self.device))
        self._check(self.L.gs_register_pressure(self.h, k_begin, k_end, out.data_ptr()), "gs_register_pressure")
        return out

    def last_hist_mode(self) -> int:
        return self.L.gs_last_hist_mode(self.h)

    def last_attribute_ms(self) -> float:
        """GPU time of the last device-input attribute_samples call (events around its kernels)."""
        ms = ctypes.c_float()
        self._check(self.L.gs_last_attribute_ms(self.h, ctypes.byref(ms)), "gs_last_attribute_ms")
        return ms.value

    # ---- a-11, a-12
    def rank_sites(self, hist, k: int | None = None, out=None, slot_begin: int = 0,
                   slot_end: int | None = None) -> np.ndarray:
        """Returns a numpy RANKED_DTYPE array (host) or fills `out` (a device uint8 tensor of k*168 B).
        `hist` holds the rows of slots [slot_begin, slot_end) (default: all slots)."""
        kk = (1 << 64) - 1 if k is None else k
        slot_end = self.n_instr if slot_end is None else slot_end
        n_out = ctypes.c_uint64()
        if out is None:
            _, _, ns, _ = self.sites_device()
            m = ns if k is None else min(k, ns)
            res = np.zeros(m, RANKED_DTYPE)
            self._check(self.L.gs_rank_sites_slice(self.h, hist.data_ptr(), slot_begin, slot_end, kk,
                                                   res.ctypes.data if m else None, ctypes.byref(n_out)),
                        "gs_rank_sites")
            return res[: n_out.value]
        self._check(self.L.gs_rank_sites_slice(self.h, hist.data_ptr(), slot_begin, slot_end, kk, _ptr(out),
                                               ctypes.byref(n_out)), "gs_rank_sites")
        return n_out.value


# ------------------------------------------------------------------------- C-ABI-named functions
def gs_load_sass(ctx: Context, text) -> tuple[int, int]:
    return ctx.load_sass(text)


def gs_detect(ctx: Context, k_begin: int = 0, k_end: int | None = None) -> int:
    return ctx.detect(k_begin, k_end)


def gs_pack_samples(ctx: Context, raw, words=None, n_invalid=None):
    return ctx.pack_samples(raw, words, n_invalid)


def gs_attribute_samples(ctx: Context, samples, hist=None, n_invalid=None, accumulate: bool = False):
    return ctx.attribute_samples(samples, hist, n_invalid, accumulate)


def gs_attribute_counts(ctx: Context, recs, hist=None, n_invalid=None, accumulate: bool = False):
    return ctx.attribute_counts(recs, hist, n_invalid, accumulate)


def gs_register_pressure(ctx: Context, k_begin: int = 0, k_end: int | None = None, out=None):
    return ctx.register_pressure(k_begin, k_end, out)


def gs_rank_sites(ctx: Context, hist, k: int | None = None, out=None):
    return ctx.rank_sites(hist, k, out)


def gs_rank_sites_slice(ctx: Context, hist, slot_begin: int, slot_end: int, k: int | None = None, out=None):
    return ctx.rank_sites(hist, k, out, slot_begin=slot_begin, slot_end=slot_end)
