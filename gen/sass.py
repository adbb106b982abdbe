"""ctypes front-end of gen/sassgen.c plus the per-config SASS recipes.

Test / bench input infrastructure: no method arithmetic lives here.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libgsgen.so")

SH_GENERIC, SH_C1, SH_MIXBENCH, SH_JACOBI, SH_MATMUL, SH_CHAIN, SH_ATOMICS = range(7)


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "sassgen.c")
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", LIB, src])
    return LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.gsgen_kernels.restype = ctypes.c_int64
        _lib.gsgen_kernels.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p,
                                       ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p,
                                       ctypes.c_char_p]
    return _lib


class Sass:
    """Generated SASS text + kernel table + per-instruction class bytes."""

    def __init__(self, text: bytes, sizes: np.ndarray, cls: np.ndarray):
        self.text = text
        self.n_instr = np.asarray(sizes, dtype=np.int64)
        self.first_slot = np.concatenate([[0], np.cumsum(self.n_instr)[:-1]]).astype(np.int64)
        self.cls = cls
        self.P = int(self.n_instr.sum())


def generate(shapes, sizes, seed: int, args=None, prefix: str = "k") -> Sass:
    lib = _load()
    n = len(shapes)
    shapes = np.ascontiguousarray(shapes, dtype=np.int32)
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    args = np.ascontiguousarray(np.zeros(n) if args is None else args, dtype=np.int32)
    total = int(sizes.astype(np.int64).sum())
    cls = np.zeros(total, dtype=np.uint8)
    cap = 4096 + 112 * total + 256 * n
    buf = ctypes.create_string_buffer(cap)
    got = lib.gsgen_kernels(buf, cap, n, shapes.ctypes.data, args.ctypes.data, sizes.ctypes.data,
                            ctypes.c_uint64(seed), cls.ctypes.data, prefix.encode())
    if got < 0:
        raise RuntimeError(f"gsgen_kernels failed ({got})")
    return Sass(buf.raw[:got], sizes, cls)


# ------------------------------------------------------------------ config recipes
SEED_BASE = 0x6E5C0000


def config_sass(cfg: str, scale: float = 1.0) -> Sass:
    """C1..C5 SASS. `scale` < 1 shrinks C3/C4/C5 for tests (same recipe, fewer kernels)."""
    seed = SEED_BASE + int(cfg[1])
    if cfg == "C1":
        return generate([SH_C1], [256], seed)
    if cfg == "C2":
        return generate([SH_MIXBENCH, SH_JACOBI, SH_MATMUL], [2048, 2048, 2048], seed)
    if cfg == "C3":
        n_k = max(4, int(10000 * scale))
        total = int(50_000_000 * scale)
        rng = np.random.default_rng(seed)
        s = np.exp(rng.normal(np.log(2048.0), 1.0, n_k))
        s = np.clip(s, 64, 131072)
        s = np.clip(np.round(s * total / s.sum()), 64, 131072).astype(np.int64)
        return generate([SH_GENERIC] * n_k, s, seed)
    if cfg == "C4":
        n_k = max(2, int(256 * scale))
        return generate([SH_GENERIC] * n_k, [4096] * n_k, seed)
    if cfg == "C5":
        n_k = max(2, int(256 * scale))
        shapes = [SH_GENERIC] * n_k + [SH_CHAIN] * 3
        sizes = [4096] * n_k + [128] * 3
        args = [0] * n_k + [62, 63, 64]   # chains needing exactly 63 / 64 / 65 steps
        return generate(shapes, sizes, seed, args=args)
    raise ValueError(cfg)
