"""Device-side sample-stream generation (gen/samplegen.cu) for large configs — the same stream as
gen/samples.Trace.packed(), produced on the GPU so 2^30-sample traces never touch the host.
Test / bench input infrastructure."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .samples import Trace, mix32

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libgssample.so")
SRC = os.path.join(HERE, "samplegen.cu")


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", "-o", LIB, SRC])
    return LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        _lib.gsgen_expand.argtypes = [P, P, ctypes.c_int64, P, ctypes.c_int, P, ctypes.c_int, ctypes.c_int64,
                                      ctypes.c_int64, ctypes.c_uint32, P, P]
        _lib.gsgen_expand.restype = ctypes.c_int
    return _lib


def feistel_keys(key: int) -> list[int]:
    return [int(mix32(np.array([key * 4 + r + 0x9E3779B9]))[0]) for r in range(4)]


class DeviceTrace:
    ORDER = {"sorted": 0, "shuffled": 1, "trace": 2}

    def __init__(self, trace: Trace, device: int = 0):
        import torch
        self.tr = trace
        dev = torch.device("cuda", device)
        self.dev = dev
        self.nz = torch.from_numpy(trace.nz.astype(np.int64)).to(dev)
        self.cum = torch.from_numpy(trace.cum.astype(np.int64)).to(dev)
        self.kstart = torch.from_numpy(trace.kstart.astype(np.int64)).to(dev)
        if trace.order == "trace":
            keys = np.array([feistel_keys(trace.seed * 1000003 + k) for k in range(len(trace.kstart) - 1)],
                            dtype=np.uint32).reshape(-1)
        else:
            keys = np.array(feistel_keys(trace.seed), dtype=np.uint32)
        self.keys = torch.from_numpy(keys.view(np.int32)).to(dev)
        self.N = trace.N

    def packed(self, a: int = 0, b: int | None = None, out=None, stream=None, n_reasons: int = 19):
        import torch
        b = self.N if b is None else b
        if out is None:
            out = torch.empty(b - a, dtype=torch.int32, device=self.dev)
        st = (stream or torch.cuda.current_stream(self.dev)).cuda_stream
        rc = _load().gsgen_expand(self.nz.data_ptr(), self.cum.data_ptr(), len(self.tr.nz), self.kstart.data_ptr(),
                                  len(self.tr.kstart) - 1, self.keys.data_ptr(), self.ORDER[self.tr.order], a, b,
                                  n_reasons, out.data_ptr(), ctypes.c_void_p(st))
        if rc != 0:
            raise RuntimeError(f"gsgen_expand failed ({rc})")
        return out
