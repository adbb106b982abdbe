"""Counting ceiling on the real C4 stream: words reduced mod (4096 slots x 19 reasons), i.e. every
sample already in its kernel's window (all C4 kernels have 4096 instructions)."""
import ctypes, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch
import bench
from gen.device import DeviceTrace
L = ctypes.CDLL(os.path.join(ROOT, "tools/microbench/gk.so"))
L.run_g.restype = ctypes.c_float
L.run_g.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_int]
import time
for order in ("trace", "shuffled"):
    t0 = time.time()
    s, tr = bench.build_workload("C4", order)
    w = DeviceTrace(tr).packed()
    torch.cuda.synchronize()
    print("generated", time.time() - t0, flush=True)
    w.remainder_(4096 * 19)   # words < 2^31: int32 remainder is exact
    torch.cuda.synchronize()
    print("reduced", time.time() - t0, flush=True)
    ms = L.run_g(w.data_ptr(), w.numel(), 4096 * 19, 148, 10)
    print(f"C4 {order} mod-window: {ms:.3f} ms  {tr.N / ms / 1e6:.1f} G samples/s")
    del w
