"""Builds libgpuscout_b200.so in-tree (nvcc, sm_100a only).

    python -m paper_conf_sc_senvs23_b200.build [--force]
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libgpuscout_b200.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CUDA_SRCS = ["api.cu", "detect.cu", "scan.cu", "attrib.cu", "rank.cu", "liveness.cu"]
CXX_SRCS = ["loader.cpp", "cupti.cpp"]
HEADERS = ["ctx.h", "record.h", "loader.h"]


def _stale(lib: str) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = [os.path.join(CSRC, f) for f in CUDA_SRCS + CXX_SRCS + HEADERS]
    deps.append(os.path.join(os.path.dirname(HERE), "include", "gpuscout_b200.h"))
    deps.append(os.path.abspath(__file__))
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd):
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        raise RuntimeError(f"build failed: {' '.join(cmd)}\n{p.stdout}\n{p.stderr}")
    return p.stderr


def build(force: bool = False, verbose: bool = False, defines: tuple[str, ...] = (), out: str | None = None) -> str:
    """defines/out: diagnostic variants only (tools/), e.g. defines=("GS_DIAG=1",), out=tools/libgs_diag.so."""
    lib = out or LIB
    if not force and not defines and not _stale(lib):
        return lib
    bdir = BUILD if not defines else os.path.join(BUILD, "diag_" + "_".join(d.replace("=", "") for d in defines))
    os.makedirs(bdir, exist_ok=True)
    common = ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-lineinfo", "-I", CSRC, *("-D" + d for d in defines)]
    jobs = []
    objs = []
    for f in CUDA_SRCS:
        o = os.path.join(bdir, f + ".o")
        objs.append(o)
        jobs.append([NVCC, *ARCH, *common, "-Xptxas", "-v", "-c", os.path.join(CSRC, f), "-o", o])
    for f in CXX_SRCS:
        o = os.path.join(bdir, f + ".o")
        objs.append(o)
        jobs.append([NVCC, *common, "-Xcompiler", "-Wall", "-c", os.path.join(CSRC, f), "-o", o])
    with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
        logs = list(ex.map(_run, jobs))
    if verbose:
        for lg in logs:
            sys.stderr.write(lg)
    tmp = lib + ".tmp"
    _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-lpthread"])
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    defs = tuple(a[2:] for a in sys.argv[1:] if a.startswith("-D"))
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, defines=defs, out=outs[0] if outs else None))
