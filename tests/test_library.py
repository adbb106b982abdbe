"""CPU-side checks of the product library: it builds for sm_100a, loads, and exports every entry
point include/gpuscout_b200.h declares (no compute calls without a GPU)."""
import ctypes
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    text = open(os.path.join(ROOT, "include", "gpuscout_b200.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(gs_[a-z_0-9]+)\s*\(", text)))


def test_library_builds_and_exports_header_symbols():
    from paper_conf_sc_senvs23_b200 import binding, build
    lib = build.build()
    names = declared_functions()
    assert len(names) >= 15
    L = ctypes.CDLL(lib)
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(binding.EXPORTS)
    L.gs_version.restype = ctypes.c_char_p
    assert b"sm_100a" in L.gs_version()


def test_library_is_sm100a_sass():
    from paper_conf_sc_senvs23_b200 import build
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", build.build()], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_context_requires_gpu_no_fallback():
    import torch
    import pytest
    import paper_conf_sc_senvs23_b200 as g
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(g.GsError):
        g.Context()
