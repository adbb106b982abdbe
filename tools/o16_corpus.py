"""Agreement of the oracle's register model (O16, R36/R38) with nvdisasm's life-range
table on real sm_100 SASS from the torch wheel (SURVEY [probe 7]). Test/measurement tooling only.

usage: python tools/o16_corpus.py ELF_INDEX [ELF_INDEX ...]   (indices of libtorch_cuda.so's ELF files)
Per cubin: kernels whose every instruction has the same live GPR set, and instructions with equal
sets; the oracle reads `cuobjdump -sass -res-usage` text, nvdisasm -lrm narrow is the reference."""
import os
import subprocess
import sys
import tempfile

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "tests"))
import lrm_table  # noqa: E402
import oracle_run as orc  # noqa: E402


def main():
    import torch
    lib = os.path.join(os.path.dirname(torch.__file__), "lib", "libtorch_cuda.so")
    listing = subprocess.run(["cuobjdump", "-lelf", lib], capture_output=True, text=True).stdout
    names = {int(l.split()[2].rstrip(":")): l.split()[3] for l in listing.splitlines() if l.startswith("ELF file")}
    tk = ti = tke = tie = 0
    with tempfile.TemporaryDirectory() as d:
        for idx in map(int, sys.argv[1:]):
            name = names[idx]
            subprocess.run(["cuobjdump", "-xelf", name, lib], cwd=d, capture_output=True, check=True)
            cub = os.path.join(d, name)
            text = subprocess.run(["cuobjdump", "-sass", "-res-usage", cub], capture_output=True, text=True).stdout
            nar = subprocess.run(["nvdisasm", "-lrm", "narrow", "-c", cub], capture_output=True, text=True).stdout
            want = lrm_table.parse(nar.splitlines(keepends=True))
            got = orc.regsets(text)
            ke = ie = n = 0
            for k, fn in enumerate(want):
                bad = sum(got[(k, i)][2] != live for i, (_, _, _, _, live) in enumerate(fn))
                ke += bad == 0
                ie += len(fn) - bad
                n += len(fn)
            print(f"{name}: kernels exact {ke}/{len(want)}, instructions with equal live sets {ie}/{n}")
            tk += len(want); tke += ke; ti += n; tie += ie
    print(f"TOTAL: kernels exact {tke}/{tk}, instructions {tie}/{ti} ({100.0 * tie / max(ti, 1):.1f}%)")


if __name__ == "__main__":
    main()
