#!/usr/bin/env bash
# Regenerates the frozen SASS text fixtures from tests/golden/src/*.cu with this box's
# nvcc 12.9 (cuobjdump -sass). The .sass files are committed; rerunning must give
# identical text for the same toolchain. Spill fixtures also record ptxas -v output.
set -euo pipefail
cd "$(dirname "$0")"
T=$(mktemp -d)
for arch in sm_100a sm_70; do
  for k in sgemm_naive jacobi mixbench atomics conv; do
    nvcc -arch=$arch -cubin -O3 -o $T/$k.$arch.cubin src/$k.cu
    cuobjdump -sass $T/$k.$arch.cubin > $k.$arch.sass
    nvdisasm -lrm count -c $T/$k.$arch.cubin > $k.$arch.lrm.txt   # nvdisasm's register life ranges
  done
done
for cap in 24 32 40 64; do
  nvcc -arch=sm_100a -cubin -O3 -maxrregcount=$cap -Xptxas -v -o $T/spill.$cap.cubin src/spill.cu \
     2> spill.r$cap.ptxas.txt
  cuobjdump -sass $T/spill.$cap.cubin > spill.r$cap.sm_100a.sass
  nvdisasm -lrm count -c $T/spill.$cap.cubin > spill.r$cap.sm_100a.lrm.txt
done
rm -rf $T
# Line-info pairs: ONE cubin per kernel (compiled with -lineinfo), disassembled twice — cuobjdump
# -sass (hex branch targets, no lines) and nvdisasm -g -c (".text.f:" labels, `(.L_x_N) branch
# labels, //## File "f", line N). Both texts must give the same detection (tests/test_oracle_pins.py).
mkdir -p lineinfo
T=$(mktemp -d)
for k in sgemm_naive jacobi mixbench atomics spill; do
  nvcc -arch=sm_100a -cubin -O3 -lineinfo -maxrregcount=32 -o $T/$k.cubin src/$k.cu
  cuobjdump -sass $T/$k.cubin > lineinfo/$k.cuobjdump.sass
  nvdisasm -g -c $T/$k.cubin > lineinfo/$k.nvdisasm.sass
  # nvdisasm's own register life ranges (GPR/PRED/UGPR counts per instruction): the pin of O16
  nvdisasm -lrm count -c $T/$k.cubin > lineinfo/$k.lrm.txt
done
rm -rf $T
# sm_100a-native register forms (R38): wmma (HMMA / LDSM / CS2R pairs), 256-bit vector
# loads and stores (LDG/STG.E.ENL2.256, two register quads), tcgen05 tensor memory (LDTM / STTM,
# guardrail CALL / RET subroutines). The SASS text carries the -res-usage block (REG:N, R38k);
# nvdisasm -lrm count gives the pinned live counts, -lrm narrow the per-register def/use/live table.
mkdir -p b200
T=$(mktemp -d)
for k in wmma v8 tmem; do
  nvcc -arch=sm_100a -cubin -O3 -o $T/$k.cubin src/$k.cu
  cuobjdump -sass -res-usage $T/$k.cubin > b200/$k.sm_100a.sass
  nvdisasm -lrm count -c $T/$k.cubin > b200/$k.sm_100a.lrm.txt
  nvdisasm -lrm narrow -c $T/$k.cubin > b200/$k.sm_100a.narrow.txt
done
rm -rf $T
