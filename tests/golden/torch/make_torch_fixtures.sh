#!/usr/bin/env bash
# Real sm_100 SASS from the torch wheel in this image (torch 2.11.0+cu128, lib/libtorch_cuda.so),
# frozen as xz-compressed text (SURVEY [probe 7]: the box's real sm_100 corpus). Provenance:
#   cubin1810            ELF file 1810 of libtorch_cuda.so (libtorch_cuda.1810.sm_100.cubin): 200
#                        elementwise/reduction kernels, 38,585 instructions, no calls
#   k1779_tcgen05_gemm   function 24 of ELF file 1779 (libtorch_cuda.1779.sm_100a.cubin): a
#                        CUTLASS tcgen05 block-scaled GEMM (UTCQMMA, LDTM, STSM, CS2R, guardrail
#                        CALL/RET subroutines), 1,789 instructions
# Each is disassembled with cuobjdump -sass -res-usage (the text gs_load_sass and the oracle read)
# and with nvdisasm -lrm count / -lrm narrow (the pins of O16: live GPRs per instruction and the
# per-register def/use/live table).
set -euo pipefail
cd "$(dirname "$0")"
LIB=$(python -c 'import torch, os; print(os.path.join(os.path.dirname(torch.__file__), "lib", "libtorch_cuda.so"))')
T=$(mktemp -d)
(cd $T && cuobjdump -xelf libtorch_cuda.1810.sm_100.cubin $LIB && cuobjdump -xelf libtorch_cuda.1779.sm_100a.cubin $LIB)
C=$T/libtorch_cuda.1810.sm_100.cubin
cuobjdump -sass -res-usage $C | xz -9 > cubin1810.sass.xz
nvdisasm -lrm count -c $C | xz -9 > cubin1810.lrm.txt.xz
nvdisasm -lrm narrow -c $C | xz -9 > cubin1810.narrow.txt.xz
C=$T/libtorch_cuda.1779.sm_100a.cubin
NAME=$(cuobjdump -sass $C | grep -o 'Function : [^ ]*' | sed -n '25p' | cut -d' ' -f3)
cuobjdump -sass -res-usage -fun "$NAME" $C | xz -9 > k1779_tcgen05_gemm.sass.xz
# the function's section of the narrow life-range table
nvdisasm -lrm narrow -c $C | awk -v n=".text.$NAME" '/^\/\/-------------------/ {on = index($0, n" ") > 0} on' \
  | xz -9 > k1779_tcgen05_gemm.narrow.txt.xz
rm -rf $T
