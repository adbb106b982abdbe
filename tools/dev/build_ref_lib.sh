#!/bin/bash
# Developer helper: builds the library at git revision $1 into tools/libgs_$2.so (same-box A/B timing).
set -e
rev=$1; name=$2
d=$(mktemp -d)
git archive "$rev" paper_conf_sc_senvs23_b200/csrc include | tar -x -C "$d"
objs=""
for f in api detect scan attrib rank liveness; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC -lineinfo -I "$d/paper_conf_sc_senvs23_b200/csrc" -c "$d/paper_conf_sc_senvs23_b200/csrc/$f.cu" -o "$d/$f.o" &
  objs="$objs $d/$f.o"
done
for f in loader cupti; do
  /usr/local/cuda/bin/nvcc -O3 -std=c++17 -Xcompiler -fPIC -I "$d/paper_conf_sc_senvs23_b200/csrc" -c "$d/paper_conf_sc_senvs23_b200/csrc/$f.cpp" -o "$d/$f.o" &
  objs="$objs $d/$f.o"
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o "tools/libgs_$name.so" $objs -lpthread
rm -rf "$d"
echo "tools/libgs_$name.so"
