#!/bin/bash
# $1 = name, $2.. = files to take from working tree (others from HEAD)
set -e
name=$1; shift
d=$(mktemp -d)
git archive HEAD paper_conf_sc_senvs23_b200/csrc include | tar -x -C "$d"
for f in "$@"; do cp "$f" "$d/$f"; done
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
rm -rf "$d"; echo tools/libgs_$name.so
