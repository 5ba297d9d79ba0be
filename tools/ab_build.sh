#!/bin/bash
# Build library variants for tools/ab.sh: ab_build.sh name "-DFLAG=1 ..." [name "flags"] ...
set -e
mkdir -p build_ab
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC \
     -Iinclude $flags -o build_ab/$name.so paper_conf_sc_awanhedbdoy21_b200/csrc/locassm.cu paper_conf_sc_awanhedbdoy21_b200/csrc/la_cpu.cpp &
done
wait
ls -la build_ab
