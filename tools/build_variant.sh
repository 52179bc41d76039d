#!/bin/bash
# Build libdrgpum.so with extra nvcc flags into build/ab/<name>/ (A/B timing with tools/ab.sh).
# usage: tools/build_variant.sh NAME [-DFOO=1 ...]
NAME=$1; shift
mkdir -p build/ab/$NAME
P=paper_conf_asplos_linzs23_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
  -Xcompiler -O2 -Xcompiler -fvisibility=hidden -Iinclude "$@" -shared -o build/ab/$NAME/libdrgpum.so \
  $P/*.cu $P/*.cpp
