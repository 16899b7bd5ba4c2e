#!/bin/bash
# Build libshingle.so for sm_100a (used by __graft_entry__.build()).
set -euo pipefail
cd "$(dirname "$0")"
OUT=../libshingle.so
NVCC=${NVCC:-/usr/local/cuda/bin/nvcc}
FLAGS="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v"
$NVCC $FLAGS -shared -o $OUT.tmp api.cu kernels_pass.cu kernels_group.cu exchange.cu report.cpp -ldl 2> build.log || { cat build.log; exit 1; }
mv $OUT.tmp $OUT
