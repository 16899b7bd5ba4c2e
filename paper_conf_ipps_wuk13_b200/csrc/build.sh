#!/bin/bash
# Build libshingle.so for sm_100a (used by __graft_entry__.build()).
set -euo pipefail
cd "$(dirname "$0")"
OUT=../libshingle.so
NVCC=${NVCC:-/usr/local/cuda/bin/nvcc}
FLAGS="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v"
SRCS="api.cu kernels_pass.cu kernels_minhash.cu kernels_group.cu kernels_local.cu kernels_report.cu exchange.cu report.cpp"
if ! $NVCC $FLAGS -shared -o $OUT.tmp $SRCS -ldl > build.log 2>&1; then
  grep -E "error|Error" build.log | head -30
  exit 1
fi
mv $OUT.tmp $OUT
