#!/bin/bash
# Build libshingle.so for sm_100a (used by __graft_entry__.build()): every
# translation unit compiled in parallel, then linked into one shared library.
set -euo pipefail
cd "$(dirname "$0")"
OUT=../libshingle.so
NVCC=${NVCC:-/usr/local/cuda/bin/nvcc}
FLAGS="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v"
SRCS="api.cu kernels_sort.cu kernels_pass.cu kernels_minhash.cu kernels_group.cu kernels_local.cu kernels_report.cu exchange.cu report.cpp shards.cpp"
OBJ=${SG_BUILD_DIR:-/tmp/sg_build_$$}
mkdir -p "$OBJ"
: > build.log
pids=()
for s in $SRCS; do
  ( $NVCC $FLAGS -c -o "$OBJ/${s%.*}.o" "$s" > "$OBJ/${s%.*}.log" 2>&1 ) &
  pids+=($!)
done
fail=0
for p in "${pids[@]}"; do wait "$p" || fail=1; done
for s in $SRCS; do cat "$OBJ/${s%.*}.log" >> build.log; done
if [ $fail -ne 0 ]; then
  grep -E "error|Error" build.log | head -30
  exit 1
fi
OBJS=""
for s in $SRCS; do OBJS="$OBJS $OBJ/${s%.*}.o"; done
$NVCC -gencode arch=compute_100a,code=sm_100a -shared -o $OUT.tmp $OBJS -ldl >> build.log 2>&1
mv $OUT.tmp $OUT
rm -rf "$OBJ"
