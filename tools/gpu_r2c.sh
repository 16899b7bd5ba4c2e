#!/bin/bash
# Round-2 (session 4) re-entry call: row-duplicate measurement, a baseline
# bench line at HEAD, and an ncu source-level capture of the level-II kernels.
set -u
TAG=${1:-r2c}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
timeout 600 python tools/row_dups.py --config gos2m > gpurun_out/${TAG}_dups.json 2> gpurun_out/${TAG}_dups.err
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
timeout 1500 ncu --set full --import-source on --clock-control none \
  -k regex:"scatter_kernel|scatter2_kernel|warp_local_kernel|minhash_tile_kernel|hist_kernel" --launch-skip 5 -c 5 \
  -o gpurun_out/${TAG}_full python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full.log 2>&1
ls -la gpurun_out | tail
