#!/bin/bash
# One GPU call: bench line, ncu launch list of one bench step, and
# `ncu --set full` captures of the level-II kernels (results in gpurun_out/).
set -u
TAG=${1:-r1}
python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline \
  > gpurun_out/launches_$TAG.log 2>&1
# level II at c2 = 64 (one min-hash launch, one of each grouping kernel)
timeout 900 ncu --set full --import-source on --clock-control none \
  -k regex:"minhash_tile|hist_kernel|scatter_kernel|scatter2_kernel|warp_local" --launch-skip 5 -c 5 \
  -o gpurun_out/full_$TAG python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/full_$TAG.log 2>&1
