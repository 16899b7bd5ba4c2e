#!/bin/bash
# ncu --set full of the level-II grouping and min-hash kernels (gos2m, c2 = 64:
# one trial chunk), plus the free host memory of the box.
set -u
TAG=${1:-v3}
mkdir -p gpurun_out
free -g > gpurun_out/${TAG}_free.txt
timeout 1500 ncu --set full --import-source on --clock-control none \
  -k regex:"bucket_c|scatter_c|minhash_rows|minhash_tile|hist_c" --launch-skip 4 -c 5 \
  -o gpurun_out/${TAG}_full python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full.log 2>&1
echo "ncu rc=$?"
