#!/bin/bash
# ncu --set full of the level-II grouping kernels on hub2m (c2 = 64), for the
# bench line's roofline.traffic.
set -u
TAG=${1:-nh}
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none \
  -k regex:"hist_bytes|colscan|scatter_kernel|scatter2_kernel|warp_local" --launch-skip 5 -c 5 \
  -o gpurun_out/${TAG}_full_hub2m python tools/profile_run.py --config hub2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full_hub2m.log 2>&1
echo "ncu rc=$?"
grep -E "pairs2|counts" gpurun_out/${TAG}_full_hub2m.log | tail -2
