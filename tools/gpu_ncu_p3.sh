#!/bin/bash
# ncu source-level captures: the windowed pass-II kernel (gos2m, c2 = 64) and
# the Phase III kernels of one report.
set -u
TAG=${1:-np}
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"minhash_win" -c 1 \
  -o gpurun_out/${TAG}_win python tools/profile_run.py --config gos2m --c2 64 --reps 1 > gpurun_out/${TAG}_win.log 2>&1
echo "win rc=$?"
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"g2_unions|mask_long|rep1_kernel|mask_rows" -c 4 \
  -o gpurun_out/${TAG}_p3 python tools/report_profile.py --config gos2m > gpurun_out/${TAG}_p3.log 2>&1
echo "p3 rc=$?"
