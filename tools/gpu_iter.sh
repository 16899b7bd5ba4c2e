#!/bin/bash
# Quick iteration call: parity tests, a short bench line, ncu --set full of
# the level-II kernels (gos2m, c2 = 64).  Results in gpurun_out/.
set -u
TAG=${1:-it}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"bucket_c|scatter_c|minhash_rows|minhash_tile|hist_c|segsort" --launch-skip 6 -c 7 \
  -o gpurun_out/${TAG}_full python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full.log 2>&1
tail -n 2 gpurun_out/${TAG}_t1.log
