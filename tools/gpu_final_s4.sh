#!/bin/bash
# Final evidence of round 2 (session 4): headline bench line, reference arm,
# ncu launch list of one gos2m step, ncu --set full of the level-II kernels
# (+ traffic json), hub2m and pacific640m lines, the trial sweep.
set -u
TAG=${1:-fs4}
mkdir -p gpurun_out
python bench.py > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_ref.json 2> gpurun_out/${TAG}_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1200 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline \
  > gpurun_out/${TAG}_launches.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"minhash_tile|hist_bytes|colscan|scatter_kernel|scatter2_kernel|warp_local" --launch-skip 6 -c 6 \
  -o gpurun_out/${TAG}_full_gos2m python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full_gos2m.log 2>&1
SG_BENCH_CACHE=1 python bench.py --config hub2m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
SG_BENCH_CACHE=1 python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_pacific640m.json 2> gpurun_out/${TAG}_bench_pacific640m.err
timeout 1500 python tools/sweep.py --steps 3 --warmup 1 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
ls gpurun_out | grep ${TAG}
