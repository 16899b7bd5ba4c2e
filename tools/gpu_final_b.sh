#!/bin/bash
# Final round-2 evidence, part B: bench lines, the ncu launch list of one
# gos2m step, ncu --set full of the level-II kernels, the trial sweep.
set -u
TAG=${1:-fb}
mkdir -p gpurun_out
python bench.py > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_ref.json 2> gpurun_out/${TAG}_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline \
  > gpurun_out/${TAG}_launches.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"minhash_tile|hist_kernel|scatter_kernel|scatter2_kernel|warp_local" --launch-skip 5 -c 5 \
  -o gpurun_out/${TAG}_full_gos2m python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full_gos2m.log 2>&1
SG_BENCH_CACHE=1 python bench.py --config hub2m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
timeout 1500 python tools/sweep.py --steps 3 --warmup 1 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
SG_BENCH_CACHE=1 python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_pacific640m.json 2> gpurun_out/${TAG}_bench_pacific640m.err
ls gpurun_out | grep ${TAG}
