#!/bin/bash
# Bench lines (gos2m, hub2m, pacific640m), the integer-peak microbenchmark, the
# ncu launch list of one gos2m step and ncu --set full captures (level-II
# grouping + min-hash on gos2m at c2 = 64; pass-I tile + hub kernels on
# hub2m).  Results in gpurun_out/.
set -u
TAG=${1:-r2}
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/int_peak tools/int_peak.cu && /tmp/int_peak > gpurun_out/${TAG}_int_peak.json
python bench.py > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
python bench.py --config hub2m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline \
  > gpurun_out/${TAG}_launches.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"minhash_tile|hist_kernel|scatter_kernel|scatter2_kernel|warp_local" --launch-skip 6 -c 6 \
  -o gpurun_out/${TAG}_full_gos2m python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
  > gpurun_out/${TAG}_full_gos2m.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"minhash_tile|hub_kernel" -c 2 \
  -o gpurun_out/${TAG}_full_hub2m python tools/profile_run.py --config hub2m --c1 64 --reps 1 --pass1-only \
  > gpurun_out/${TAG}_full_hub2m.log 2>&1
python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_pacific640m.json 2> gpurun_out/${TAG}_bench_pacific640m.err
ls -la gpurun_out | tail -20
