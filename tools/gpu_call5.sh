#!/bin/bash
set -u
TAG=${1:-c5}
mkdir -p gpurun_out
python tools/profile_run.py --config hub2m --reps 3 > gpurun_out/${TAG}_hub2m_prof.log 2>&1
SG_NO_CLOCKS=1 python bench.py --config hub2m --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_bench_hub2m_noclk.json 2> gpurun_out/${TAG}_bench_hub2m_noclk.err
python bench.py --config hub2m --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/${TAG}_launches_hub2m.csv python bench.py --config hub2m --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-phase3 \
  > gpurun_out/${TAG}_launches_hub2m.log 2>&1
timeout 600 python -m pytest tests/test_shards.py -q > gpurun_out/${TAG}_shards.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_shards.log
tail -n 2 gpurun_out/${TAG}_shards.log
