#!/bin/bash
set -u
TAG=${1:-c6}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_shards.py tests/test_nccl_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
python tools/profile_run.py --config hub2m --reps 3 > gpurun_out/${TAG}_hub2m_prof.log 2>&1
SG_BENCH_CACHE=1 python bench.py --config hub2m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
SG_BENCH_CACHE=1 python bench.py --config hub2m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_bench_hub2m_b.json 2> gpurun_out/${TAG}_bench_hub2m_b.err
python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
SG_BENCH_CACHE=1 python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_pacific640m.json 2> gpurun_out/${TAG}_bench_pacific640m.err
tail -n 2 gpurun_out/${TAG}_t1.log
