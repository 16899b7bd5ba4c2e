#!/bin/bash
set -u
TAG=${1:-c4}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
SG_DEBUG_HOST=1 python tools/profile_run.py --config hub2m --pass1-only --reps 3 > gpurun_out/${TAG}_hub2m_p1.log 2>&1
python bench.py --config hub2m --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_bench_hub2m.json 2> gpurun_out/${TAG}_bench_hub2m.err
timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/${TAG}_san_racecheck.log 2>&1
tail -n 2 gpurun_out/${TAG}_t1.log; grep -h "SUMMARY" gpurun_out/${TAG}_san_*.log
