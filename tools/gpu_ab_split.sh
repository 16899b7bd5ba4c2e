#!/bin/bash
set -u
TAG=${1:-ab}
mkdir -p gpurun_out
SG_SPLIT_ATOMIC=1 timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_multirank_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_b0.json 2> gpurun_out/${TAG}_b0.err
SG_SPLIT_ATOMIC=1 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/${TAG}_b1.json 2> gpurun_out/${TAG}_b1.err
tail -n 2 gpurun_out/${TAG}_t1.log
for f in gpurun_out/${TAG}_b0.json gpurun_out/${TAG}_b1.json; do python -c "import json,sys; d=json.load(open('$f')); print(d['ms_per_step'], {k: d['stage_ms'][k] for k in ('hist2','scatter2','fine2','local2','scatter1','fine1')})"; done
