#!/bin/bash
# One GPU call: parity tests, bench lines (default path and an A/B variant),
# then the full-size and multi-rank tests.  Results in gpurun_out/.
set -u
TAG=${1:-chk}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_nccl_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
timeout 1200 python -m pytest tests/test_fullsize_gpu.py tests/test_multirank_gpu.py -x -q > gpurun_out/${TAG}_t2.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t2.log
tail -n 3 gpurun_out/${TAG}_t1.log gpurun_out/${TAG}_t2.log
