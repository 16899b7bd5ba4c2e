#!/bin/bash
set -u
TAG=${1:-c8}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_multirank_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
timeout 2400 python -m pytest tests/test_fullsize_digests_gpu.py tests/test_fullsize_gpu.py -x -q -k "c400 or s5c50 or fullsize_digests_every" > gpurun_out/${TAG}_t2.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t2.log
tail -n 2 gpurun_out/${TAG}_t1.log gpurun_out/${TAG}_t2.log
