#!/bin/bash
set -u
TAG=${1:-c3}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_nccl_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/${TAG}_launches_hub2m_p1.csv python tools/profile_run.py --config hub2m --pass1-only --reps 1 \
  > gpurun_out/${TAG}_launches_hub2m_p1.log 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --print-limit 20 python tools/sanitize_run.py > gpurun_out/${TAG}_san_${tool}.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/${TAG}_san_${tool}.log
done
tail -n 2 gpurun_out/${TAG}_t1.log; grep -h "SUMMARY" gpurun_out/${TAG}_san_*.log
