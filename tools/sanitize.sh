#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on the tiny config (both
# grouping designs); summaries in gpurun_out/.
set -u
TAG=${1:-san}
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  for v in v1 v3; do
    timeout 1200 $CS --tool $tool --print-limit 20 python tools/sanitize_run.py $v > gpurun_out/${TAG}_${tool}_${v}.log 2>&1
    echo "$tool $v rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/${TAG}_${tool}_${v}.log | tail -1)"
  done
done
