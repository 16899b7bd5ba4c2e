#!/bin/bash
# A/B of the warp-tier placement (SG_LOCAL_ATOMIC) + the fused-exchange tests.
set -u
TAG=${1:-ab}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_multirank_gpu.py tests/test_nccl_gpu.py -x -q > gpurun_out/${TAG}_xch.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_xch.log
tail -n 3 gpurun_out/${TAG}_xch.log
SG_LOCAL_ATOMIC=1 timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1a.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1a.log
tail -n 3 gpurun_out/${TAG}_t1a.log
for v in 0 1; do
  SG_LOCAL_ATOMIC=$v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_b$v.json 2> gpurun_out/${TAG}_b$v.err
  python - "$TAG" "$v" <<'PY'
import json, sys
t, v = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/{t}_b{v}.json"))
    print("atomic", v, d["ms_per_step"], {k: x for k, x in d["stage_ms"].items() if x > 5})
except Exception as e:
    print("bench failed", e, open(f"gpurun_out/{t}_b{v}.err").read()[-1500:])
PY
done
