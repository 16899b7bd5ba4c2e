#!/bin/bash
# A/B call: atomic-order probe, parity (default / SG_SPLIT_ATOMIC=1), fused
# exchange tests, bench lines for the variants.
set -u
TAG=${1:-ab2}
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/atom_order tools/atom_order.cu && timeout 120 /tmp/atom_order > gpurun_out/${TAG}_atom_order.jsonl 2>&1
cat gpurun_out/${TAG}_atom_order.jsonl
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
tail -n 2 gpurun_out/${TAG}_t1.log
SG_SPLIT_ATOMIC=1 timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1s.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1s.log
tail -n 2 gpurun_out/${TAG}_t1s.log
timeout 900 python -m pytest tests/test_multirank_gpu.py tests/test_nccl_gpu.py -x -q > gpurun_out/${TAG}_xch.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_xch.log
tail -n 2 gpurun_out/${TAG}_xch.log
for v in "base:" "splitat:SG_SPLIT_ATOMIC=1" "nokbin:SG_NO_KBIN=1" "matchlocal:SG_LOCAL_ATOMIC=0"; do
  name=${v%%:*}; envs=${v#*:}
  env $envs timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_b_$name.json 2> gpurun_out/${TAG}_b_$name.err
  python - "$TAG" "$name" <<'PY'
import json, sys
t, v = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/{t}_b_{v}.json"))
    print(v, d["ms_per_step"], {k: x for k, x in d["stage_ms"].items() if x > 5})
except Exception as e:
    print(v, "bench failed", e, open(f"gpurun_out/{t}_b_{v}.err").read()[-1500:])
PY
done
