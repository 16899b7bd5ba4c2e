#!/bin/bash
# Call 7: parity (element-wise, multi-rank) + bench lines of gos2m, hub2m,
# pacific640m with 18-bit plans.
set -u
TAG=${1:-ab7}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_multirank_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
tail -n 2 gpurun_out/${TAG}_t1.log
for v in "g:gos2m:" "h:hub2m:" "p:pacific640m:SG_ALLOC_LOG=1"; do
  IFS=: read name cfg envs <<< "$v"
  env $envs timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_b_$name.json 2> gpurun_out/${TAG}_b_$name.err
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
grep "sg alloc" gpurun_out/${TAG}_b_p.err | tail -2
