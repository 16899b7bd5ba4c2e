#!/bin/bash
# Call 9: incremental cache release (pacific640m), gos2m check.
set -u
TAG=${1:-ab9}
mkdir -p gpurun_out
for v in "g:gos2m:SG_ALLOC_LOG=1" "p:pacific640m:SG_ALLOC_LOG=1"; do
  IFS=: read name cfg envs <<< "$v"
  env $envs SG_BENCH_CACHE=1 timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_b_$name.json 2> gpurun_out/${TAG}_b_$name.err
  python - "$TAG" "$name" <<'PY'
import json, sys
t, v = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/{t}_b_{v}.json"))
    print(v, d["ms_per_step"], {k: x for k, x in d["stage_ms"].items() if x > 5})
except Exception as e:
    print(v, "bench failed", e, open(f"gpurun_out/{t}_b_{v}.err").read()[-1500:])
PY
  grep "sg alloc" gpurun_out/${TAG}_b_$name.err | tail -2
done
