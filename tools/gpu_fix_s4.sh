#!/bin/bash
# Re-measure after reverting the largest-first cache release: pacific640m
# (as in the final script), the sweep, and the Phase III L2-persistence A/B
# on gos2m (report inside the e2e leg).
set -u
TAG=${1:-fx}
mkdir -p gpurun_out
SG_ALLOC_LOG=1 SG_BENCH_CACHE=1 python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_pacific640m.json 2> gpurun_out/${TAG}_bench_pacific640m.err
python -c "import json; d=json.load(open('gpurun_out/${TAG}_bench_pacific640m.json')); print('pacific', d['ms_per_step'], d['e2e']['ms_per_step'], {k: v for k, v in d['stage_ms'].items() if v > 50})"
grep "sg alloc" gpurun_out/${TAG}_bench_pacific640m.err | tail -3
for v in "l2:" "nol2:SG_NO_L2_PERSIST=1"; do
  IFS=: read name envs <<< "$v"
  env $envs timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_b_$name.json 2> gpurun_out/${TAG}_b_$name.err
  python -c "import json; d=json.load(open('gpurun_out/${TAG}_b_$name.json')); print('$name', d['ms_per_step'], d['e2e']['ms_per_step'], d['phase3']['ms'])"
done
timeout 1500 python tools/sweep.py --steps 3 --warmup 1 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
python -c "
import json
for l in open('gpurun_out/${TAG}_sweep.jsonl'):
    d = json.loads(l); print(d.get('s'), d.get('c'), d.get('ms_per_step'))"
