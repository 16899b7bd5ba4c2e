#!/bin/bash
set -u
TAG=${1:-pl2}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
tail -n 2 gpurun_out/${TAG}_t1.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
python -c "import json; d=json.load(open('gpurun_out/${TAG}_b.json')); print('gos2m', d['ms_per_step'], {k: v for k, v in d['stage_ms'].items() if v > 5})"
timeout 1500 python tools/sweep.py --steps 3 --warmup 2 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
python -c "
import json
for l in open('gpurun_out/${TAG}_sweep.jsonl'):
    d = json.loads(l); print(d.get('s'), d.get('c'), d.get('ms_per_step'), d.get('counts', {}).get('chunks1'), d.get('counts', {}).get('chunks2'), d.get('error', ''))"
