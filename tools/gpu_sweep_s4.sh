#!/bin/bash
set -u
TAG=${1:-sw}
mkdir -p gpurun_out
timeout 2400 python tools/sweep.py --steps 3 --warmup 2 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
python -c "
import json
for l in open('gpurun_out/${TAG}_sweep.jsonl'):
    d = json.loads(l); print(d.get('s'), d.get('c'), d.get('ms_per_step'), d.get('error', ''))"
