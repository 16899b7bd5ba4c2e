#!/bin/bash
# A/B call 4: windowed pass-II kernel (length-specific pads, 16-trial passes,
# split long rows) vs the tile kernel; parity of both.
set -u
TAG=${1:-ab4}
mkdir -p gpurun_out
SG_MH_WIN=1 timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1w.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1w.log
tail -n 2 gpurun_out/${TAG}_t1w.log
for v in "tile:" "win:SG_MH_WIN=1"; do
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
SG_MH_WIN=1 timeout 900 ncu --set full --import-source on --clock-control none -k regex:"minhash_win" -c 1 \
  -o gpurun_out/${TAG}_win python tools/profile_run.py --config gos2m --c2 64 --reps 1 > gpurun_out/${TAG}_win.log 2>&1
echo "ncu rc=$?"
