#!/bin/bash
# A/B call 3: parity with the windowed pass-II kernel (default), bench lines
# for the pass-II kernel and the split ranking modes.
set -u
TAG=${1:-ab3}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
tail -n 2 gpurun_out/${TAG}_t1.log
for v in "base:" "tile16:SG_MH_TILE16=1" "coarse2:SG_SPLIT_COARSE=2" "coarse3:SG_SPLIT_COARSE=3" "fine2:SG_SPLIT_FINE=2" "fine3:SG_SPLIT_FINE=3" ${EXTRA_AB:-}; do
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
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_b_full.json 2> gpurun_out/${TAG}_b_full.err
python - "$TAG" <<'PY'
import json, sys
t = sys.argv[1]
try:
    d = json.load(open(f"gpurun_out/{t}_b_full.json"))
    print("full", d["ms_per_step"], d["e2e"]["ms_per_step"], d["phase3"]["ms"])
except Exception as e:
    print("full bench failed", e, open(f"gpurun_out/{t}_b_full.err").read()[-1500:])
PY
