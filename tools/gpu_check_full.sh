#!/bin/bash
# Checkpoint call: the whole GPU suite (incl. the 640M digest test), smoke,
# and a default gos2m bench line.
set -u
TAG=${1:-cf}
mkdir -p gpurun_out
SG_FULLSIZE_640M=1 timeout 3000 python -m pytest tests -m gpu -q -rA --durations=15 > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -n 3 gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -n 2 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - "$TAG" <<'PY'
import json, sys
t = sys.argv[1]
try:
    d = json.load(open(f"gpurun_out/{t}_bench.json"))
    print("bench", d["ms_per_step"], d["value"], d["e2e"], d["roofline"]["frac"], d.get("clocks"))
except Exception as e:
    print("bench failed", e, open(f"gpurun_out/{t}_bench.err").read()[-2000:])
PY
