#!/bin/bash
# Iteration call: element-wise parity suite, a short gos2m bench line, and
# (NCU=1) an ncu --set full capture of the level-II grouping kernels
# (gos2m, c2 = 64: one trial chunk).  Results in gpurun_out/<TAG>_*.
set -u
TAG=${1:-it}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
tail -n 3 gpurun_out/${TAG}_t1.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 ${BENCH_ARGS:-} > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
python - "$TAG" <<'PY'
import json, sys
t = sys.argv[1]
try:
    d = json.load(open(f"gpurun_out/{t}_b.json"))
    print("bench", d["ms_per_step"], d["value"], d.get("clocks"))
    print({k: v for k, v in d["stage_ms"].items() if v > 1})
except Exception as e:
    print("bench failed", e, open(f"gpurun_out/{t}_b.err").read()[-2000:])
PY
if [ "${NCU:-0}" = "1" ]; then
  timeout 1500 ncu --set full --import-source on --clock-control none \
    -k regex:"${NCU_K:-scatter_kernel|scatter2_kernel|warp_local_kernel}" --launch-skip ${NCU_SKIP:-3} -c ${NCU_C:-3} \
    -o gpurun_out/${TAG}_full python tools/profile_run.py --config gos2m --c2 64 --reps 1 \
    > gpurun_out/${TAG}_full.log 2>&1
  echo "ncu rc=$?"
fi
