#!/bin/bash
# The whole GPU test suite + smoke, logs in gpurun_out/.
set -u
TAG=${1:-tests}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 5400 python -m pytest tests -m gpu -q -rA --durations=25 > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -n 3 gpurun_out/${TAG}_pytest.log gpurun_out/${TAG}_smoke.log
