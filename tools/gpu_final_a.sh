#!/bin/bash
# Final round-2 evidence, part A: the whole GPU suite and smoke.
set -u
TAG=${1:-fa}
mkdir -p gpurun_out
SG_FULLSIZE_640M=1 timeout 3300 python -m pytest tests -m gpu -q -rA --durations=30 > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -n 3 gpurun_out/${TAG}_pytest.log gpurun_out/${TAG}_smoke.log
