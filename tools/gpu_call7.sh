#!/bin/bash
set -u
TAG=${1:-c7}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "tiny or sweep or small or host_csr or edge" > gpurun_out/${TAG}_t1.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_t1.log
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_gos2m.json 2> gpurun_out/${TAG}_bench_gos2m.err
SG_NO_CACHE=1 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-phase3 > gpurun_out/${TAG}_bench_gos2m_nc.json 2> gpurun_out/${TAG}_bench_gos2m_nc.err
SG_BENCH_CACHE=1 SG_NO_CACHE=1 python bench.py --config pacific640m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_bench_pac_nc.json 2> gpurun_out/${TAG}_bench_pac_nc.err
SG_BENCH_CACHE=1 SG_NO_CACHE=1 python bench.py --config hub2m --steps 3 --warmup 3 --no-cpu-baseline --no-phase3 --no-e2e > gpurun_out/${TAG}_bench_hub_nc.json 2> gpurun_out/${TAG}_bench_hub_nc.err
tail -n 2 gpurun_out/${TAG}_t1.log
