set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_nccl_gpu.py -x -q > gpurun_out/t1.log 2>&1; echo "rc=$?" >> gpurun_out/t1.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b1.json 2> gpurun_out/b1.err
SG_GROUP_V1=1 timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --no-phase3 > gpurun_out/b1_v1.json 2> gpurun_out/b1_v1.err
timeout 1200 python -m pytest tests/test_fullsize_gpu.py tests/test_multirank_gpu.py -x -q > gpurun_out/t2.log 2>&1; echo "rc=$?" >> gpurun_out/t2.log
tail -3 gpurun_out/t1.log gpurun_out/t2.log
