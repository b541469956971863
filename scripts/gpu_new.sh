#!/bin/bash
mkdir -p gpurun_out
nproc > gpurun_out/host.txt; free -g >> gpurun_out/host.txt
timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_range.py tests/test_gpu_delete.py tests/test_gpu_route.py -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_new.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new.log
timeout 1200 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_c5.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c5.log
