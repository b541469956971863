#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py tests/test_gpu_route.py tests/test_gpu_mixed.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
timeout 1500 python bench.py --config c5 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5.log 2>&1
