#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none -k regex:'k_lookup' --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
