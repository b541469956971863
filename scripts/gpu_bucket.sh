#!/bin/bash
# K-BUCKET iteration: bucket parity tests, c3/c2 bench, launch list
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "prebucket or c3_full or c2_full" > gpurun_out/pytest_bucket.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_bucket.log
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_c3.log
timeout 900 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
