#!/bin/bash
# k_bscatter phase 3 fully unrolled (256 x 4 launch bounds) + c5 bench line with its roofline fields
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_iter7.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3_iter7.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_iter7.log 2>&1
timeout 1500 python bench.py --config c5 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_iter7.log 2>&1
timeout 1200 python -m pytest -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_mixed.py > gpurun_out/pytest_iter7.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter7.log
