#!/bin/bash
# k_bscatter with per-position destination slots staged in smem: parity + c3/c2 bench + launch list
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py tests/test_gpu_route.py > gpurun_out/pytest_gpu_iter5.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_iter5.log
timeout 600 python bench.py --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_iter5.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_iter5.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3_iter5.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_iter5.log 2>&1
