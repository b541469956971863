#!/bin/bash
# tests touching the walk/update kernels, c3 bench, launch list + ncu --set full of the bucketed walk and stage 1
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py tests/test_gpu_mixed.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
CUART_ILP=1 timeout 900 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_ilp1.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:'k_lookup_wq|k_upd1_wq' -c 2 -o gpurun_out/c3_wq_full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
