#!/bin/bash
# stable partition / unroute (c5's mixed rounds): route + mixed + dist tests, c5 (N=1 and the P=8 share) bench + launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 1500 python -m pytest tests/test_gpu_route.py tests/test_gpu_mixed.py tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_c5.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_c5.log
timeout 1500 python bench.py --config c5 --no-e2e --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c5.log 2>&1
timeout 900 python bench.py --config c5 --c5-share 8 --no-e2e --no-cpu-baseline > gpurun_out/bench_c5_share8.log 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:'k_pf|k_unroute' --csv --log-file gpurun_out/launches_c5_share8_pf.csv python bench.py --config c5 --c5-share 8 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
