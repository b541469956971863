#!/bin/bash
# byte-string direct walk capped at 8 CTAs/SM (32 registers) with the skip table: parity + c4 bench + launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 900 python -m pytest tests/test_gpu_skip.py tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "skip or bytes or string or c4" > gpurun_out/pytest_skip.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_skip.log
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4.log 2>&1
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline --skip-log2 26 > gpurun_out/bench_c4_skip26.log 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:'k_lookup' -c 1 --csv --log-file gpurun_out/launches_c4_skip.csv python bench.py --config c4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
