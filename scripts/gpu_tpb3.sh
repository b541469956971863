#!/bin/bash
mkdir -p gpurun_out
timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
CUART_ILP=4 timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_ilp4.log 2>&1
CUART_UPD2_TPB=64 timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_u64.log 2>&1
CUART_ILP=4 timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_ilp4.log 2>&1
timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
