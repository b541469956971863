#!/bin/bash
# c4 bench lines with the skip-aware sector model (default cap and D = 16)
mkdir -p gpurun_out
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4.log 2>&1
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline --skip-log2 26 > gpurun_out/bench_c4_skip26.log 2>&1
