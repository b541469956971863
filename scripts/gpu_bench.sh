#!/bin/bash
# default bench line (e2e + CPU baseline incl. the f3 layout engine) and the reference arm
mkdir -p gpurun_out
timeout 1200 python bench.py > gpurun_out/bench_c3.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_c3.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.log 2>&1
