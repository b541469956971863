#!/bin/bash
mkdir -p gpurun_out
for c in c2 c4; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
CUART_PREBUCKET=0 timeout 900 python bench.py --config c4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c4_direct.log 2>&1
timeout 1200 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/bench_c5.log 2>&1
