#!/bin/bash
mkdir -p gpurun_out
for lp in 0 1 2 3; do
  CUART_WQ_LEAFPOL=$lp timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_lp$lp.log 2>&1
  CUART_WQ_LEAFPOL=$lp timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_lp$lp.log 2>&1
done
