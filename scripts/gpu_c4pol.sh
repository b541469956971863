#!/bin/bash
mkdir -p gpurun_out
for p in 5 3 0 1 2 4; do CUART_POLICY=$p timeout 900 python bench.py --config c4 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_c4_p$p.log 2>&1; done
