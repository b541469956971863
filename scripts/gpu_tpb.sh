#!/bin/bash
mkdir -p gpurun_out
for c in c3 c2; do for t in 256 128 64; do CUART_WQ_TPB=$t timeout 600 python bench.py --config $c --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_t$t.log 2>&1; done; done
