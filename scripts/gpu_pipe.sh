#!/bin/bash
mkdir -p gpurun_out
for c in 1 2 4 8; do
  CUART_PIPE=$c timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/pipe_$c.log 2>&1
done
CUART_PIPE=4 CUART_GRID_CTAS_PER_SM=4 timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/pipe_4_g4.log 2>&1
CUART_PIPE=4 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "c3_full" > gpurun_out/pipe_test.log 2>&1
