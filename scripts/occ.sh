#!/bin/bash
mkdir -p gpurun_out
for c in 32 512 2048 -1 0; do
  if [ $c = 0 ]; then unset CUART_GRID_CTAS_PER_SM; else export CUART_GRID_CTAS_PER_SM=$c; fi
  echo "ctas_per_sm=$c"
  timeout 300 python tools/sweep.py --config c3 --formats 1,2,3 --policies 1 --reps 3
done > gpurun_out/occ.json 2> gpurun_out/occ.err
