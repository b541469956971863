#!/bin/bash
mkdir -p gpurun_out
for f in rank compact32 links; do
  for c in c3 c2; do
    timeout 600 python bench.py --config $c --lut-format $f --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/lutfmt_${c}_$f.log 2>&1
  done
done
