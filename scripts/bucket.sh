#!/bin/bash
mkdir -p gpurun_out
for pb in 0 1; do
  export CUART_PREBUCKET=$pb
  echo "prebucket=$pb"
  timeout 600 python tools/sweep.py --config c3 --formats 3 --policies 5 --reps 5
  timeout 600 python tools/sweep.py --config c2 --formats 3 --policies 5 --reps 5
done > gpurun_out/bucket.json 2> gpurun_out/bucket.err
export CUART_PREBUCKET=1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_b|k_lookup" --csv --log-file gpurun_out/bucket_ncu.csv python tools/profile_variants.py > /dev/null 2>&1
