#!/bin/bash
# ncu --set full of the K-BUCKET streaming kernels (one launch each) on c3
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:'k_bhist|k_bscatter|k_bgather' -c 4 \
  -o gpurun_out/bucket_full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/prof_bucket.log 2>&1
echo "ncu rc=$?" >> gpurun_out/prof_bucket.log
