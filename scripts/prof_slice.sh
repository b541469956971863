#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'k_lookup' -c 1 -o gpurun_out/slice_c3 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/prof_slice.log 2>&1
CUART_SLICE=1 timeout 900 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_noslice.log 2>&1
