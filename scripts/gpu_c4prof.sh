#!/bin/bash
# new parity test (misaligned queries), c4 ncu --set full of the direct walk and of the global-form bucketed walk
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "misaligned or prebucket" > gpurun_out/pytest_mis.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_mis.log
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:'k_lookup' -c 1 \
  -o gpurun_out/c4_direct_full python bench.py --config c4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/prof_c4.log 2>&1
CUART_PREBUCKET=1 timeout 1500 ncu --set full --clock-control none --import-source on -k regex:'k_lookup' -c 1 \
  -o gpurun_out/c4_bucketed_full python bench.py --config c4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/prof_c4b.log 2>&1
