#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1
for t in 256 128 64; do
  CUART_LOOKUP_TPB=$t timeout 600 python bench.py --config c4 --steps 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_t$t.log 2>&1
  CUART_PREBUCKET=0 CUART_LOOKUP_TPB=$t timeout 600 python bench.py --steps 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3d_t$t.log 2>&1
done
