#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py -k "skew or prebucket" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for m in 1 32; do for c in c3 c2; do CUART_WQ_MINB=$m timeout 600 python bench.py --config $c --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_m$m.log 2>&1; done; done
