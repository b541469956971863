#!/bin/bash
# e2e (host-buffer pipeline) experiments: PCIe probe, host-path tests, c3 e2e at two chunk sizes
mkdir -p gpurun_out
timeout 300 python tools/pcie_probe.py > gpurun_out/pcie_probe.json 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "host" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for ch in 8388608 33554432; do
  CUART_STAGE_CHUNK=$ch timeout 900 python bench.py --steps 3 --no-cpu-baseline --e2e-steps 3 > gpurun_out/bench_c3_chunk$ch.log 2>&1
done
