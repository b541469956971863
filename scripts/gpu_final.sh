#!/bin/bash
# head check: new gather-alignment parity test, smoke, default bench line
mkdir -p gpurun_out
timeout 600 python -m pytest -m gpu -q -p no:cacheprovider tests/test_gpu_parity.py -k "misaligned or prebucket" > gpurun_out/pytest_final.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_final.log
timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_final.log
