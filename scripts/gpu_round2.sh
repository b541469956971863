#!/bin/bash
# c4 pre-bucketed vs direct, c5 (N=1 and the P=8 share) with the budget-sized dist chunks, full GPU suite
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CUART_PREBUCKET=1 timeout 900 python bench.py --config c4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_c4_bucketed.log 2>&1
timeout 900 python bench.py --config c5 --c5-share 8 --steps 5 --warmup 3 > gpurun_out/bench_c5_share8.log 2>&1
timeout 1500 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/bench_c5.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 1200 --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
