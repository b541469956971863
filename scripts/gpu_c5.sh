#!/bin/bash
# c3 default bench (regression check), c5 at N=1 and the P=8 per-GPU share, c5 full-size parity test
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c3.log
timeout 1200 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/bench_c5.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c5.log
timeout 900 python bench.py --config c5 --c5-share 8 --steps 5 --warmup 3 > gpurun_out/bench_c5_share8.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c5_share8.log
timeout 1500 python -m pytest tests/test_gpu_mixed.py -m gpu -q -x -p no:cacheprovider --durations=5 > gpurun_out/pytest_c5.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_c5.log
