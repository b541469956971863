#!/bin/bash
# k_bgather: position pairs per thread (4-B jpos loads, 16-B result stores)
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_iter8.log 2>&1
timeout 600 python bench.py --config c2 --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_iter8.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3_iter8.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_iter8.log 2>&1
timeout 1200 python -m pytest -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_route.py tests/test_gpu_mixed.py > gpurun_out/pytest_iter8.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter8.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_iter8.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_iter8.log
