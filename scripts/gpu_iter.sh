#!/bin/bash
# iteration call: targeted GPU tests, then c3 / c2 / c4 bench lines (kernel-only), optional wide-table A/B
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider ${TESTS:-tests/test_gpu_parity.py tests/test_gpu_delete.py} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in ${CFGS:-c3 c2 c4}; do
  timeout 900 python bench.py --config $c --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
if [ -n "$AB" ]; then
  for w in 1 2; do CUART_WIDE=$w timeout 900 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_wide$w.log 2>&1; done
fi
if [ -n "$LAUNCH" ]; then
  for c in ${CFGS:-c3 c2 c4}; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_$c.log 2>&1
  done
fi
