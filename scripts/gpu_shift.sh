#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for sh in 0 1 2 3 4; do
  CUART_BUCKET_SHIFT=$sh timeout 600 python bench.py --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_s$sh.log 2>&1
done
for sh in 0 2; do CUART_BUCKET_SHIFT=$sh timeout 600 python bench.py --config c2 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_c2_s$sh.log 2>&1; done
CUART_BUCKET_SHIFT=2 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3_s2.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
