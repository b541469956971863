#!/bin/bash
# bench lines for c2 / c4 / c5 (N=1 and the P=8 per-GPU share) and their ncu launch lists
# (per-kernel time + DRAM bytes + L2 sectors), the l2_persist variant of c3, the l2 test
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -k l2_persist -m gpu -q -p no:cacheprovider > gpurun_out/pytest_l2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_l2.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_hit_rate.pct
for c in c2 c4; do
  timeout 900 python bench.py --config $c --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$c.log
  timeout 900 ncu --metrics $M --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$c.log 2>&1
done
timeout 900 python bench.py --config c5 --c5-share 8 --steps 5 --warmup 3 > gpurun_out/bench_c5_share8.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c5_share8.log
timeout 1200 ncu --metrics $M --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c5_share8.csv python bench.py --config c5 --c5-share 8 --steps 1 --warmup 1 > gpurun_out/ncu_c5_share8.log 2>&1
timeout 1500 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/bench_c5.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c5.log
timeout 900 python bench.py --no-e2e --no-cpu-baseline --l2-persist 1 > gpurun_out/bench_c3_l2.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c3_l2.log
