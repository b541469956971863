#!/bin/bash
# full round check at HEAD: GPU test suite, smoke, the default bench line (e2e + CPU baseline),
# the reference arm, and the c3 ncu launch list + ncu --set full of the step's kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2700 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python bench.py > gpurun_out/bench_c3.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_c3.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:'k_' --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:'k_tsort|k_lookup_wt|k_tgather|k_bscatter|k_upd1_wq|k_upd2|k_bhist' -c 7 -o gpurun_out/c3_full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
for c in c2 c4; do timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 1500 python bench.py --config c5 --no-e2e --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c5.log 2>&1
timeout 900 python bench.py --config c5 --c5-share 8 --no-e2e --no-cpu-baseline > gpurun_out/bench_c5_share8.log 2>&1
timeout 900 python bench.py --dist --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_dist1.log 2>&1
