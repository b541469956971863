#!/bin/bash
# k_bscatter one-pass ranking/staging vs two-pass, k_bgather at 5 vs 1 min CTAs/SM: c3 bench + launch lists, parity
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_ab.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab.log
for o in 1 0; do
  CUART_SCATTER_ONEPASS=$o timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_onepass$o.log 2>&1
  CUART_SCATTER_ONEPASS=$o timeout 900 ncu --metrics $M --clock-control none -k regex:'k_b' --csv --log-file gpurun_out/launches_c3_onepass$o.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
CUART_DEFS=-DCUART_GATHER_MIN_BLOCKS=1 python -c "from paper_conf_icpp_koppehelggp21_b200.build import build; build(force=True)" > gpurun_out/build_g1.log 2>&1
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_gather1.log 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:'k_b' --csv --log-file gpurun_out/launches_c3_gather1.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
