#!/bin/bash
# byte-string tile form variants (1k-thread sort, walk shapes): parity under the variants, c4 bench + launch lists
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
CUART_TSORT_B1K=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket or misaligned" > gpurun_out/pytest_c4tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_c4tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config c4 --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_' -c 3 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config c4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c4_b1k CUART_PREBUCKET=1 CUART_TSORT_B1K=1
run c4_b1k_m6 CUART_PREBUCKET=1 CUART_TSORT_B1K=1 CUART_WT_MINB=6
run c4_b1k_t128 CUART_PREBUCKET=1 CUART_TSORT_B1K=1 CUART_WT_TPB=128
run c4_b1k_s0 CUART_PREBUCKET=1 CUART_TSORT_B1K=1 CUART_BUCKET_SHIFT=0
