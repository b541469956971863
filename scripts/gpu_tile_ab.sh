#!/bin/bash
# tile walk register cap: 20 CTAs/SM (48 registers) vs 24 (40 registers + 24 B spill), c3 bench + launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_m20
run c3_m24 CUART_WT_MINB=24
