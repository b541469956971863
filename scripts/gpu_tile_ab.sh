#!/bin/bash
# tile walk leaf-load policy A/B on c3, c2 launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_' -c 3 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_lp3
run c3_lp2 CUART_WQ_LEAFPOL=2
run c3_lp1 CUART_WQ_LEAFPOL=1
CFG=c2 run c2_tile
