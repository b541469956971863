#!/bin/bash
# tile walk with the next round's keys prefetched to L2 (CUART_WT_PF): parity under it, c3/c2/c4 bench + launch lists
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
CUART_WT_PF=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket or misaligned" > gpurun_out/pytest_pf.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_pf.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_pf0
run c3_pf1 CUART_WT_PF=1
CFG=c2 run c2_pf0
CFG=c2 run c2_pf1 CUART_WT_PF=1
CFG=c4 run c4_pf0 CUART_PREBUCKET=1
CFG=c4 run c4_pf1 CUART_PREBUCKET=1 CUART_WT_PF=1
