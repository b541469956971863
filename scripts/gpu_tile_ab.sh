#!/bin/bash
# tile form: walk CTA size, tile-sort 16-B loads; parity of the variants; c3 bench + launch list each
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active
CUART_TSORT_VEC=1 CUART_WT_TPB=128 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket" > gpurun_out/pytest_tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt|k_tsort' -c 2 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_def
run c3_tpb128 CUART_WT_TPB=128
run c3_tpb256 CUART_WT_TPB=256
run c3_vec CUART_TSORT_VEC=1
CFG=c2 run c2_vec CUART_TSORT_VEC=1
CFG=c2 run c2_def
