#!/bin/bash
# K-BUCKET tile form knob sweep (profiles/r02/tile_form.txt): parity of the prebucket tests, then c3 / c2 bench lines
# and k_lookup_wt / k_tsort / k_tgather ncu launch lists for the default and each variant
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket or misaligned" > gpurun_out/pytest_tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_w|k_tsort|k_tgather' -c 3 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_def
run c3_tg16 CUART_TILE_GROUP=16
run c3_minb1 CUART_WT_MINB=1
run c3_s1 CUART_BUCKET_SHIFT=1
run c3_global CUART_BUCKET_FORM=1
CFG=c2 run c2_def
CFG=c2 run c2_global CUART_BUCKET_FORM=1
