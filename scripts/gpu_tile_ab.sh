#!/bin/bash
# tile walk with up to 64 tiles per CTA: parity (prebucket tests), c3 / c2 bench at 32 / 48 / 64 tiles + launch lists
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket or misaligned" > gpurun_out/pytest_tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_tg32
run c3_tg48 CUART_TILE_GROUP=48
run c3_tg64 CUART_TILE_GROUP=64
CFG=c2 run c2_tg32
CFG=c2 run c2_tg64 CUART_TILE_GROUP=64
