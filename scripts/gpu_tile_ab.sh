#!/bin/bash
# K-BUCKET tile form: parity, walk variants on c3 (bench + ncu launch list each)
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket" > gpurun_out/pytest_tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_def
run c3_m20 CUART_WT_MINB=20
run c3_s1 CUART_BUCKET_SHIFT=1
run c3_s1m20 CUART_BUCKET_SHIFT=1 CUART_WT_MINB=20
run c3_s3 CUART_BUCKET_SHIFT=3
run c3_tg16 CUART_TILE_GROUP=16
