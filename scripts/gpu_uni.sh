#!/bin/bash
# uniform node-step walk (CUART_UNIFORM=1): parity suite under it, c4 / c3-direct / c5-share bench A/B, c4 launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active
CUART_UNIFORM=1 timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_delete.py -m gpu -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_uni.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_uni.log
for u in 0 1; do
  CUART_UNIFORM=$u timeout 600 python bench.py --config c4 --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_c4_u$u.log 2>&1
  CUART_UNIFORM=$u CUART_PREBUCKET=0 timeout 600 python bench.py --config c3 --no-e2e --no-cpu-baseline --steps 3 > gpurun_out/ab_c3d_u$u.log 2>&1
  CUART_UNIFORM=$u timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup' -c 1 --csv --log-file gpurun_out/ll_c4_u$u.csv python bench.py --config c4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
