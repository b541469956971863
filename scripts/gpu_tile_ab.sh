#!/bin/bash
# tile walk leaf-load cache policy (CUART_WQ_LEAFPOL: 0 evict_first+L2::64B, 1 evict_last+L2::64B, 2 plain, 3 evict_last)
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
for lp in 3 0 1 2; do
  CUART_WQ_LEAFPOL=$lp timeout 600 python bench.py --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_lp$lp.log 2>&1
  CUART_WQ_LEAFPOL=$lp timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_lp$lp.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
