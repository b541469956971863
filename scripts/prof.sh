#!/bin/bash
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/kg3 tools/kgather3.cu && /tmp/kg3 > gpurun_out/kgather3.json 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,lts__t_requests_srcunit_tex_op_read.sum,smsp__inst_executed.sum
ncu --metrics $M --clock-control none -k regex:k_lookup --csv --log-file gpurun_out/prof_variants.csv python tools/profile_variants.py > gpurun_out/prof_variants.log 2>&1
