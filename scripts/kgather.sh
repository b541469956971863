#!/bin/bash
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/kgather tools/kgather.cu
/tmp/kgather 8 1024 > gpurun_out/kgather.json 2>&1
/tmp/kgather 0.0625 1024 > gpurun_out/kgather_l2.json 2>&1
ncu --metrics gpu__time_duration.sum,dram__sectors_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum --clock-control none --csv --log-file gpurun_out/kgather_ncu.csv /tmp/kgather 8 256 > gpurun_out/kgather_ncu.log 2>&1
