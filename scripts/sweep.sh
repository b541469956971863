#!/bin/bash
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/kgather tools/kgather.cu
/tmp/kgather 8 1024 p > gpurun_out/kgather_pair.json 2>&1
/tmp/kgather 8 1024 f > gpurun_out/kgather_footprint.json 2>&1
python tools/sweep.py --config c3 > gpurun_out/sweep_c3.json 2> gpurun_out/sweep_c3.err
python tools/sweep.py --config c2 --policies 0,1,3 > gpurun_out/sweep_c2.json 2> gpurun_out/sweep_c2.err
