#!/bin/bash
# quick iteration: GPU tests + variant sweep
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/sweep.py --config c3 --formats ${FORMATS:-1,2,3} --policies ${POLICIES:-0,1} > gpurun_out/sweep_c3.json 2> gpurun_out/sweep_c3.err
timeout 600 python tools/sweep.py --config c2 --formats ${FORMATS:-1,2,3} --policies 1 > gpurun_out/sweep_c2.json 2> gpurun_out/sweep_c2.err
