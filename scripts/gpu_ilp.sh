#!/bin/bash
# A/B of the wide walk's queries per thread (CUART_ILP) on c3 / c2, plus the parity tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_delete.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in c3 c2; do for q in 1 2 4; do
  CUART_ILP=$q timeout 900 python bench.py --config $c --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_ilp$q.log 2>&1
done; done
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -I paper_conf_icpp_koppehelggp21_b200/csrc tools/bucket_micro.cu -o /tmp/bm && timeout 300 /tmp/bm > gpurun_out/bucket_micro.json 2>&1
