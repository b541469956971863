#!/bin/bash
# direct walk with two queries per thread (k_lookup2) vs one (k_lookup): c4, the c5 share, parity tests
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
  CUART_DIRECT_ILP=$i timeout 900 python bench.py --config c4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_c4_ilp$i.log 2>&1
  CUART_DIRECT_ILP=$i timeout 900 python bench.py --config c5 --c5-share 8 --steps 5 --warmup 3 > gpurun_out/bench_c5s8_ilp$i.log 2>&1
done
CUART_DIRECT_ILP=2 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_ilp2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ilp2.log
