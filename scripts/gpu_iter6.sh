#!/bin/bash
# k_lookup_wq launch shape sweep: threads per CTA (32/64/128) x queries per thread (2/3) on c3 and c2
mkdir -p gpurun_out
for cfg in "64 2" "32 2" "64 3" "32 3" "128 3"; do set -- $cfg
  for c in c3 c2; do
    echo "tpb=$1 ilp=$2 $c $(CUART_WQ_TPB=$1 CUART_ILP=$2 timeout 600 python bench.py --config $c --steps 10 --no-e2e --no-cpu-baseline 2>&1 | grep '^{' | tail -1)" >> gpurun_out/wq_sweep.log
  done
done
CUART_WQ_TPB=32 CUART_ILP=3 timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider tests/test_gpu_parity.py > gpurun_out/pytest_iter6.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter6.log
