#!/bin/bash
# the fused mixed round (cuart_dist_mixed): dist GPU tests, c5 lines fused vs unfused, 2-rank replica smoke (c1)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_dist.py tests/test_gpu_mixed.py tests/test_gpu_dist_procs.py -m gpu -q -p no:cacheprovider --timeout 900 -k "not full_size" > gpurun_out/pytest_mixed.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_mixed.log
for f in 1 0; do
  timeout 900 python bench.py --config c5 --c5-share 8 --c5-fused $f --steps 5 --warmup 3 > gpurun_out/bench_c5_share8_f$f.log 2>&1
done
timeout 1500 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/bench_c5_f1.log 2>&1
CUART_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 \
    bench.py --gpus 2 --config c1 --steps 3 --warmup 3 --mode replica --transport p2p --no-e2e > gpurun_out/bench_2rank_replica_c1.log 2>&1
echo "rc=$?" >> gpurun_out/bench_2rank_replica_c1.log
timeout 1800 python -m pytest tests/test_gpu_mixed.py -m gpu -q -p no:cacheprovider -k full_size > gpurun_out/pytest_c5full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_c5full.log
