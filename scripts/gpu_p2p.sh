#!/bin/bash
# fused p2p exchange: loopback kernels, 2-process IPC protocol, multi-rank bench smoke
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_route.py tests/test_gpu_dist_procs.py -m gpu -q -p no:cacheprovider -x > gpurun_out/pytest_p2p.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_p2p.log
for t in p2p nccl; do
CUART_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 2 --warmup 1 --config c1 --transport $t --no-e2e > gpurun_out/bench2_$t.log 2>&1; echo "rc=$?" >> gpurun_out/bench2_$t.log
done
