#!/bin/bash
# 2 ranks sharing one GPU (gloo for the host-side collectives): the multi-GPU bench path end to end on c3
# (pre-bucketed walks + fused p2p exchange), range and replica; plus c4 with pre-bucketing forced on
mkdir -p gpurun_out
for t in p2p nccl; do
CUART_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 2 --warmup 3 --config c3 --transport $t --no-e2e > gpurun_out/bench2_c3_$t.log 2>&1; echo "rc=$?" >> gpurun_out/bench2_c3_$t.log
done
CUART_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 2 --warmup 3 --config c3 --mode replica --no-e2e > gpurun_out/bench2_c3_replica.log 2>&1; echo "rc=$?" >> gpurun_out/bench2_c3_replica.log
CUART_PREBUCKET=1 timeout 900 python bench.py --config c4 --steps 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_pb.log 2>&1
