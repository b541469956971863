#!/bin/bash
# bench.py's multi-GPU launch shape smoke-tested with 2 ranks sharing one GPU: torchrun,
# host bootstrap over gloo (NCCL refuses two ranks on one device), transport p2p (CUDA IPC
# windows between the two processes).  The numbers measure GPU sharing, not scaling.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
# replica mode with c1 (two full c3 replicas plus their windows and batches do not fit one GPU)
for mc in "range c3" "replica c1"; do
  set -- $mc
  CUART_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 \
    bench.py --gpus 2 --steps 3 --warmup 3 --mode $1 --config $2 --transport p2p --no-e2e > gpurun_out/bench_2rank_$1.log 2>&1
  echo "rc=$?" >> gpurun_out/bench_2rank_$1.log
done
CUART_DIST_BACKEND=gloo timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --config c5 --c5-share 0 --steps 2 --warmup 2 > gpurun_out/bench_2rank_c5.log 2>&1
echo "rc=$?" >> gpurun_out/bench_2rank_c5.log
