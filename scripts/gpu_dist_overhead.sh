#!/bin/bash
# the multi-GPU layer at one rank: its protocol overhead on c3 (plain path vs --dist p2p vs --dist nccl)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_plain.log 2>&1
for t in p2p nccl; do
  timeout 900 python bench.py --dist --transport $t --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_dist_$t.log 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_dist_p2p.csv python bench.py --dist --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
