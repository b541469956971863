#!/bin/bash
# tile sort CTA shape: 256 x 16 keys vs 512 x 8 (2 CTAs/SM, 47 registers; 3 CTAs/SM, 40 + spill): parity + c3 launch lists
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
CUART_TSORT_TPB=512 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket or misaligned" > gpurun_out/pytest_tile.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tile.log
run() { # name env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --config ${CFG:-c3} --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_$name.log 2>&1
  env "$@" timeout 600 ncu --metrics $M --clock-control none -k regex:'k_tsort' -c 1 --csv --log-file gpurun_out/ll_$name.csv python bench.py --config ${CFG:-c3} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
}
run c3_t256
run c3_t512 CUART_TSORT_TPB=512
CFG=c2 run c2_t512 CUART_TSORT_TPB=512
CUART_DEFS="-DCUART_TSORT512_MINB=3" python -c "from paper_conf_icpp_koppehelggp21_b200.build import build; build(force=True)" > gpurun_out/build_mb3.log 2>&1
run c3_t512mb3 CUART_TSORT_TPB=512
