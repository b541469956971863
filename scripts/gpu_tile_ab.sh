#!/bin/bash
# wide walk's inline N4 step with evict_last (build-time CUART_WQ_NODEKEEP=1) vs default: c3 bench + launch list
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 600 python bench.py --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_nk0.log 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_nk0.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
CUART_DEFS="-DCUART_WQ_NODEKEEP=1" python -c "from paper_conf_icpp_koppehelggp21_b200.build import build; build(force=True)" > gpurun_out/build_nk.log 2>&1
timeout 600 python bench.py --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/ab_nk1.log 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:'k_lookup_wt' -c 1 --csv --log-file gpurun_out/ll_nk1.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "prebucket" > gpurun_out/pytest_nk.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_nk.log
