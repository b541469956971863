#!/bin/bash
# register caps (min CTAs/SM) of k_bscatter / k_bhist: per-kernel times from ncu launch lists on c3
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in "base:" "s5:-DCUART_SCATTER_MIN_BLOCKS=5" "h5:-DCUART_HIST_MIN_BLOCKS=5" "h6:-DCUART_HIST_MIN_BLOCKS=6"; do
  name=${v%%:*}; defs=${v#*:}
  CUART_DEFS="$defs" python -c "from paper_conf_icpp_koppehelggp21_b200.build import build; build(force=True)" > gpurun_out/build_$name.log 2>&1
  timeout 900 ncu --metrics $M --clock-control none -k regex:'k_b' --csv --log-file gpurun_out/launches_mb_$name.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
python -c "from paper_conf_icpp_koppehelggp21_b200.build import build; build(force=True)" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_c3_mb.log 2>&1
