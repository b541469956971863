#!/bin/bash
mkdir -p gpurun_out
export CUART_PREBUCKET=1
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_delete.py tests/test_gpu_range.py -m gpu -q -x -p no:cacheprovider \
    -k "golden or edge or reserved or hand_pins or single_key or range_with_deletes or prebucket_equals_direct or prebucket_updates_equal_direct or bucketed_wide_walk or full_n256 or many_chunks" > gpurun_out/sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_$tool.log
done
