#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over the parity tests of the hot path,
# the bucketed variants (both K-BUCKET forms), the skip table, the two-way partition and the
# multi-GPU layer at one rank.  (Virtual ranks >= 2 in one
# process are excluded: the sanitizer serialises kernels across streams, so one rank's
# device-side wait would spin until its timeout for a peer kernel queued behind it.)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export CUART_PREBUCKET=1
SEL="golden or edge or reserved or hand_pins or single_key or range_with_deletes or prebucket_equals_direct or prebucket_updates_equal_direct or bucketed_wide_walk or full_n256 or many_chunks or byte_strings or epoch_wrap or p2p-1 or nccl-1 or p_independent[1 or prebucket_bucket_counts or misaligned or skip_table or partition_by_flag"
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_delete.py tests/test_gpu_range.py tests/test_gpu_dist.py tests/test_gpu_skip.py tests/test_gpu_route.py -m gpu -q -p no:cacheprovider \
    -k "$SEL" > gpurun_out/sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_$tool.log
done
