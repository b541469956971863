#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "prebucket or c2_full or c1_full" > gpurun_out/pytest_b2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_b2.log
timeout 600 python tools/sweep.py --config c3 --formats 3 --policies 5 --reps 5 > gpurun_out/bucket.json 2> gpurun_out/bucket.err
timeout 600 python tools/sweep.py --config c2 --formats 3 --policies 5 --reps 5 >> gpurun_out/bucket.json 2>> gpurun_out/bucket.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_b|k_lookup" --csv --log-file gpurun_out/bucket_ncu.csv python tools/profile_variants.py > /dev/null 2>&1
