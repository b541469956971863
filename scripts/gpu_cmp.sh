#!/bin/bash
# A/B: co-located conflict word (current build) vs separate array (rebuilt variant)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_colo.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_colo.log
timeout 600 python tools/sweep.py --config c3 --formats 3 --policies 5 > gpurun_out/sweep_colo_c3.json 2>&1
timeout 600 python tools/sweep.py --config c2 --formats 3 --policies 5 > gpurun_out/sweep_colo_c2.json 2>&1
CUART_DEFS="-DCUART_COLOCATED_WINNER=0" python -m paper_conf_icpp_koppehelggp21_b200.build --force > /dev/null 2>&1
timeout 600 python tools/sweep.py --config c3 --formats 3 --policies 5 > gpurun_out/sweep_sep_c3.json 2>&1
timeout 600 python tools/sweep.py --config c2 --formats 3 --policies 5 > gpurun_out/sweep_sep_c2.json 2>&1
