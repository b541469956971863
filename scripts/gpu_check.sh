#!/bin/bash
# GPU test suite (all -m gpu tests, full-size parity included) + smoke; logs under gpurun_out/
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout ${PYTEST_TIMEOUT:-2400} python -m pytest ${PYTEST_ARGS:-tests} -m gpu -q -x -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
