#!/bin/bash
# end-of-round check at HEAD: full GPU suite + smoke, then the 2-rank bench smokes (shared GPU)
mkdir -p gpurun_out
bash scripts/gpu_check.sh
bash scripts/gpu_2rank.sh
