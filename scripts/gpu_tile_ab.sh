#!/bin/bash
mkdir -p gpurun_out
bash scripts/gpu_2rank.sh
