#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -2
VARIANTS=$'\n-DSPH_NBR_DISCARD=0\n' bash tools/ab.sh 2>&1 | tee gpurun_out/discard_ab.log
K=neighbors_kernel VARIANTS=$'\n-DSPH_NBR_DISCARD=0\n' bash tools/ncu_dram.sh 2>&1 | tee gpurun_out/discard_dram.log
