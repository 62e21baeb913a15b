#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/copy_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/copy_tests.log
tail -2 gpurun_out/copy_tests.log
VARIANTS=$'\n-DSPH_NBR_COPYPIPE=0\n' bash tools/ab.sh 2>&1 | tee gpurun_out/copy_ab.log
