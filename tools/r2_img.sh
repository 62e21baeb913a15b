#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/img_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/img_tests.log
tail -3 gpurun_out/img_tests.log
VARIANTS=$'\n-DSPH_NBR_IMGSKIP=0\n' bash tools/ab.sh 2>&1 | tee gpurun_out/img_ab.log
