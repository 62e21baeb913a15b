#!/bin/bash
# neighbour search: batched flattened append (SPH_NBR_BATCH) -- tests, then A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decomp.py -q -x > gpurun_out/batch_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/batch_tests.log
tail -3 gpurun_out/batch_tests.log
VARIANTS=$'\n-DSPH_NBR_BATCH=0\n-DSPH_NBR_BATCH=4\n-DSPH_NBR_BATCH=16\n' bash tools/ab.sh 2>&1 | tee gpurun_out/batch_ab.log
