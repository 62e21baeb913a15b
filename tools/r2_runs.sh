#!/bin/bash
# neighbour search: small run table (more L1) -- tests, then A/B vs the 512-run table
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decomp.py -q -x > gpurun_out/runs_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/runs_tests.log
tail -3 gpurun_out/runs_tests.log
VARIANTS=$'\n-DSPH_NBR_MAXRUNS=512\n' bash tools/ab.sh 2>&1 | tee gpurun_out/runs_ab.log
