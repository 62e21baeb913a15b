#!/bin/bash
# neighbour search: warp run scan (SPH_NBR_RUNSCAN) and CTAs per SM -- tests, then A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decomp.py -q -x > gpurun_out/scan_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/scan_tests.log
tail -3 gpurun_out/scan_tests.log
VARIANTS=$'\n-DSPH_NBR_RUNSCAN=0\n-DSPH_NBR_MINB=7\n-DSPH_NBR_MINB=5\n' bash tools/ab.sh 2>&1 | tee gpurun_out/scan_ab.log
