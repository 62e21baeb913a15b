#!/bin/bash
# neighbour search: segmented mask expansion (SPH_NBR_SEG=1) -- tests, then A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decomp.py tests/test_gpu_physics.py -q -x > gpurun_out/seg_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/seg_tests.log
tail -3 gpurun_out/seg_tests.log
VARIANTS=$'\n-DSPH_NBR_SEG=0\n' bash tools/ab.sh 2>&1 | tee gpurun_out/seg_ab.log
