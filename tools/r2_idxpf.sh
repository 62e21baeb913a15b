#!/bin/bash
mkdir -p gpurun_out
VARIANTS=$'\n-DSPH_IDX_PF=0\n-DSPH_IDX_PF=16\n-DSPH_IDX_PF=8 -DSPH_IDX_PF_L1=1\n' bash tools/ab.sh 2>&1 | tee gpurun_out/idxpf_ab.log
