#!/bin/bash
mkdir -p gpurun_out
VARIANTS=$'\n-DSPH_MOM_PF=1 -DSPH_MOM_THREADS=384\n-DSPH_MOM_THREADS=384\n-DSPH_MOM_PF=1 -DSPH_MOM_THREADS=320\n' bash tools/ab.sh 2>&1 | tee gpurun_out/mompf_ab.log
