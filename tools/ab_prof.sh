#!/bin/bash
# ncu --set full of the neighbour sums under two SPH_SUM_LANES settings.
mkdir -p gpurun_out
for G in ${LANES:-1 8}; do
  SPH_SUM_LANES=$G K='density|momentum' TAG=ab_prof_$G SKIP=${SKIP:-2} COUNT=2 bash tools/ncu_one.sh
done
