#!/bin/bash
# A/B of the neighbour-sum layouts (SPH_SUM_LANES = lanes per target).
mkdir -p gpurun_out
for G in ${LANES:-1 4 8 16}; do
  SPH_SUM_LANES=$G timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --energy-steps 0 --no-cpu-baseline > gpurun_out/ab_$G.log 2>&1
  echo "G=$G rc=$?"
done
SPH_SUM_LANES=${TEST_LANES:-8} timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab.log 2>&1; echo "pytest rc=$?"
