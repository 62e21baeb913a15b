#!/bin/bash
# ncu --set full of one kernel (regex $K) on a short bench run; writes gpurun_out/$TAG.ncu-rep
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$K" -s ${SKIP:-1} -c ${COUNT:-1} \
  -o gpurun_out/${TAG} python bench.py --steps 2 --warmup 1 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/${TAG}.log 2>&1
echo "rc=$?"
