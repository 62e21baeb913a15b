#!/bin/bash
# ncu evidence for one round: (1) the launch list of a short bench run,
# (2) one full-set capture of each neighbour-sum kernel.  Writes gpurun_out/.
TAG=${TAG:-r01}
mkdir -p gpurun_out
ARGS="--steps 2 --warmup 1 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline ${BENCH_ARGS}"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py $ARGS > gpurun_out/${TAG}_ncu_launch_bench.log 2>&1
echo "launch list rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on \
  -k regex:"neighbors_kernel|momentum_energy_kernel|density_kernel|iad_kernel|onesweep|permute|sort_fixup|update_kernel|eos_kernel" -s 12 -c 12 \
  -o gpurun_out/${TAG}_full python bench.py $ARGS > gpurun_out/${TAG}_ncu_full.log 2>&1
echo "full rc=$?"
