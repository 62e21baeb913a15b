#!/bin/bash
# Round-2 GPU session: DP instruction counts (ncu), GPU tests, smoke, full bench.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  -k regex:"density_kernel|iad_kernel|momentum_energy_kernel|neighbors_kernel" -c 4 --clock-control none --csv --log-file gpurun_out/dp.csv \
  python bench.py --steps 1 --warmup 0 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline > gpurun_out/dp_bench.log 2>&1
python tools/ncu_dp_counts.py gpurun_out/dp.csv gpurun_out/dp_bench.log > gpurun_out/dp_counts.txt 2>&1
cp profiles/r02_dp_counts.json gpurun_out/ 2>/dev/null
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; cat gpurun_out/dp_counts.txt; tail -c 600 gpurun_out/bench.log
