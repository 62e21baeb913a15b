#!/bin/bash
# Round-2 evidence: GPU tests, smoke, the default bench line, ncu launch list and
# full-set captures (tools/ncu_profile.sh), summaries for profiles/.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
TAG=r02 bash tools/ncu_profile.sh > gpurun_out/ncu_profile.log 2>&1
python tools/ncu_summary.py gpurun_out/r02_full.ncu-rep > gpurun_out/r02_ncu_full_summary.json 2>&1
python tools/ncu_summary.py --launches gpurun_out/r02_launches.csv > gpurun_out/r02_launch_shares.json 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; tail -c 300 gpurun_out/bench.log; cat gpurun_out/ncu_profile.log
