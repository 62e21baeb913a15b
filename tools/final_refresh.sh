#!/bin/bash
# End-of-round evidence on one GPU: GPU tests, smoke, the default bench line, the
# paper's function set, the ncu launch list and one full-set capture per kernel.
mkdir -p gpurun_out
TAG=${TAG:-r02f}
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" | tee -a gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py --out gpurun_out/${TAG}_bench.json > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?"
timeout 600 python bench.py --av-switch --gradh --dt-vsig --ve --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline > gpurun_out/${TAG}_bench_paper_functions.log 2>&1; echo "bench paper rc=$?"
TAG=${TAG} bash tools/ncu_profile.sh
