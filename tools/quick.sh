#!/bin/bash
# Quick GPU iteration: build, short bench (no e2e/energy/cpu legs), parity tests.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { echo build failed; tail gpurun_out/build.log; exit 1; }
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds ${TRACE:-0} --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/quick_bench.log 2>&1; echo "bench rc=$?"
python - <<'PY'
import json
for l in open('gpurun_out/quick_bench.log'):
    if l.startswith('{'):
        d = json.loads(l)
        print(round(d['value'] / 1e6, 1), 'M/s', round(d['ms_per_step'], 2), 'ms', {k: round(v, 2) for k, v in d['phase_ms'].items()})
        if d.get('dvfs_trace'):
            print('dvfs', json.dumps(d['dvfs_trace']))
PY
if [ -z "$NOTEST" ]; then timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/quick_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/quick_pytest.log; fi
