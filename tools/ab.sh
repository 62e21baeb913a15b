#!/bin/bash
# A/B of compile-time variants: each line of $VARIANTS is an SPH_NVCC_EXTRA value
mkdir -p gpurun_out
while IFS= read -r v; do
  SPH_NVCC_EXTRA="$v" python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1 || { echo "build failed: $v"; continue; }
  timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ab.log 2>&1
  python - "$v" <<'PY'
import json, sys
for l in open('gpurun_out/ab.log'):
    if l.startswith('{'):
        d = json.loads(l)
        print(sys.argv[1] or 'base', round(d['value'] / 1e6, 1), 'M/s', {k: round(v, 2) for k, v in d['phase_ms'].items() if v > 0.5})
PY
done <<< "$VARIANTS"
