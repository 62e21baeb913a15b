#!/bin/bash
# Round-2 extra bench lines: the paper's function set, Sedov 100^3 (configs[1]),
# Noh 300^3 on one GPU (configs[3]'s workload), Evrard with gravity.
mkdir -p gpurun_out
A="--steps 10 --warmup 3 --energy-seconds 3 --energy-repeats 1 --trace-seconds 0 --cpu-sample 24"
timeout 900 python bench.py $A --av-switch --gradh --dt-vsig --ve > gpurun_out/r02_bench_paper_functions.log 2>&1
timeout 900 python bench.py $A --workload sedov100 > gpurun_out/r02_bench_sedov100.log 2>&1
timeout 900 python bench.py $A --workload noh300 --dt-vsig > gpurun_out/r02_bench_noh300.log 2>&1
timeout 900 python bench.py $A --workload evrard100 --no-cpu-baseline > gpurun_out/r02_bench_evrard.log 2>&1
for f in paper_functions sedov100 noh300 evrard; do
  python - gpurun_out/r02_bench_$f.log <<'PY'
import json, sys
try:
    l = [x for x in open(sys.argv[1]) if x.startswith('{"metric"')][-1]
    d = json.loads(l)
    print(sys.argv[1], d["config"]["workload"], round(d["value"] / 1e6, 1), "M/s", round(d["ms_per_step"], 2), "ms",
          "parity", (d.get("parity") or {}).get("pass"), {k: round(v, 2) for k, v in d["phase_ms"].items() if v > 0.3})
except Exception as e:
    print(sys.argv[1], "failed", e, open(sys.argv[1]).read()[-800:])
PY
done
