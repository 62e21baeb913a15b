VARIANTS=$(printf "\n-DSPH_MOM_DIAG=1\n-DSPH_MOM_DIAG=2\n") bash tools/ab.sh
python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)"
A="--steps 10 --warmup 3 --energy-seconds 3 --energy-repeats 1 --trace-seconds 0 --cpu-sample 24"
timeout 900 python bench.py $A --av-switch --gradh --dt-vsig --ve > gpurun_out/r02_bench_paper_functions.log 2>&1
timeout 900 python bench.py $A --workload sedov100 > gpurun_out/r02_bench_sedov100.log 2>&1
for f in paper_functions sedov100; do
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
