"""Counted FP64 work of the neighbour-sum kernels (VERDICT r1 'Next round' 3):
parses an ncu CSV with sm__sass_thread_inst_executed_op_{dfma,dmul,dadd}_pred_on.sum
(+ time, DRAM bytes) of one bench step, and the bench line of the same run (for
the neighbour-pair count n x mean_nc), and writes profiles/r02_dp_counts.json:
per kernel the DP flops per pair = (2 DFMA + DMUL + DADD) / pairs, next to
SURVEY.md 8(d)'s algorithmic counts (density 44, IAD 60, momentum 171).

    python tools/ncu_dp_counts.py gpurun_out/dp.csv gpurun_out/dp_bench.log
"""
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ALGO = {"density_kernel": 44, "iad_kernel": 60, "momentum_energy_kernel": 171}


def main(csv_path, log_path):
    txt = open(csv_path).read()
    txt = txt[txt.index('"ID"'):]
    rows = list(csv.DictReader(io.StringIO(txt)))
    line = [l for l in open(log_path) if l.startswith('{"metric"')][-1]
    bench = json.loads(line)
    n = bench["config"]["n_particles_per_gpu"]
    pairs = n * bench["config"]["mean_nc"]
    per = {}
    for r in rows:
        k = r["Kernel Name"].split("(")[0].replace("void ", "")
        v = r["Metric Value"].replace(",", "")
        try:
            v = float(v)
        except ValueError:
            continue
        unit = r.get("Metric Unit", "")
        scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "msecond": 1e-3, "usecond": 1e-6,
                 "nsecond": 1e-9, "second": 1.0}.get(unit, 1.0)
        per.setdefault((r["ID"], k), {})[r["Metric Name"]] = v * scale
    out = {}
    for (_, k), m in per.items():
        if k in out:
            continue
        dfma = m.get("sm__sass_thread_inst_executed_op_dfma_pred_on.sum", 0.0)
        dmul = m.get("sm__sass_thread_inst_executed_op_dmul_pred_on.sum", 0.0)
        dadd = m.get("sm__sass_thread_inst_executed_op_dadd_pred_on.sum", 0.0)
        fl = 2 * dfma + dmul + dadd
        t = m.get("gpu__time_duration.sum")
        out[k] = {"dfma": dfma, "dmul": dmul, "dadd": dadd, "dp_flops": fl,
                  "dp_flops_per_pair": fl / pairs, "algorithmic_flops_per_pair": ALGO.get(k),
                  "time_s": t, "tflops_counted_ncu": fl / t / 1e12 if t else None,
                  "dram_bytes": m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)}
    res = {"what": "FP64 instructions executed per neighbour pair, ncu SASS counters, one step of "
                   f"{bench['config']['workload']} (n = {n}, mean nc = {bench['config']['mean_nc']:.3f}); "
                   "DP flops = 2 DFMA + DMUL + DADD (thread-level, predicated on)",
           "pairs": pairs, "kernels": out}
    path = os.path.join(ROOT, "profiles", "r02_dp_counts.json")
    json.dump(res, open(path, "w"), indent=1)
    print(json.dumps({k: round(v["dp_flops_per_pair"], 2) for k, v in out.items()}))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
