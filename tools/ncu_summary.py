"""Summarise ncu captures for profiles/: per-kernel duration, DRAM bytes, FP64
pipe, L1 wavefronts, occupancy (full set), or the share of each kernel in a
launch list (--launches CSV)."""
import collections
import csv
import io
import json
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
           "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
           "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
           "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
           "sm__sass_thread_inst_executed_op_dfma_pred_on.sum",
           "sm__sass_thread_inst_executed_op_dmul_pred_on.sum",
           "sm__sass_thread_inst_executed_op_dadd_pred_on.sum",
           "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
           "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio"]


def full(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(METRICS)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        item = {"kernel": d["Kernel Name"].split("(")[0].replace("void ", "")}
        for m in METRICS:
            if m in d and d[m] not in ("", "n/a"):
                try:
                    item[m] = float(d[m].replace(",", ""))
                    item[m + ".unit"] = u.get(m, "")
                except ValueError:
                    pass
        dfma = item.get("sm__sass_thread_inst_executed_op_dfma_pred_on.sum", 0)
        dmul = item.get("sm__sass_thread_inst_executed_op_dmul_pred_on.sum", 0)
        dadd = item.get("sm__sass_thread_inst_executed_op_dadd_pred_on.sum", 0)
        item["dp_flops_executed"] = 2 * dfma + dmul + dadd
        res.append(item)
    return res


def launches(csvfile):
    rows = list(csv.reader(open(csvfile)))
    for hi, r in enumerate(rows):
        if "Kernel Name" in r:
            break
    hdr = rows[hi]
    ik, im, iv = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    tot = collections.Counter()
    cnt = collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) > iv and r[im] == "gpu__time_duration.sum":
            k = r[ik].split("(")[0].replace("void ", "")
            tot[k] += float(r[iv].replace(",", ""))
            cnt[k] += 1
    s = sum(tot.values())
    return [{"kernel": k, "launches": cnt[k], "total": v, "share": v / s} for k, v in tot.most_common()]


if __name__ == "__main__":
    if sys.argv[1] == "--launches":
        print(json.dumps(launches(sys.argv[2]), indent=1))
    else:
        print(json.dumps(full(sys.argv[1]), indent=1))
