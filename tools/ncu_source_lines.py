"""Per-source-line totals (instructions executed, stall samples) from
`ncu -i REP --page source --csv --print-source cuda,sass --kernel-name K`.
Usage: python tools/ncu_source_lines.py CSV [TOP]"""
import csv
import sys
from collections import defaultdict


def main(path, top=40):
    inst = defaultdict(int)
    samp = defaultdict(int)
    text = {}
    f = None
    cur = None
    hdr = None
    for row in csv.reader(open(path)):
        if not row:
            continue
        if row[0] == "File Path":
            f = row[1].split("/")[-1]
            continue
        if row[0] == "Line No":
            hdr = row
            continue
        if hdr is None or len(row) < 8:
            continue
        if row[0]:  # a source line row (aggregate of its SASS); keep it
            cur = (f, int(row[0]))
            text[cur] = row[1].strip()[:90]
            try:
                inst[cur] += int(row[hdr.index("Instructions Executed")])
                samp[cur] += int(row[hdr.index("Warp Stall Sampling (All Samples)")])
            except ValueError:
                pass
    ti = sum(inst.values()) or 1
    ts = sum(samp.values()) or 1
    print(f"total instructions {ti:.4g}, samples {ts}")
    for k in sorted(inst, key=lambda k: -samp[k])[:top]:
        print(f"{k[0]}:{k[1]:<5} inst {100 * inst[k] / ti:5.1f}%  samples {100 * samp[k] / ts:5.1f}%  {text[k]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)


def stalls(path, lines):
    """Stall-reason breakdown (sampled) of the given source lines."""
    hdr = None
    f = None
    out = {}
    for row in csv.reader(open(path)):
        if not row:
            continue
        if row[0] == "File Path":
            f = row[1].split("/")[-1]
            continue
        if row[0] == "Line No":
            hdr = row
            continue
        if hdr is None or not row[0]:
            continue
        key = f"{f}:{row[0]}"
        if key in lines:
            cols = [(h, row[k]) for k, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
            out[key] = {h[6:]: int(v) for h, v in cols if v not in ("", "-", "0")}
    return out
