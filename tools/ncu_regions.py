"""Instructions executed per source line of one kernel from an ncu source page
(--page source --csv --print-source=cuda,sass), summed over named line ranges.
Usage: python tools/ncu_regions.py page.csv file.cu name:a-b [name:a-b ...]"""
import csv
import collections
import sys

rows = list(csv.reader(open(sys.argv[1])))
target = sys.argv[2]
agg, src = collections.Counter(), {}
fname, ix = None, None
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if "Instructions Executed" in r:
        ix = r.index("Instructions Executed")
        continue
    if ix is None or len(r) <= ix or not r[0].isdigit():
        continue
    key = (fname, int(r[0]))
    src[key] = r[1]
    try:
        agg[key] += float(r[ix] or 0)
    except ValueError:
        pass
tot = sum(agg.values())
print(f"total warp instructions {tot:.4g}")
for spec in sys.argv[3:]:
    name, rng = spec.rsplit(":", 1)
    a, b = map(int, rng.split("-"))
    v = sum(c for (f, l), c in agg.items() if f == target and a <= l <= b)
    print(f"{name:24s} {100 * v / tot:5.1f}%")
print(f"{'other files':24s} {100 * sum(c for (f, l), c in agg.items() if f != target) / tot:5.1f}%")
for k, c in sorted(agg.items(), key=lambda x: -x[1])[:15]:
    print(k, f"{100 * c / tot:.1f}%", src.get(k, "")[:80])
