"""Aggregate an ncu source page (--print-source=cuda,sass CSV) by CUDA source line."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
for hi, r in enumerate(rows):
    if "Instructions Executed" in r:
        break
hdr = rows[hi]
ix = hdr.index("Instructions Executed")
iss = hdr.index("Warp Stall Sampling (All Samples)")
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
agg_i, agg_s, src, st = collections.Counter(), collections.Counter(), {}, collections.Counter()
cur = None
for r in rows[hi + 1:]:
    if len(r) < 4:
        continue
    if r[0]:
        cur = r[0]
        src[cur] = r[1][:90]
    try:
        agg_i[cur] += int(r[ix] or 0)
        agg_s[cur] += int(r[iss] or 0)
        for h in stalls:
            st[h] += int(r[hdr.index(h)] or 0)
    except (ValueError, IndexError):
        pass
ts, ti = sum(agg_s.values()), sum(agg_i.values())
print("samples", ts, "inst", ti)
print(st.most_common(6))
for ln, v in agg_s.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 25):
    print(ln, round(v / ts, 3), agg_i[ln], src.get(ln))
