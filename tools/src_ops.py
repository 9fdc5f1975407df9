"""Summarise an ncu --page source --print-source sass CSV by opcode and stall reason."""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
recs = [dict(zip(h, r)) for r in rows[2:] if len(r) == len(h)]


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


ti = sum(f(r["Instructions Executed"]) for r in recs) or 1
ts = sum(f(r["Warp Stall Sampling (All Samples)"]) for r in recs) or 1
ci, cs = Counter(), Counter()
for r in recs:
    toks = r["Source"].split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
    op = op.split(".")[0]
    ci[op] += f(r["Instructions Executed"])
    cs[op] += f(r["Warp Stall Sampling (All Samples)"])
print("warp insts %.4g, stall samples %d" % (ti, ts))
for op, v in ci.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 15):
    print("%-10s %6.2f%% inst %6.2f%% stall" % (op, 100 * v / ti, 100 * cs[op] / ts))
stalls = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
tot = {k: sum(f(r[k]) for r in recs) for k in stalls}
print(" ".join("%s=%.1f%%" % (k[6:], 100 * v / ts) for k, v in sorted(tot.items(), key=lambda x: -x[1])[:9]))
