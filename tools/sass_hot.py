"""Rank SASS instructions of an ncu --page source --print-source sass CSV by
executed instructions and stall samples; print contiguous hot regions."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
recs = []
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    recs.append((int(d["Address"], 16) if d["Address"].startswith("0x") else int(d["Address"]), d["Source"],
                 float(d["Instructions Executed"] or 0), float(d["Warp Stall Sampling (All Samples)"] or 0)))
ti = sum(x[2] for x in recs) or 1
ts = sum(x[3] for x in recs) or 1
print("total warp insts %.3g, samples %d" % (ti, ts))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 0
if n:
    for i, x in enumerate(recs):
        if x[2] / ti > 1e-3 or x[3] / ts > 5e-3:
            print("%5d %6.2f%% %6.2f%%  %s" % (i, 100 * x[2] / ti, 100 * x[3] / ts, x[1][:80]))
