"""Sum an ncu --metrics gpu__time_duration.sum --csv launch list by kernel name."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h = rows[0]
ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    name = r[ki].split("(")[0]
    v = float(r[vi].replace(",", ""))
    unit = r[h.index("Metric Unit")] if "Metric Unit" in h else "ns"
    v *= {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3}.get(unit, 1.0)
    tot[name] += v
    cnt[name] += 1
T = sum(tot.values())
for n, v in sorted(tot.items(), key=lambda x: -x[1]):
    print("%10.1f us %5.1f%% %5d  %s" % (v, 100 * v / T, cnt[n], n[:100]))
print("total %.1f us" % T)
