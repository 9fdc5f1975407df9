"""One-line summary of a bench.py JSON output file (the last line of it)."""
import json
import sys

t = open(sys.argv[1]).read().strip()
d = json.loads(t.splitlines()[-1])
ph = {k: round(v, 3) for k, v in d.get("phase_ms_per_step", {}).items() if v > 0.01}
rf = d.get("roofline", {})
print("%.1f MQ/s  %.3f ms/step  %s  dominant %s frac %.3f  clk %s %s" % (
    d["value"], d["ms_per_step"], ph, rf.get("kernel"), rf.get("frac", 0), d.get("clocks", {}).get("sm_mhz"),
    d.get("clocks", {}).get("reasons")))
