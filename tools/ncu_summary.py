"""Summarise an ncu --set full report into profiles/: one markdown table plus a
JSON of per-kernel DRAM traffic normalised per master query (read by bench.py
for the roofline's `traffic` key).

    python tools/ncu_summary.py gpurun_out/r01/prof_c2.ncu-rep profiles/r01 --mq 32
"""
import argparse
import csv
import io
import json
import os
import subprocess

KEYS = [
    ("gpu__time_duration.sum", "time_us", "time"),
    ("dram__bytes_read.sum", "dram_read_MB", None),
    ("dram__bytes_write.sum", "dram_write_MB", None),
    ("FBSP.TriageCompute.dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct", 1),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_pct", 1),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_pct", 1),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "alu_pipe_pct", 1),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "fma_pipe_pct", 1),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_pct", 1),
    ("launch__registers_per_thread", "regs", 1),
    ("launch__grid_size", "grid", 1),
    ("launch__block_size", "block", 1),
]


def to_bytes(v, unit):
    u = (unit or "").strip().lower()
    mult = {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9}.get(u, 1)
    return float(v) * mult


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("outdir")
    ap.add_argument("--mq", type=int, required=True, help="master queries per launch in the profiled run")
    a = ap.parse_args()
    raw = subprocess.run(["ncu", "-i", a.rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    os.makedirs(a.outdir, exist_ok=True)
    lines = ["| kernel | " + " | ".join(k[1] for k in KEYS) + " |", "|" + "---|" * (len(KEYS) + 1)]
    traffic = {}
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        name = d["Kernel Name"].split("(")[0].replace("void ", "")
        cells = []
        for key, lab, sc in KEYS:
            v = d.get(key, "")
            try:
                float(v.replace(",", ""))
            except ValueError:
                v = ""
            if v == "":
                cells.append("")
                continue
            if sc == "time":
                tu = (u.get(key) or "").strip().lower()
                f = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3,
                     "second": 1e6, "s": 1e6}.get(tu, 1.0)
                cells.append("%.1f" % (float(v.replace(",", "")) * f))
            elif sc is None:
                cells.append("%.1f" % (to_bytes(v, u.get(key)) / 1e6))
            else:
                cells.append("%.4g" % (float(v.replace(",", "")) * sc))
        lines.append("| %s | %s |" % (name, " | ".join(cells)))
        if "dram__bytes_read.sum" in d:
            b = to_bytes(d["dram__bytes_read.sum"], u.get("dram__bytes_read.sum")) + \
                to_bytes(d["dram__bytes_write.sum"], u.get("dram__bytes_write.sum"))
            traffic.setdefault(name, []).append(b / a.mq)
    base = os.path.splitext(os.path.basename(a.rep))[0]
    with open(os.path.join(a.outdir, base + "_summary.md"), "w") as f:
        f.write("ncu --set full summary of `%s` (%d master queries per launch; DRAM MB per launch)\n\n" %
                (os.path.basename(a.rep), a.mq))
        f.write("\n".join(lines) + "\n")
    with open(os.path.join(a.outdir, base + "_traffic_per_mq.json"), "w") as f:
        json.dump({k: sorted(v)[len(v) // 2] for k, v in traffic.items()}, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
