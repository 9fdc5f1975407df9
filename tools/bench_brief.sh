# one bench run, one summary line: bench_brief.sh CONFIG [extra bench args]
c=$1; shift
timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu "$@" > /tmp/bb.json 2>/tmp/bb.err || tail -3 /tmp/bb.err
python - $c <<'PY'
import json,sys
d=json.loads(open("/tmp/bb.json").read().strip().splitlines()[-1])
print(sys.argv[1], round(d["value"]), round(d["ms_per_step"],3), {k:round(v,3) for k,v in d["phase_ms_per_step"].items()}, d["roofline"]["kernel"], round(d["roofline"]["frac"],3), {k: round(v["frac"],3) for k,v in d.get("kernels",{}).items()})
PY
