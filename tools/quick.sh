# quick GPU check: parity subset + LB timings + C2/C4 bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pt.txt 2>&1; tail -2 gpurun_out/pt.txt
for c in C2 C4; do python tools/prof_lb.py $c f32 3; done
for c in ${QUICK_CONFIGS:-C2 C4}; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > gpurun_out/q_$c.json 2>gpurun_out/q_$c.err; python - $c <<'PY'
import json,sys
c=sys.argv[1]
d=json.loads(open(f"gpurun_out/q_{c}.json").read().strip().splitlines()[-1])
print(c, round(d["value"]), round(d["ms_per_step"],3), {k:round(v,3) for k,v in d["phase_ms_per_step"].items()}, d["roofline"]["kernel"], round(d["roofline"]["frac"],3))
PY
done
