mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "stream or continuous or shared_running_tau" 2>&1 | tail -3
for c in C3 C5; do for ab in 0 8; do
SMILER_AB=$ab timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/p_${c}_$ab.json 2>gpurun_out/p_${c}_$ab.err
python - $c $ab <<'PY'
import json,sys
d=json.loads(open(f'gpurun_out/p_{sys.argv[1]}_{sys.argv[2]}.json').read().strip().splitlines()[-1])
print(sys.argv[1], 'AB', sys.argv[2], round(d['value']), 'ms', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phase_ms_per_step'].items()}, 'gs frac', round(d['kernels'].get('group_scan_a4',{}).get('frac',0),3), 'surv', round(d['survivor_frac'],4))
PY
done; done
