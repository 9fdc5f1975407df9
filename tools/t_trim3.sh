timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "trim or c2_reduced or stream_steps_c5 or c5_reduced" 2>&1 | tail -1
bash tools/bench_brief.sh C2 --no-e2e --two-level-steps 0
bash tools/bench_brief.sh C3 --no-e2e
python - <<'PY'
import json
d=json.loads(open("/tmp/bb.json").read().strip().splitlines()[-1]); print(d["clocks"])
PY
