timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "stream or continuous or shared_running_tau" 2>&1 | tail -4
for c in C5 C3; do bash tools/bench_brief.sh $c; done
timeout 600 python tools/shared_tau_bench.py
