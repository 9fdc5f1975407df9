bash tools/ab.sh bash -c 'timeout 600 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "stream" 2>&1 | tail -1; for c in C3; do bash tools/bench_brief.sh $c --no-e2e; done'
