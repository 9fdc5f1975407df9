timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -1
bash tools/bench_brief.sh C2 --no-e2e --two-level-steps 0
bash tools/bench_brief.sh C5 --no-e2e
bash tools/bench_brief.sh C4 --no-e2e
bash tools/bench_brief.sh C3 --no-e2e
