bash tools/ab.sh bash -c 'for c in C2 C5; do bash tools/bench_brief.sh $c --no-e2e --two-level-steps 0; done'
