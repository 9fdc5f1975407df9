timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "trim or c4 or c2_reduced or stream_steps_c5" 2>&1 | tail -3
for kp in -1 0 32; do echo -n "keep $kp: "; SMILER_TAU_KEEP=$kp bash tools/bench_brief.sh C4 --no-e2e; done
