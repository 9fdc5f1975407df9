timeout 600 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "stream_steps_c5 or c2 or C2" 2>&1 | tail -2
for kp in 0 4 8 16; do echo -n "keep $kp: "; SMILER_TAU_KEEP=$kp bash tools/bench_brief.sh C2 --no-e2e --two-level-steps 0; done
for kp in 0 1 2; do echo -n "keep $kp: "; SMILER_TAU_KEEP=$kp bash tools/bench_brief.sh C5 --no-e2e; done
for kp in 0 1 2; do echo -n "keep $kp: "; SMILER_TAU_KEEP=$kp bash tools/bench_brief.sh C3 --no-e2e; done
for kp in 0 2 8; do echo -n "keep $kp: "; SMILER_TAU_KEEP=$kp bash tools/bench_brief.sh C4 --no-e2e; done
