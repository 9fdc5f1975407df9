timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -4
for c in C5 C3; do bash tools/bench_brief.sh $c; bash tools/bench_brief.sh $c --tau-mult -1; done
bash tools/prof_gs.sh 2>&1 | grep -E "==|dram__throughput|issue_active|warps_active|long_score|duration"
bash tools/prof_pred.sh 2>&1 | tail -25
