O=gpurun_out/g12; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "dtw or stream or cascade or c2 or C2" > $O/pytest.txt 2>&1; tail -2 $O/pytest.txt
for r in 1 2; do for c in C5 C3 C2; do timeout 600 python bench.py --config $c --no-cpu --no-e2e --two-level-steps 0 --prof-steps 5 2>/dev/null | python tools/bench_brief.py /dev/stdin; done; done
