mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pt.txt 2>&1; tail -3 gpurun_out/pt.txt
timeout 600 python bench.py > gpurun_out/bench_default.json 2>gpurun_out/bench_default.err; tail -c 3000 gpurun_out/bench_default.json
for c in C2 C3 C5 C4; do timeout 600 python bench.py --config $c --dtype f32 --steps 10 --warmup 3 > gpurun_out/gs_$c.json 2>gpurun_out/gs_$c.err; tail -c 400 gpurun_out/gs_$c.json; echo; done
