mkdir -p gpurun_out
for c in C2 C3 C5; do python bench.py --config $c --dtype f32 --steps 10 --warmup 3 > gpurun_out/gs_$c.json 2>gpurun_out/gs_$c.err; done
python bench.py --config C2 --dtype i16 --steps 10 --warmup 3 > gpurun_out/gs_C2i.json 2>gpurun_out/gs_C2i.err
python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pt.txt 2>&1; tail -1 gpurun_out/pt.txt
