#!/bin/bash
# Round-2 evidence for HEAD (run under gpurun on one B200): the GPU test suite, smoke,
# bench lines of every config (C5 with the 60 s sustained protocol), the reference arm,
# the default command's ncu launch list, ncu --set full summaries of the top kernels
# (C2 one-shot, C3 / C5 streams) with per-MQ DRAM traffic, and the ALU micro-benchmark.
# Reports are summarised on the box and deleted (gpurun_out is capped at 64 MiB).
O=${1:-gpurun_out/r02e}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.limit --format=csv > $O/gpu.txt
(nproc; grep -m1 "model name" /proc/cpuinfo) > $O/host.txt
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.txt 2>&1; tail -2 $O/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
paper_conf_sigmod_zhout15_b200/_build/alu_bench 400 > $O/alu_peaks.json
timeout 900 python bench.py > $O/bench_C2_f32.json 2> $O/bench_C2_f32.err
timeout 900 python bench.py --dtype i16 > $O/bench_C2_i16.json 2> $O/bench_C2_i16.err
timeout 900 python bench.py --config C3 > $O/bench_C3_f32.json 2> $O/bench_C3_f32.err
timeout 900 python bench.py --config C4 > $O/bench_C4_f32.json 2> $O/bench_C4_f32.err
timeout 900 python bench.py --config C5 --sustain-s 60 > $O/bench_C5_f32.json 2> $O/bench_C5_f32.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err
for f in $O/bench_*.json; do echo "$(basename $f): $(python tools/bench_brief.py $f 2>&1 | cut -c1-200)"; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/ncu_launches_c2.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e --two-level-steps 0 --prof-steps 1 > $O/ncu_launches_c2.log 2>&1
python tools/launch_summary.py $O/ncu_launches_c2.csv > $O/ncu_launches_c2.txt
ncu --set full --import-source on --clock-control none -k regex:"lb_diag|dtw_kernel|filter_kernel|tau_|topk|cascade" -c 30 \
    -o $O/prof_c2 -f python tools/prof_lb.py C2 f32 1 > $O/prof_c2.log 2>&1
python tools/ncu_summary.py $O/prof_c2.ncu-rep $O --mq 32 > /dev/null 2>&1
for c in C5 C3; do
  mq=$(python tools/prof_stream.py $c f32 1024 1 2>/dev/null | grep MQ_PER_LAUNCH | cut -d= -f2)
  ncu --set full --import-source on --clock-control none \
      -k regex:"group_scan_tma|dtw_kernel|window_lb_inc|tau_trim|filter_kernel|cascade" -s 12 -c 14 \
      -o $O/prof_$c -f python tools/prof_stream.py $c f32 1024 3 > $O/prof_$c.log 2>&1
  python tools/ncu_summary.py $O/prof_$c.ncu-rep $O --mq ${mq:-1024} > /dev/null 2>&1
done
for f in $O/*.ncu-rep; do
  b=${f%.ncu-rep}
  python tools/ncu_brief.py $f > ${b}_brief.txt 2>&1
  ncu -i $f --page source --csv --print-source sass 2>/dev/null | gzip > ${b}_src.csv.gz
  rm -f $f
done
ls -la $O
