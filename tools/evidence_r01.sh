# Round-1 evidence for HEAD: bench lines (all configs), the default command's ncu launch list,
# ncu --set full summaries of the top kernels (reports reduced on the box: gpurun_out cap 64 MiB)
O=${1:-gpurun_out/r01e}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $O/pytest_gpu.txt 2>&1; tail -2 $O/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print(\"smoke ok\")" > $O/smoke.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt
timeout 900 python bench.py > $O/bench_C2_f32.json 2> $O/bench_C2_f32.err
timeout 900 python bench.py --dtype i16 > $O/bench_C2_i16.json 2> $O/bench_C2_i16.err
for c in C3 C4 C5; do timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/ncu_launches_c2.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e --two-level-steps 0 > $O/ncu_launches_c2.log 2>&1
python tools/launch_summary.py $O/ncu_launches_c2.csv > $O/ncu_launches_c2.txt
ncu --set full --import-source on --clock-control none -k regex:"lb_diag|dtw_kernel|filter_kernel|tau_|topk" -c 24 \
    -o $O/prof_c2 -f python tools/prof_lb.py C2 f32 1 > $O/prof_c2.log 2>&1
python tools/ncu_summary.py $O/prof_c2.ncu-rep $O --mq 32 > /dev/null 2>&1
for c in C5 C3; do
  ncu --set full --import-source on --clock-control none -k regex:"group_scan_tma|dtw_kernel|window_lb_inc|tau_trim|filter_kernel" \
      -s 10 -c 12 -o $O/prof_$c -f python tools/prof_stream.py $c f32 1024 3 > $O/prof_$c.log 2>&1
  python tools/ncu_summary.py $O/prof_$c.ncu-rep $O --mq $([ $c = C5 ] && echo 10240 || echo 1024) > /dev/null 2>&1
done
for f in $O/*.ncu-rep; do
  b=${f%.ncu-rep}
  python tools/ncu_brief.py $f > ${b}_brief.txt 2>&1
  ncu -i $f --page source --csv --print-source sass 2>/dev/null | gzip > ${b}_src.csv.gz
  rm -f $f
done
ls -la $O
