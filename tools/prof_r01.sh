# Round-1 evidence for HEAD: launch lists of the bench commands + ncu --set full of the top kernels.
# Reports are reduced on the box to raw/source CSVs (gpurun_out is capped at 64 MiB).
O=gpurun_out/r01p; mkdir -p $O
for c in C2 C3 C5; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$c.csv \
      python bench.py --config $c --steps 1 --warmup 1 --no-cpu --no-e2e > $O/launches_$c.log 2>&1
  python tools/launch_summary.py $O/launches_$c.csv > $O/launches_$c.txt
done
ncu --set full --import-source on --clock-control none -k regex:lb_diag -c 1 \
    -o $O/prof_lb_C2 -f python tools/prof_lb.py C2 f32 1 > $O/prof_lb_C2.log 2>&1
for c in C3 C5; do
ncu --set full --import-source on --clock-control none -k regex:"group_scan_tma|dtw_kernel" -s 4 -c 6 \
    -o $O/prof_stream_$c -f python tools/prof_stream.py $c f32 1024 3 > $O/prof_stream_$c.log 2>&1
done
for f in $O/*.ncu-rep; do
  b=${f%.ncu-rep}
  python tools/ncu_brief.py $f > ${b}_brief.txt 2>&1
  ncu -i $f --page raw --csv > ${b}_raw.csv 2>/dev/null
  ncu -i $f --page source --csv --print-source sass > ${b}_src.csv 2>/dev/null
  gzip -f ${b}_src.csv ${b}_raw.csv
  rm -f $f
done
ls -la $O
