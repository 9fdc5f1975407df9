# ncu --set full of the DTW kernels on a C5-shaped run (64 sensors), source-level SASS export
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:dtw_kernel -c 8 \
    -o gpurun_out/prof_dtw -f python tools/prof_c5.py f32 64 > gpurun_out/prof_dtw.log 2>&1
ncu -i gpurun_out/prof_dtw.ncu-rep --page raw --csv > gpurun_out/prof_dtw.raw.csv
for i in 0 1 2 3 4 5 6 7; do
  ncu -i gpurun_out/prof_dtw.ncu-rep --page source --csv --print-source sass --launch-skip $i --launch-count 1 > gpurun_out/prof_dtw_src$i.csv 2>/dev/null
done
tail -3 gpurun_out/prof_dtw.log
