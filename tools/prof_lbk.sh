# ncu --set full of lb_diag_kernel (w=8 on C2, w=16 on C4-shaped), source-level SASS export
mkdir -p gpurun_out
for c in C2 C4; do
ncu --set full --import-source on --clock-control none -k regex:lb_diag -c 1 \
    -o gpurun_out/prof_lb_$c -f python tools/prof_lb.py $c f32 1 > gpurun_out/prof_lb_$c.log 2>&1
ncu -i gpurun_out/prof_lb_$c.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_lb_${c}_src.csv 2>/dev/null
done
for c in C2 C4; do python tools/prof_lb.py $c f32 3; done
