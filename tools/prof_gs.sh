# ncu --set full of the ring group scan (C5 streams, 256 sensors): fp16 ring vs exact f32 ring
mkdir -p gpurun_out
for v in half exact; do
ncu --set full --import-source on --clock-control none -k regex:group_scan_reg -s 2 -c 1 \
    -o gpurun_out/prof_gs_$v -f python tools/prof_stream.py C5 f32 256 4 $v > gpurun_out/prof_gs_$v.log 2>&1
ncu -i gpurun_out/prof_gs_$v.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_gs_${v}_src.csv 2>/dev/null
python tools/ncu_brief.py gpurun_out/prof_gs_$v.ncu-rep
done
