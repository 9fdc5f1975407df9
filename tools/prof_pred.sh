# ncu --set full of predict_kernel (C5 shape, 64 sensors, EKV 32,64,128), source-level SASS export
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:predict_kernel -c 1 \
    -o gpurun_out/prof_pred -f python tools/predict_bench.py --sensors 64 --reps 1 > gpurun_out/prof_pred.log 2>&1
ncu -i gpurun_out/prof_pred.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_pred_src.csv 2>/dev/null
python tools/ncu_brief.py gpurun_out/prof_pred.ncu-rep
python tools/src_ops.py gpurun_out/prof_pred_src.csv 20
