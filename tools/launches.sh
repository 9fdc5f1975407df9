# ncu launch list (kernel durations) of one bench step: launches.sh CONFIG OUTNAME
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$2.csv \
    python bench.py --config $1 --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/$2.log 2>&1
python tools/launch_summary.py gpurun_out/$2.csv
