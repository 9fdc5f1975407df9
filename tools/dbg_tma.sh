mkdir -p gpurun_out
for a in "0 256 -8 1 0" "0 256 8 1 0" "0 256 3 1 0" "0 8 -8 0 0"; do ./tools/tma_probe $a; done
python tools/dbg_tma.py i16; python tools/dbg_tma.py f32
bash tools/v1.sh
