# build libsmiler.so variants into _build/var/<name>.so: name=flags pairs.
# smiler.cu (with kernels.cuh / lb.cuh) and dtw.cu are recompiled with the extra
# flags; predict.o is the current build's.
set -e
cd "$(dirname "$0")/.."
P=paper_conf_sigmod_zhout15_b200
python -c "from $P.build import build; build()" > /dev/null
mkdir -p $P/_build/var
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -I include"
pids=()
for spec in "$@"; do
  name=${spec%%=*}; flags=${spec#*=}
  ( $NV $flags -c $P/csrc/smiler.cu -o $P/_build/var/$name.o && \
    $NV $flags -c $P/csrc/dtw.cu -o $P/_build/var/${name}_dtw.o && \
    $NV -shared -cudart static -o $P/_build/var/$name.so $P/_build/var/$name.o $P/_build/var/${name}_dtw.o $P/_build/predict.o && \
    rm $P/_build/var/$name.o $P/_build/var/${name}_dtw.o && echo "built $name: $flags" ) &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
