#!/bin/bash
# A/B of smiler_knn_opts.variant values on one config (same box, alternating runs).
#   tools/ab_variant.sh <out_dir> <config> <dtype> <variant_a> <variant_b> [rounds]
O=$1; C=$2; T=$3; A=$4; B=$5; R=${6:-2}
mkdir -p $O
for r in $(seq 1 $R); do
  for v in $A $B; do
    SMILER_AB=$v timeout 600 python bench.py --config $C --dtype $T --no-cpu --no-e2e --two-level-steps 0 \
        > $O/ab_${C}_${T}_v${v}_r${r}.json 2> $O/ab_${C}_${T}_v${v}_r${r}.err
    python -c "import json,sys; d=json.load(open('$O/ab_${C}_${T}_v${v}_r${r}.json')); print('$C $T variant $v round $r: %.1f MQ/s %.3f ms/step' % (d['value'], d['ms_per_step']), 'phases', {k: round(x,3) for k,x in d['phase_ms_per_step'].items()}, 'clk', d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'))"
  done
done
