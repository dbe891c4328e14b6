#!/bin/bash
# A/B of environment settings on bench workloads: for each workload in $WL and
# each setting in $ENVS (";"-separated, e.g. "SB_TILE_GMODE=0;SB_TILE_GMODE=2"),
# one bench line (no CPU baseline / e2e); prints ms/step and the kernel.
O=gpurun_out/${O:-abenv}
mkdir -p $O
IFS=';' read -ra SETS <<< "${ENVS:-X=0}"
for w in ${WL:-C2 C3G C3H}; do
  for e in "${SETS[@]}"; do
    tag=$(echo "$e" | tr ' =/' '___' | cut -c1-60)
    timeout ${BENCH_TIMEOUT:-180} env $e python bench.py --workload $w --no-cpu-baseline --no-e2e ${BENCH_ARGS} > $O/${w}_$tag.json 2> $O/${w}_$tag.err
    python -c "
import json; d=json.load(open('$O/${w}_$tag.json')); print('$w', '$e', round(d['ms_per_step'],4), round(d['roofline']['frac'],3), d['config'].get('kernel'), d['clocks']['reasons'])" 2>/dev/null || echo "$w $e failed"
  done
done
