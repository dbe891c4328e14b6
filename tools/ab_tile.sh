#!/bin/bash
# A/B of builds of the library on tile-kernel workloads: bench lines (no CPU
# baseline / e2e) for each workload in $WL with the shipped library ("main")
# and with each variant libsb_<name>.so named in $LIBS (tools/build_variant.py).
O=gpurun_out/${O:-ab}
mkdir -p $O
for w in ${WL:-C2 C3G C3H}; do
  timeout ${BENCH_TIMEOUT:-180} python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/main_$w.json 2> $O/main_$w.err
  for v in $LIBS; do
    SB_LIB_PATH=$PWD/paper_conf_sc_asahilbpbgo24_b200/libsb_$v.so timeout ${BENCH_TIMEOUT:-180} python bench.py --workload $w --no-cpu-baseline --no-e2e \
      > $O/${v}_$w.json 2> $O/${v}_$w.err
  done
done
for f in $O/*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', round(d['ms_per_step'],4), round(d['roofline']['frac'],3), d['clocks']['reasons'])" 2>/dev/null || echo "$f failed"; done
