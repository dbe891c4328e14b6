#!/bin/bash
# Advection A/B: parity tests of the advect path, then ADV / ADVNU / C4 under each warp-kernel loader.
O=gpurun_out/adv
mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q -k "advect or point_contiguous or 2d" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for b in auto 1 0; do
  for w in ADV ADVNU C4; do
    if [ $b = auto ]; then unset SB_WARP_BULK; else export SB_WARP_BULK=$b; fi
    timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_${w}_$b.json 2> $O/bench_${w}_$b.err
  done
done
unset SB_WARP_BULK
timeout 300 python bench.py --workload C6 --no-cpu-baseline --no-e2e > $O/bench_C6.json 2> $O/bench_C6.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_ADVNU -f \
      python tools/prof_run.py --workload ADVNU --n 3 > $O/prof_ADVNU.log 2>&1
tail -2 $O/pytest.log
for f in $O/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', round(d['value'],2), d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3))" 2>/dev/null || echo "$f failed"; done
