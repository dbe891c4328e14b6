#!/bin/bash
# ADVNU occupancy check, C3G ncu capture (source-level), Table V / Fig. 2 sweep.
O=gpurun_out/r2
mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q -k "advect or point_contiguous or strided" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for w in ADVNU ADV C4 C4F32; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 900 python tools/table5.py --steps 20 --out $O/table5.jsonl > $O/table5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_tile -s 2 -c 1 -o $O/prof_C3G -f \
      python tools/prof_run.py --workload C3G --n 3 > $O/prof_C3G.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_ADVNU -f \
      python tools/prof_run.py --workload ADVNU --n 3 > $O/prof_ADVNU.log 2>&1
tail -2 $O/pytest.log
for f in $O/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', round(d['value'],2), d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3))" 2>/dev/null || echo "$f failed"; done
