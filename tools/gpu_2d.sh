#!/bin/bash
# 2-D / slabs parity + benches, and an ncu capture of the non-uniform advection kernel.
O=gpurun_out/twod
mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for w in C6 C6NU C6F32 C4M C2; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err
done
for mb in 0 24 96; do
  SB_2D_CHUNK_MB=$mb timeout 300 python bench.py --workload C6 --no-cpu-baseline --no-e2e > $O/bench_C6_chunk$mb.json 2> $O/bench_C6_chunk$mb.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_ADVNU -f \
      python tools/prof_run.py --workload ADVNU --n 3 > $O/prof_ADVNU.log 2>&1
tail -3 $O/pytest.log
for f in $O/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', '%.4g'%d['value'], d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3), d.get('e2e') and '%.3g'%d['e2e']['value'])" 2>/dev/null || echo "$f failed"; done
