#!/bin/bash
# full GPU parity + the main bench lines + Table V / Fig. 2 sweep
O=gpurun_out/r3
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for w in C2 C1 C3G C3H C4 C4F32 C4M ADV ADVNU C6 C6NU; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 900 python tools/table5.py --steps 20 --out $O/table5.jsonl > $O/table5.log 2>&1
tail -2 $O/pytest.log; tail -1 $O/smoke.log
for f in $O/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', '%.4g'%d['value'], d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3))" 2>/dev/null || echo "$f failed"; done
