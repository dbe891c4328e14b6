#!/bin/bash
# usage: tools/gpu_run.sh OUTDIR "W1 W2 ..." [pytest-k-expr]
# GPU parity (all or -k), smoke, bench lines for the given workloads (no cpu baseline / e2e).
O=gpurun_out/$1
mkdir -p $O
if [ -n "$3" ]; then K=(-k "$3"); else K=(); fi
timeout 1500 python -m pytest tests -m gpu -x -q "${K[@]}" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for w in $2; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_$w.json 2> $O/bench_$w.err
done
tail -2 $O/pytest.log; tail -1 $O/smoke.log
for f in $O/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', '%.4g'%d['value'], d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3))" 2>/dev/null || echo "$f failed"; done
