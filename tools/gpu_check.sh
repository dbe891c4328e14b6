#!/bin/bash
# Quick GPU check: parity tests, smoke, default bench line.
O=gpurun_out/check
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.limit --format=csv > $O/gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err
for w in ${EXTRA_WORKLOADS}; do
  timeout 600 python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err
done
cp MEASURED_PEAKS.json $O/ 2>/dev/null
tail -3 $O/pytest_gpu.log; tail -2 $O/smoke.log; cat $O/bench_C2.json
