#!/bin/bash
# The default bench command (as the driver runs it) with its wall time and a summary of every extra workload
mkdir -p gpurun_out/fb
t0=$(date +%s)
timeout 800 python bench.py > gpurun_out/fb/bench_C2.json 2> gpurun_out/fb/bench_C2.err
echo "rc=$? wall=$(( $(date +%s) - t0 )) s"
python3 - <<'PY'
import json
d=json.loads(open("gpurun_out/fb/bench_C2.json").read().strip().splitlines()[-1])
print(d["ms_per_step"], d["roofline"]["frac"], d["e2e"]["value"], d["clocks"])
for w,v in d["extra_workloads"].items(): print(w, round(v.get("ms_per_step",0),4), v.get("kernel"), v.get("error"))
PY
