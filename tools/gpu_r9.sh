#!/bin/bash
O=gpurun_out/r9
mkdir -p $O
for c in 0 1; do SB_TILE_CBOX=$c timeout 300 python bench.py --workload C3G --no-cpu-baseline --no-e2e > $O/bench_C3G_cbox$c.json 2>&1; done
timeout 120 ./tools/stream_probe > $O/stream_probe.txt 2>&1
timeout 120 ./tools/stream_probe2 > $O/stream_probe2.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_NUsolve -f \
      python tools/prof_run.py --workload ADVNU --solve --n 3 > $O/prof_NUsolve.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_Usolve_p4 -f \
      python tools/prof_run.py --workload ADV --solve --degree 4 --n 3 > $O/prof_Usolve_p4.log 2>&1
for f in $O/bench_*.json; do python -c "
import json; d=[json.loads(l) for l in open('$f') if l.startswith('{')][-1]; print('$f', '%.4g'%d['value'], d['unit'], round(d['ms_per_step'],4), round(d['roofline']['frac'],3))" 2>/dev/null || echo "$f failed"; done
tail -5 $O/stream_probe.txt
