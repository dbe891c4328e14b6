#!/bin/bash
# Table V / Fig. 2 sweep (graph-timed, with build-only times) + ncu of the p=4 advection kernels
O=gpurun_out/r7
mkdir -p $O
timeout 900 python tools/table5.py --steps 20 --out $O/table5.jsonl > $O/table5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_ADVNU_p4 -f \
      python tools/prof_run.py --workload ADVNU --degree 4 --n 3 > $O/prof_ADVNU_p4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sb_warp -s 2 -c 1 -o $O/prof_ADV_p4 -f \
      python tools/prof_run.py --workload ADV --degree 4 --n 3 > $O/prof_ADV_p4.log 2>&1
grep -c figure $O/table5.jsonl
