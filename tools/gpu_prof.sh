#!/bin/bash
# ncu --set full of the solve kernel for each workload in $WL (one launch each)
mkdir -p gpurun_out
for w in ${WL:-C2}; do
  ncu --set full --clock-control none --import-source on -k regex:sb_ -s 2 -c 1 -o gpurun_out/prof_${w}${TAG} -f \
      python tools/prof_run.py --workload $w --n 3 > gpurun_out/prof_${w}.log 2>&1
done
