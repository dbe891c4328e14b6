#!/bin/bash
# quick bench lines (no cpu baseline / e2e) for the workloads in $WL
for w in ${WL:-C2}; do
  python bench.py --workload $w --no-cpu-baseline --no-e2e ${ARGS} 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.readline())
print('$w', 'ms=%.4f'%d['ms_per_step'], 'GB/s=%.0f'%d['achieved_gbs'], 'frac=%.3f'%d['roofline']['frac'], 'sm=%s'%d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done
