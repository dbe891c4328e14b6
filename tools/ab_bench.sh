#!/bin/bash
# A/B: alternate env settings within one session, REPS rounds each
for rep in $(seq ${REPS:-2}); do
  for w in ${WL:-C2}; do
    for envs in "${ENVA:-X=0}" "${ENVB:-X=1}"; do
      echo -n "$envs "; env $envs WL=$w bash tools/quick_bench.sh
    done
  done
done
