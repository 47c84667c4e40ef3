#!/bin/bash
# usage (GPU box): scripts/team_sweep.sh VARIANT -> attention + step timings for team sizes 1, 2, 4
export LMO_LIB=build/variants/$1.so
for s in team1 team2 team4; do
  echo "=== $1 $s"
  LMO_ATTN_SCHED=$s python scripts/attn_perf.py ${CFGS:-c2 c3 c5 c4}
  LMO_ATTN_SCHED=$s python scripts/step_perf.py ${CFGS:-c2 c3 c5}
done
