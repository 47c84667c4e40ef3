#!/bin/bash
# Attention-only timing per scheduling mode (LMO_ATTN_SCHED), then a timeline build.
# usage: scripts/sched_sweep.sh   (on the GPU box)
for s in team1 team2 team4 streamk; do
  echo "=== $s"; LMO_ATTN_SCHED=$s python scripts/attn_perf.py c2 c3 c5 c4
done
