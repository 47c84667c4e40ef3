#!/bin/bash
# usage (GPU box): CFGS="c4 c5" scripts/attn_sweep.sh v1 v2 ...   attention-only timings per build/variants/<v>.so
for v in "$@"; do echo "=== $v"; LMO_LIB=build/variants/$v.so python scripts/attn_perf.py ${CFGS:-c2 c3 c5 c4}; done
