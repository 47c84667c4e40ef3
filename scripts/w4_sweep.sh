#!/bin/bash
# usage (GPU box): [PACKED=0|1] [SPLIT=s] scripts/w4_sweep.sh v1 v2 ...   W4A16 layer timings per build/variants/<v>.so
for v in "$@"; do echo "=== $v"; LMO_LIB=build/variants/$v.so python scripts/w4a16_perf.py ${SPLIT:-0}; done
