#!/bin/bash
# usage (GPU box): scripts/cmp_variants.sh "c2 c5 c3 c4" v1 v2 ...  (default build = "base")
CFGS=$1; shift
for rep in 1 2; do
for v in base "$@"; do
  lib=build/variants/$v.so; [ $v = base ] && lib=""
  LMO_LIB=$lib python scripts/step_vs_attn.py $CFGS 2>&1 | sed "s/^/$v /" | awk '{print $1, $2, $5, $6, $7, $8}'
done; done
