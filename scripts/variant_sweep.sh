#!/bin/bash
# usage (GPU box): scripts/variant_sweep.sh v1 v2 ...  -> attention/step timings per build/variants/<v>.so
for v in "$@"; do
  echo "=== $v"
  export LMO_LIB=build/variants/$v.so
  python scripts/smsp_probe.py ${PROBE_KS:-1 2 6}
  python scripts/attn_perf.py ${CFGS:-c2 c3 c5}
  python scripts/step_perf.py ${CFGS:-c2 c3 c5}
done
