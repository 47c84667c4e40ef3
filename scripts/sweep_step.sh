#!/bin/bash
# Build variants on the GPU box and time the fused decode step for each.
# usage: sweep_step.sh "CFGS" "DEFS1" "DEFS2" ...   (CFGS e.g. "c2 c3 c5 c4")
cfgs=$1; shift
for defs in "$@"; do
  echo "=== $defs"
  LMO_NVCC_DEFS="$defs" python -m paper_conf_ipps_wurypgll25_b200.build --force > /dev/null 2>&1 || echo BUILD FAILED
  python scripts/step_perf.py $cfgs
done
python -m paper_conf_ipps_wurypgll25_b200.build --force > /dev/null 2>&1
