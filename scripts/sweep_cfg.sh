#!/bin/bash
# Build variants on the GPU box and time attention for each.  usage: sweep_cfg.sh "DEFS1" "DEFS2" ...
for defs in "$@"; do
  echo "=== $defs"
  LMO_NVCC_DEFS="$defs" python -m paper_conf_ipps_wurypgll25_b200.build --force 2>&1 | grep -A1 "decode_attn_q4_kernelILi128" | grep -E "Used|spill" | head -2
  python scripts/attn_perf.py c2 c3 c4 c5
done
python -m paper_conf_ipps_wurypgll25_b200.build --force > /dev/null 2>&1
