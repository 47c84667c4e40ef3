#!/bin/bash
# usage (GPU box): CFGS="c2 c5" scripts/bench_variants.sh v1 v2 ...   short bench.py runs per build/variants/<v>.so
for v in "$@"; do for c in ${CFGS:-c2 c5}; do
  r=$(LMO_LIB=build/variants/$v.so python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-stream --no-offload --cpu-sample-seconds 0.2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), 'tok/s attn', round(d['roofline']['per_launch_us'],1), 'us frac', round(d['roofline']['frac'],3))")
  echo "$v $c $r"
done; done
