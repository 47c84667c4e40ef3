for sp in 0 2 4; do
  LMO_LIB=build/variants/nomerge.so SPLITS=$sp python scripts/step_vs_attn.py c2 c5 c3 2>&1 | sed "s/^/nomerge sp$sp /" | awk '{print $1, $2, $3, $6, $7}'
done
