for sp in 0 1 2 4; do
  SPLITS=$sp python scripts/step_vs_attn.py c2 c5 c3 c4 2>&1 | sed "s/^/sp$sp /" | awk '{print $1, $2, $5, $6, $7, $8}'
done
