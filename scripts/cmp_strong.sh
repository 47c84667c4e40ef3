for sp in 0 1 2 4; do
  SPLITS=$sp python scripts/step_vs_attn.py c4:8 c4:16 c4:32 c5:16 c5:32 c5:64 c2:4 c2:8 c2:16 2>&1 | sed "s/^/sp$sp /" | awk '{print $1, $2, $5, $6, $7, $8}'
done
