for rep in 1 2; do
for cap in 0 444 296; do
  LMO_LIB=build/variants/exp.so LMO_ATTN_MAX_CTAS=$cap python scripts/step_vs_attn.py c2 c5 c3 c4 2>&1 | sed "s/^/cap$cap /" | awk '{print $1, $2, $5, $6, $7, $8}'
done; done
