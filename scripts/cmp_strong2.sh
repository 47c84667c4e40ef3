for v in base ringonly; do
lib=build/variants/$v.so; [ $v = base ] && lib=""
for sp in 2 4; do
  LMO_LIB=$lib SPLITS=$sp python scripts/step_vs_attn.py c4:8 c4:16 c5:16 c5:32 c5:64 c2:4 c2:8 c2:16 2>&1 | sed "s/^/$v sp$sp /" | awk '{print $1, $2, $3, $6, $7, $8, $9}'
done; done
