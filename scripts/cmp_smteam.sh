for v in base sm8 sm12; do
  lib=build/variants/$v.so; [ $v = base ] && lib=""
  for sp in 0 -2; do
    LMO_LIB=$lib SPLITS=$sp python scripts/step_vs_attn.py c2 c5 c3 c4 2>&1 | sed "s/^/$v sp$sp /" | awk '{print $1, $2, $3, $6, $7, $8, $9}'
  done
done
