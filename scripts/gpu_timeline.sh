mkdir -p gpurun_out
for a in "32 32 1 528" "64 56 1 128" "128 8 8 1088"; do
  echo "=== $a"; LMO_LIB=build/variants/prof.so timeout 300 python scripts/attn_timeline.py $a step 2>&1 | tail -32
done > gpurun_out/timeline_r2d.txt 2>&1
