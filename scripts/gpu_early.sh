# fused-step time vs the number of stages streamed before griddepcontrol.wait (experiments build)
for d in 0 1 2 3; do echo "== early depth $d"; LMO_LIB=build/variants/exp.so LMO_EARLY_DEPTH=$d python scripts/step_vs_attn.py $@ 2>&1 | awk '{print $1, $4, $5, $6, $7, $8, $9}'; done
