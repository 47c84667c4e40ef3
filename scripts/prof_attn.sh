#!/bin/bash
# usage: scripts/prof_attn.sh TAG CONFIG[:LEN]...  (ncu --set full of one attention launch per config,
# at LEN = the bench's mid length s + t_mid when given)
TAG=${1:-x}; shift
mkdir -p gpurun_out
for SPEC in "$@"; do
CFG=${SPEC%%:*}; LEN=0; [ "$SPEC" != "$CFG" ] && LEN=${SPEC##*:}
LEN=$LEN REPS=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:decode_attn -s 3 -c 1 \
  -o gpurun_out/prof_${CFG}_${TAG} -f python scripts/attn_perf.py $CFG > gpurun_out/ncu_${CFG}_${TAG}.log 2>&1
tail -2 gpurun_out/ncu_${CFG}_${TAG}.log
done
