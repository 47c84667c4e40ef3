#!/bin/bash
# usage: scripts/gpu_bench_prof.sh CONFIG TAG   (run on the GPU box under gpurun)
set -x
CFG=${1:-c2}; TAG=${2:-r1}
mkdir -p gpurun_out
python bench.py --config $CFG --steps 20 --warmup 3 > gpurun_out/bench_${CFG}_${TAG}.json 2> gpurun_out/bench_${CFG}_${TAG}.err
tail -c 3000 gpurun_out/bench_${CFG}_${TAG}.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_${TAG}.csv \
   python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --cpu-sample-seconds 0.1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:decode_attn -s 40 -c 2 \
   -o gpurun_out/prof_${CFG}_${TAG} -f python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --cpu-sample-seconds 0.1 > gpurun_out/ncu_${CFG}_${TAG}.log 2>&1
ls -la gpurun_out
