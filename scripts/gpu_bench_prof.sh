#!/bin/bash
# usage: scripts/gpu_bench_prof.sh CONFIG TAG   (run on the GPU box under gpurun)
CFG=${1:-c2}; TAG=${2:-r1}
mkdir -p gpurun_out
python bench.py --config $CFG --steps 20 --warmup 3 > gpurun_out/bench_${CFG}_${TAG}.json 2> gpurun_out/bench_${CFG}_${TAG}.err
tail -c 4000 gpurun_out/bench_${CFG}_${TAG}.json
# launch list of a short bench (graph-replayed kernels are profiled per node; cold-cache, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_${TAG}.csv \
   python bench.py --config $CFG --steps 2 --warmup 3 --no-e2e --cpu-sample-seconds 0.1 > /dev/null 2>&1
# one full capture of the dominant kernel inside the bench
timeout 900 ncu --set full --clock-control none --import-source on -k regex:decode_attn -s 200 -c 1 \
   -o gpurun_out/prof_${CFG}_${TAG} -f python bench.py --config $CFG --steps 2 --warmup 3 --no-e2e --cpu-sample-seconds 0.1 > gpurun_out/ncu_${CFG}_${TAG}.log 2>&1
tail -2 gpurun_out/ncu_${CFG}_${TAG}.log
