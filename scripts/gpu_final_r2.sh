# round-2 evidence run: ncu captures, launch list, bench lines for every config, reference arm
mkdir -p gpurun_out
TAG=${TAG:-r2b}
bash scripts/prof_attn.sh $TAG c4:528 c2:528 c5:1088 c3:128
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_c4_$TAG.csv python bench.py --steps 2 --warmup 1 --no-stream --no-offload --no-e2e --cpu-sample-seconds 1 > gpurun_out/launches_bench.log 2>&1
for cfg in c4 c2 c5 c3 c1; do
  timeout 900 python bench.py --config $cfg > gpurun_out/bench_${cfg}_$TAG.json 2> gpurun_out/bench_${cfg}_$TAG.err
  echo "$cfg rc=$?"; tail -c 400 gpurun_out/bench_${cfg}_$TAG.json; echo
done
timeout 900 python bench.py --impl reference > gpurun_out/ref_c4_$TAG.json 2> gpurun_out/ref_c4_$TAG.err; echo "ref rc=$?"
