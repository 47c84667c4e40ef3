mkdir -p gpurun_out
for v in default c8 c4 c8s3; do
  lib=build/variants/$v.so; [ $v = default ] && lib=""
  echo "== $v"; LMO_LIB=$lib timeout 300 python scripts/w4_check.py 28672 7168 64 3 2>&1 | tail -3
done
echo "== synccheck c8"
LMO_LIB=build/variants/c8.so timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python scripts/w4_check.py 28672 7168 64 1 > gpurun_out/w4_synccheck_c8.log 2>&1; tail -30 gpurun_out/w4_synccheck_c8.log
echo "== racecheck c8"
LMO_LIB=build/variants/c8.so timeout 1200 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python scripts/w4_check.py 28672 7168 64 1 > gpurun_out/w4_racecheck_c8.log 2>&1; tail -40 gpurun_out/w4_racecheck_c8.log
