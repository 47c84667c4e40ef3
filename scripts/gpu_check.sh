#!/bin/bash
# GPU-box helper: parity tests + short bench lines for new vs reference builds.
#   scripts/gpu_check.sh "<pytest selection>" "<configs>" [alt_lib ...]
mkdir -p gpurun_out
SEL=${1:-tests}
CFGS=${2:-"c2 c5 c4"}
shift 2
python -c "import torch; print(torch.cuda.get_device_name(0))"
if [ "$SEL" != "none" ]; then
  timeout 1500 python -m pytest $SEL -m gpu -q -rf -s 2>&1 | tee gpurun_out/pytest.log | grep -v "^\[parity\]" | tail -40
  grep "^\[parity\]" gpurun_out/pytest.log | sort -t' ' -k5 | tail -5
fi
for cfg in $CFGS; do
  for lib in "" "$@"; do
    LMO_LIB=$lib timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-stream --no-offload --no-e2e --cpu-sample-seconds 1 > gpurun_out/bench_${cfg}_$(basename ${lib:-new}).json 2>gpurun_out/bench_err.log
    python - "$cfg" "${lib:-new}" gpurun_out/bench_${cfg}_$(basename ${lib:-new}).json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[3]).read().strip().splitlines()[-1])
    r = d["roofline"]
    print(f"{sys.argv[1]} {sys.argv[2]:28s} step {d['value']:9.0f} tok/s {d['ms_per_step']:.3f} ms | attn {r['per_launch_us']:.1f} us frac {r['frac']:.3f} | clocks {d['clocks']['sm_mhz']} {d['clocks']['reasons']}")
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", e)
PY
  done
done
