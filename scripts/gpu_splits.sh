# bench step / attention vs explicit team size (num_splits 1/2/4) and auto (0): scripts/gpu_splits.sh "<cfgs>"
for cfg in $1; do for sp in 0 1 2 4; do
  r=$(timeout 600 python bench.py --config $cfg --splits $sp --no-stream --no-offload --no-e2e --cpu-sample-seconds 1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), round(d['roofline']['per_launch_us'],2), d['clocks']['sm_mhz'])")
  echo "$cfg splits=$sp $r"
done; done
