# c2/c3/c4 with the grid capped (experiments build): scripts/gpu_maxctas.sh "<cfgs>" "<caps>"
for cfg in $1; do for cap in $2; do
  r=$(LMO_LIB=build/variants/exp.so LMO_ATTN_MAX_CTAS=$cap timeout 600 python bench.py --config $cfg --no-stream --no-offload --no-e2e --cpu-sample-seconds 1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],4), round(d['roofline']['per_launch_us'],2), d['clocks']['sm_mhz'])")
  echo "$cfg cap=$cap $r"
done; done
