for sp in 0 2 4; do for c in c2 c5 c3; do
  r=$(python bench.py --config $c --splits $sp --steps 20 --warmup 3 --no-e2e --no-stream --no-offload --cpu-sample-seconds 0.2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), 'tok/s attn', round(d['roofline']['per_launch_us'],1), 'us frac', round(d['roofline']['frac'],3))")
  echo "splits=$sp $c $r"
done; done
