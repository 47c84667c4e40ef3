#!/bin/bash
# usage: scripts/bench_all.sh TAG CONFIG...   (GPU box) -> gpurun_out/bench_<cfg>_<TAG>.json + summary
TAG=$1; shift
mkdir -p gpurun_out
for c in "$@"; do
  t0=$(date +%s)
  timeout 900 python bench.py --config $c --steps 20 --warmup 3 > gpurun_out/bench_${c}_${TAG}.json 2> gpurun_out/bench_${c}_${TAG}.err
  echo "$c rc=$? $(( $(date +%s) - t0 )) s"
  python - "$c" "$TAG" <<'PY'
import json, sys
c, tag = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/bench_{c}_{tag}.json"))
except Exception as e:
    print(c, "no line:", e); sys.exit(0)
r = d["roofline"]; s = d.get("streaming") or {}
print(c, round(d["value"]), "tok/s frac", round(r["frac"], 3), "attn us", round(r["per_launch_us"], 1),
      "step GB/s", round(d["achieved_gbs"]), "e2e", round(d["e2e"]["value"]),
      "A1", round(s.get("quantize_A1", {}).get("GB/s", 0)), "A5", round(s.get("dequantize_A5", {}).get("GB/s", 0)),
      "cpu", d["cpu_baseline"] and d["cpu_baseline"].get("value"), d["clocks"]["reasons"])
PY
done
