"""Per-shape W4A16 (packed) time vs forced k_split (0 = auto) for a config's four
weight shapes.  usage: w4_splits.py [config] [splits,...]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo, configs as C
w = C.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c5"]
splits = [int(s) for s in (sys.argv[2] if len(sys.argv) > 2 else "0,1,2,3,4,6").split(",")]
h = w.hidden
shapes = [(3 * h, h), (h, h), (4 * h, h), (h, 4 * h)]
g = torch.Generator(device="cuda"); g.manual_seed(1)
tot = {s: 0.0 for s in splits}
for N, K in shapes:
    W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
    c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
    pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
    del W, c, m
    x = torch.randn(w.batch, K, generator=g, device="cuda").half()
    y = torch.empty(w.batch, N, device="cuda")
    row = []
    for s in splits:
        for _ in range(3):
            lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y, k_split=s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record()
        for _ in range(20):
            lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y, k_split=s)
        e1.record(); torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / 20
        tot[s] += us
        row.append(f"s{s}:{us:.1f}")
    print(f"  {N}x{K}: " + " ".join(row))
print(w.name, " ".join(f"s{s}:{v:.1f}" for s, v in tot.items()))
