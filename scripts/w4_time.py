"""Per-layer time of the packed W4A16 GEMM on a config's four weight shapes
(events over 50 launches per shape, L2-resident activations, weights > L2).
usage: [LMO_LIB=...] w4_time.py [config]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo, configs as C
w = C.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c3"]
h = w.hidden
shapes = [(3 * h, h), (h, h), (4 * h, h), (h, 4 * h)]
g = torch.Generator(device="cuda"); g.manual_seed(1)
tot = 0.0
for N, K in shapes:
    W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
    c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
    pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
    del W, c, m
    x = torch.randn(w.batch, K, generator=g, device="cuda").half()
    y = torch.empty(w.batch, N, device="cuda")
    for _ in range(5):
        lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(50):
        lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y)
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / 50
    tot += us
    print(f"  {N}x{K}: {us:.1f} us")
print(f"{w.name} layer {tot:.1f} us")
