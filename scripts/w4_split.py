"""Packed W4A16 time vs forced split-K on one shape.  usage: w4_split.py N K B splits..."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
N, K, B = (int(a) for a in sys.argv[1:4])
splits = [int(a) for a in sys.argv[4:]] or [0, 1, 2, 3, 4, 5, 6]
g = torch.Generator(device="cuda"); g.manual_seed(1)
W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
del W, c, m
x = torch.randn(B, K, generator=g, device="cuda").half()
y = torch.empty(B, N, device="cuda")
for s in splits:
    for _ in range(3):
        lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y, k_split=s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(30):
        lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y, k_split=s)
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / 30
    print(f"{N}x{K} B{B} split {s}: {us:.1f} us  {N * K * 0.5625 / us / 1e3:.0f} GB/s")
