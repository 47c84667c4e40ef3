"""One packed W4A16 launch on a given shape (for ncu).  usage: w4_one.py N K B [reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
N, K, B = (int(a) for a in sys.argv[1:4])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
g = torch.Generator(device="cuda"); g.manual_seed(1)
W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
del W, c, m
x = torch.randn(B, K, generator=g, device="cuda").half()
y = torch.empty(B, N, device="cuda")
for _ in range(reps):
    lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y)
torch.cuda.synchronize()
