"""A1 quantize + A5 dequantize of one OPT-30B layer's weights (12 h1^2 el), for ncu."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
h1 = 7168
rows, n = 12 * h1, h1
x = (torch.randn((rows, n), device="cuda") * 0.02).half()
codes = torch.empty((rows, n // 2), dtype=torch.uint8, device="cuda")
meta = torch.empty((rows, n // 64), dtype=torch.int32, device="cuda")
y = torch.empty_like(x)
for _ in range(3):
    lmo.lmo_quantize_groupwise(x, rows, n, 1, codes=codes, meta=meta)
    lmo.lmo_dequantize_groupwise(codes, meta, rows, n, 1, y=y)
torch.cuda.synchronize()
print("ok")
