"""Bandwidth of the streaming kernels: A1 quantize (c3 weights, 4h1 x h1 and
h1 x 4h1 matrices), A5 dequantize, A2 append at prefill size (c2 layer)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo

def timeit(fn, reps=20):
    st = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        fn()
    g.replay(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): g.replay()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps

h1 = 7168
n_el = 4 * h1 * h1 + 2 * h1 * 4 * h1           # one OPT-30B layer's weights (616.6 M)
W = torch.randn(n_el // h1, h1, device="cuda").half().mul_(0.02)
codes, meta = lmo.lmo_quantize_groupwise(W, n_el // h1, h1, 1)
y = torch.empty_like(W)
ms = timeit(lambda: lmo.lmo_quantize_groupwise(W, n_el // h1, h1, 1, codes=codes, meta=meta))
by = n_el * (2 + 0.5625)
print(f"A1 quantize  {n_el/1e6:.0f} M el (c3 layer weights, inner groups): {ms*1e3:8.1f} us  {by/ms/1e6:6.0f} GB/s ({by/ms/1e6/6551*100:4.1f}%)")
ms = timeit(lambda: lmo.lmo_dequantize_groupwise(codes, meta, n_el // h1, h1, 1, y=y))
print(f"A5 dequantize {n_el/1e6:.0f} M el: {ms*1e3:8.1f} us  {by/ms/1e6:6.0f} GB/s ({by/ms/1e6/6551*100:4.1f}%)")
# strided quantize_dim (group along the output dim of a [h1, 4h1] matrix)
W2 = torch.randn(h1 // 4, h1, device="cuda").half()
c2_, m2_ = lmo.lmo_quantize_groupwise(W2, 1, h1 // 4, h1)
ms = timeit(lambda: lmo.lmo_quantize_groupwise(W2, 1, h1 // 4, h1, codes=c2_, meta=m2_))
n2 = W2.numel(); by2 = n2 * 2.5625
print(f"A1 quantize strided (inner={h1}) {n2/1e6:.1f} M el: {ms*1e3:8.1f} us  {by2/ms/1e6:6.0f} GB/s")
# prefill append (c2 layer: B=32, H=32, s=512, d=128)
B, H, s, d = 32, 32, 512, 128
cache = lmo.KVCache.empty(B, H, 544, d)
k = torch.randn(B, H, s, d, device="cuda").half(); v = torch.randn_like(k)
ms = timeit(lambda: lmo.lmo_kv_append_quant(cache, k, v, 0))
n3 = 2 * k.numel(); by3 = n3 * 2.5625
print(f"A2 append prefill (c2 layer, {n3/1e6:.0f} M el): {ms*1e3:8.1f} us  {by3/ms/1e6:6.0f} GB/s ({by3/ms/1e6/6551*100:4.1f}%)")
# decode append (1 token)
k1 = torch.randn(B, H, 1, d, device="cuda").half(); v1 = torch.randn_like(k1)
ms = timeit(lambda: lmo.lmo_kv_append_quant(cache, k1, v1, 520), reps=200)
print(f"A2 append decode (c2 layer, 1 token): {ms*1e3:8.2f} us")
