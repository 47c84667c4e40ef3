"""NEXT-3 perf probe: lmo_w4a16_linear on the OPT-30B (config 3) layer GEMMs at
batch 64, vs dequantize (A5) + torch fp16 matmul.  usage: w4a16_perf.py [SPLIT]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo

split = int(sys.argv[1]) if len(sys.argv) > 1 else 0
PACKED = os.environ.get("PACKED", "1") == "1"
h1, B = 7168, 64
shapes = {"qkv": (3 * h1, h1), "o": (h1, h1), "ffn1": (4 * h1, h1), "ffn2": (h1, 4 * h1)}
tot_t = tot_b = 0
for name, (N, K) in shapes.items():
    W = (torch.randn(N, K, device="cuda") * 0.02).half()
    codes, meta = lmo.lmo_quantize_groupwise(W, N, K, 1)
    codes, meta = codes.view(N, K // 2), meta.view(N, K // 64)
    packed = lmo.lmo_w4a16_pack(codes, meta, N, K) if PACKED else None
    x = torch.randn(B, K, device="cuda").half()
    y = torch.empty(B, N, device="cuda")
    nrep = 20
    # several weight copies would exceed nothing here: one layer's weights >> L2 per GEMM for qkv/ffn
    for _ in range(3):
        (lmo.lmo_w4a16_linear_packed(packed, N, K, x, y=y, k_split=split) if PACKED else lmo.lmo_w4a16_linear(codes, meta, N, K, x, y=y, k_split=split))
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(nrep):
        (lmo.lmo_w4a16_linear_packed(packed, N, K, x, y=y, k_split=split) if PACKED else lmo.lmo_w4a16_linear(codes, meta, N, K, x, y=y, k_split=split))
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / nrep
    by = N * K * 0.5 + N * (K // 64) * 4 + B * K * 2 + B * N * 4
    fl = 2.0 * B * N * K
    # baseline: dequantize to fp16 (A5) + cuBLAS fp16 GEMM
    Wd = torch.empty(N, K, device="cuda", dtype=torch.float16)
    def base():
        lmo.lmo_dequantize_groupwise(codes, meta, N, K, 1, y=Wd.view(N, K, 1))
        return torch.matmul(x, Wd.t())
    for _ in range(3):
        base()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(nrep):
        base()
    e1.record(); torch.cuda.synchronize()
    bus = e0.elapsed_time(e1) * 1e3 / nrep
    tot_t += us; tot_b += by
    print(f"{name:5s} N={N} K={K}: {us:7.1f} us  {by/us/1e3:6.0f} GB/s ({by/us/1e3/6552*100:4.1f}% HBM)  "
          f"{fl/us/1e6:6.0f} TFLOP/s | dequant+cuBLAS {bus:7.1f} us ({bus/us:.2f}x)", flush=True)
    del W, Wd
print(f"layer: {tot_t:.1f} us, {tot_b/tot_t/1e3:.0f} GB/s ({tot_b/tot_t/1e3/6552*100:.1f}% of 6552)")
