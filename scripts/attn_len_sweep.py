"""Attention launch time vs length at a fixed (B, H, d): fixed overhead vs per-token cost."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
B, H, G, d = [int(x) for x in (sys.argv[1:5] if len(sys.argv) > 4 else (32, 32, 1, 128))]
cap = 4096
nl = max(2, int(3e9 // (B * H * cap * 144)))
caches = []
for l in range(nl):
    c = lmo.KVCache.empty(B, H, cap, d)
    c.kv.random_(0, 256)
    for nm in ("k_meta", "v_meta"):
        c.field(nm).view(torch.int32).fill_(0x2C00BC00)
    caches.append(c)
abis = [c.abi() for c in caches]
q = torch.randn(B, H * G, d, device='cuda').half()
out = torch.empty(B, H * G, d, device='cuda')
ws = lmo.attention_workspace(B, H, H * G, d)
Ls = [int(x) for x in os.environ.get("LENS", "16,32,64,128,256,512,1024,2048,4096").split(",")]
st = torch.cuda.Stream()
for L in Ls:
    g = torch.cuda.CUDAGraph()          # graph: no host launch overhead in the timing
    with torch.cuda.graph(g, stream=st):
        for l in range(nl):
            lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l])
    g.replay(); g.replay(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 10
    e0.record()
    for it in range(reps):
        g.replay()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (reps * nl)
    by = B * H * L * 144 + B * H * G * d * 6
    print(f"B={B} H={H} G={G} L={L:5d}: {ms*1e3:7.1f} us  {by/ms/1e6:6.0f} GB/s ({by/ms/1e6/6551*100:4.1f}%)", flush=True)
