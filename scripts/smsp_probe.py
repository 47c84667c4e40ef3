"""Per-SMSP throughput of the attention kernel vs busy warps per SMSP.
pairs = 592*k (B = 16k, Hkv = 37, MHA, d = 128), team size 1 -> k busy warps per
SMSP; two lengths -> the per-stage slope (head/tail removed).  MODE=l2: one cache
(L2-resident for small k); MODE=hbm: several caches (> L2).
usage: smsp_probe.py [k ...]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo

ks = [int(a) for a in sys.argv[1:]] or [1, 2, 3, 4]
mode = os.environ.get("MODE", "hbm")
splits = int(os.environ.get("SPLITS", "1"))
G = int(os.environ.get("G", "1"))
reps = 20
clk = 1.965e3   # cycles per us
for k in ks:
    B, H = 16 * k, 37
    res = {}
    for L in (256, 768):
        cap = L + 16
        nbytes = B * H * cap * 144
        nl = 1 if mode == "l2" else max(2, int(4e8 // nbytes) + 1)
        caches = []
        for _ in range(nl):
            c = lmo.KVCache.empty(B, H, cap, 128)
            c.kv.random_(0, 256)
            for nm in ("k_meta", "v_meta"):
                c.field(nm).view(torch.int32).fill_(0x2C00BC00)
            caches.append(c)
        q = torch.randn(B, H * G, 128, device='cuda').half()
        out = torch.empty(B, H * G, 128, device='cuda')
        ws = lmo.attention_workspace(B, H, H * G, 128, splits)
        abis = [c.abi() for c in caches]
        st = torch.cuda.Stream()
        def run():
            for l in range(nl):
                lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l],
                                            num_splits=splits, stream=st)
        with torch.cuda.stream(st):
            run()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(4):
                run()
        g.replay(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(st):
            e0.record(st)
            for _ in range(reps):
                g.replay()
            e1.record(st)
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / (reps * 4 * nl)
        res[L] = us
        del caches
    d_st = (768 - 256) / 32 * k                      # extra stages per SMSP
    slope = (res[768] - res[256]) / d_st             # us per stage per SMSP
    gbs = B * H * 768 * 144 / res[768] / 1e3
    print(f"{mode} G={G} k={k}: L256 {res[256]:.1f} us  L768 {res[768]:.1f} us ({gbs:.0f} GB/s)  "
          f"slope {slope*1e3:.0f} ns/stage/SMSP = {slope*clk:.0f} cyc  head {res[256] - slope*256/32*k:.1f} us",
          flush=True)
