"""Fused decode-step perf probe (append + attention, LMO_STEP_CACHE_STABLE, PDL),
back-to-back layers captured in one CUDA graph like bench.py; random q4 caches of
a config's shape (footprint > L2).  usage: step_perf.py c2 [c5 ...]
Env: REPS, LEN (default: the config's mid length)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS, attention_launch_bytes

keys = [a for a in sys.argv[1:] if not a.startswith('-')] or ["c2"]
# custom shape: SHAPE=B,Hkv,G,L (head_dim 128) replaces the config list
if os.environ.get("SHAPE"):
    import dataclasses
    B_, H_, G_, L_ = [int(x) for x in os.environ["SHAPE"].split(",")]
    CONFIGS = dict(CONFIGS)
    CONFIGS["custom"] = dataclasses.replace(CONFIGS["c2"], batch=B_, kv_heads=H_, q_heads=H_ * G_, prompt=L_, gen=2)
    keys = ["custom"]
reps = int(os.environ.get("REPS", "10"))
splits = int(os.environ.get("SPLITS", "0"))
for key in keys:
    w = CONFIGS[key]
    L = int(os.environ.get("LEN", "0")) or (w.prompt + w.gen // 2)
    nl = max(3, min(32, int(3.0e9 // (w.batch * w.kv_heads * w.capacity * 144))))
    caches = []
    for l in range(nl):
        c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
        c.kv.random_(0, 256)
        for nm in ("k_meta", "v_meta"):
            c.field(nm).view(torch.int32).fill_(0x2C00BC00)   # min -1.0, scale 1/16
        caches.append(c)
    q = torch.randn(w.batch, w.q_heads, w.head_dim, device='cuda').half()
    kn = torch.randn(w.batch, w.kv_heads, w.head_dim, device='cuda').half()
    vn = torch.randn_like(kn)
    out = torch.empty(w.batch, w.q_heads, w.head_dim, device='cuda')
    ws = lmo.attention_workspace(w.batch, w.kv_heads, w.q_heads, w.head_dim, splits)
    abis = [c.abi() for c in caches]
    st = torch.cuda.Stream()
    def layers():
        for l in range(nl):
            lmo.lmo_decode_step_q4(caches[l], kn, vn, q, L, out=out, workspace=ws, abi=abis[l],
                                   flags=lmo.LMO_STEP_CACHE_STABLE, stream=st, num_splits=splits)
    with torch.cuda.stream(st):
        layers()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        layers()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(st):
        e0.record(st)
        for _ in range(reps):
            g.replay()
        e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (reps * nl)
    by = attention_launch_bytes(w, L)
    print(f'{key} L={L} layers={nl}: step {ms*1e3:.1f} us/layer, {by/ms/1e6:.0f} GB/s '
          f'({by/ms/1e6/6551*100:.1f}% of 6551)', flush=True)
    del caches
