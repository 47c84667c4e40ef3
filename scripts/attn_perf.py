"""Attention-only perf probe: random q4 caches of a config's shape, several
layers (footprint > L2), CUDA-event timing per launch.  usage: attn_perf.py c2 [c5 ...]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS, attention_launch_bytes

keys = [a for a in sys.argv[1:] if not a.startswith('-')] or ["c2"]
reps = int(os.environ.get("REPS", "10"))
splits = int(os.environ.get("SPLITS", "0"))
for key in keys:
    w = CONFIGS[key]
    nl = max(2, min(16, int(2.0e9 // (w.batch * w.kv_heads * w.capacity * 144))))
    caches = []
    L = int(os.environ.get("LEN", "0")) or w.max_len   # LEN: the bench's mid length s + t_mid
    for l in range(nl):
        c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
        c.kv.random_(0, 256)
        for nm in ("k_meta", "v_meta"):
            c.field(nm).view(torch.int32).fill_(0x2C00BC00)   # min -1.0, scale 1/16
        caches.append(c)
    q = torch.randn(w.batch, w.q_heads, w.head_dim, device='cuda').half()
    out = torch.empty(w.batch, w.q_heads, w.head_dim, device='cuda')
    ws = lmo.attention_workspace(w.batch, w.kv_heads, w.q_heads, w.head_dim, splits)
    abis = [c.abi() for c in caches]
    for it in range(2):
        for l in range(nl):
            lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l], num_splits=splits)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for it in range(reps):
        for l in range(nl):
            lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l], num_splits=splits)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (reps * nl)
    by = attention_launch_bytes(w, L)
    print(f'{key} L={L} layers={nl}: attn {ms*1e3:.1f} us/launch, {by/ms/1e6:.0f} GB/s ({by/ms/1e6/6551*100:.1f}% of 6551)', flush=True)
    del caches
