import math, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import oracle
from paper_conf_ipps_wurypgll25_b200 import inputs as I, lmo
sys.path.insert(0, "tests")
from test_gpu_parity import build_layer, normwise_err
for (B,Hkv,G,d,L,ns) in [(2,1,8,128,4090,0),(2,1,8,128,4090,1),(2,1,1,128,4090,0),(2,1,8,128,1000,0)]:
    seed = 1000 + B*7 + L
    cache, host = build_layer(lmo, B, Hkv, L + (L%3), d, L, seed)
    Hq = Hkv*G
    q = torch.empty((B,Hq,1,d), dtype=torch.float16, device='cuda')
    lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B,Hq,d)
    out = lmo.lmo_decode_attention_q4(cache, q, L, num_splits=ns)
    torch.cuda.synchronize()
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), L, nthreads=8)
    err = normwise_err(out.cpu().numpy(), ref)
    print((B,Hkv,G,d,L,ns), 'err max %.3e mean %.3e' % (err.max(), err.mean()), 'max|ref|', np.abs(ref).max(axis=-1).min())

# ---- first perf probe: c2 shapes, 8 layers of caches (> L2), attention only
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS, attention_launch_bytes
for key in ("c2", "c5", "c3", "c4"):
    w = CONFIGS[key]
    nl = 8
    caches = []
    L = w.max_len
    for l in range(nl):
        c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
        c.kv.random_(0, 256)
        for nm in ("k_meta", "v_meta"):
            c.field(nm).view(torch.int32).fill_(0x2C00BC00)
        caches.append(c)
    q = torch.randn(w.batch, w.q_heads, w.head_dim, device='cuda').half()
    out = torch.empty(w.batch, w.q_heads, w.head_dim, device='cuda')
    ws = lmo.attention_workspace(w.batch, w.kv_heads, w.q_heads, w.head_dim)
    abis = [c.abi() for c in caches]
    for it in range(3):
        for l in range(nl):
            lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l])
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 10
    e0.record()
    for it in range(reps):
        for l in range(nl):
            lmo.lmo_decode_attention_q4(caches[l], q, L, out=out, workspace=ws, abi=abis[l])
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (reps * nl)
    by = attention_launch_bytes(w, L)
    print(key, 'attn %.1f us/launch, %.0f GB/s (%.1f%% of 6551)' % (ms*1e3, by/ms/1e6, by/ms/1e6/6551*100))
    del caches
