"""Where does the fused step lose time vs attention alone?  Graph-captured layer
loops (footprint > L2) of: attention only; fused step (CACHE_STABLE / no flags);
separate append kernel + attention.  usage: step_vs_attn.py c4 [c2 ...]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS

import dataclasses
for key in sys.argv[1:] or ["c4"]:
    w = CONFIGS[key.split(":")[0]]
    if ":" in key:                                   # c4:8 -> the config at batch 8 (strong-scaling shard)
        w = dataclasses.replace(w, batch=int(key.split(":")[1]))
    L = w.prompt + w.gen // 2
    nl = int(os.environ.get("NL", "0")) or max(4, min(64, int(6.0e9 // (w.batch * w.kv_heads * w.capacity * 144))))
    caches = []
    for l in range(nl):
        c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
        if os.environ.get("REAL") == "1":      # the bench's data: generated K/V quantized by append
            from paper_conf_ipps_wurypgll25_b200 import inputs as I
            kf = torch.empty((w.batch, w.kv_heads, w.capacity, w.head_dim), dtype=torch.float16, device="cuda")
            vf = torch.empty_like(kf)
            lmo.lmo_gen_fill_f16(kf, I.seed_for_config(w.index), I.STREAM_K, l, 0, 0, 0)
            lmo.lmo_gen_fill_f16(vf, I.seed_for_config(w.index), I.STREAM_V, l, 0, 0, 0)
            lmo.lmo_kv_append_quant(c, kf, vf, 0)
            del kf, vf
        else:
            c.kv.random_(0, 256)
            for nm in ("k_meta", "v_meta"):
                c.field(nm).view(torch.int32).fill_(0x2C00BC00)
        caches.append(c)
    # per-layer inputs (as in bench.py: not L2-resident when a layer's launch starts)
    qs = [torch.randn(w.batch, w.q_heads, w.head_dim, device='cuda').half() for _ in range(nl)]
    if os.environ.get("REAL") == "1":
        from paper_conf_ipps_wurypgll25_b200 import inputs as I
        for l in range(nl):
            lmo.lmo_gen_fill_f16(qs[l].view(w.batch, w.q_heads, 1, w.head_dim), I.seed_for_config(w.index),
                                 I.STREAM_Q, l, 0, 0, 0, group=w.group_ratio)
    kns = [torch.randn(w.batch, w.kv_heads, 1, w.head_dim, device='cuda').half() for _ in range(nl)]
    vns = [torch.randn_like(kns[0]) for _ in range(nl)]
    outs = [torch.empty(w.batch, w.q_heads, w.head_dim, device='cuda')
            for _ in range(nl if os.environ.get("OUTS") == "1" else 1)]   # OUTS=1: per-layer outputs (as bench.py)
    ws = lmo.attention_workspace(w.batch, w.kv_heads, w.q_heads, w.head_dim, int(os.environ.get("SPLITS", "0")))
    abis = [c.abi() for c in caches]
    st = torch.cuda.Stream()
    ns = int(os.environ.get("SPLITS", "0"))
    variants = {
        "attn": lambda l: lmo.lmo_decode_attention_q4(caches[l], qs[l], L, out=outs[l % len(outs)], workspace=ws, abi=abis[l], stream=st,
                                                   num_splits=ns),
        "step_stable": lambda l: lmo.lmo_decode_step_q4(caches[l], kns[l], vns[l], qs[l], L, out=outs[l % len(outs)], workspace=ws, abi=abis[l],
                                                        flags=lmo.LMO_STEP_CACHE_STABLE, stream=st, num_splits=ns),
        "step_plain": lambda l: lmo.lmo_decode_step_q4(caches[l], kns[l], vns[l], qs[l], L, out=outs[l % len(outs)], workspace=ws, abi=abis[l],
                                                       stream=st),
        "append+attn": lambda l: (lmo.lmo_kv_append_quant(caches[l], kns[l], vns[l], L - 1, abi=abis[l], stream=st),
                                  lmo.lmo_decode_attention_q4(caches[l], qs[l], L, out=outs[l % len(outs)], workspace=ws, abi=abis[l],
                                                              stream=st)),
        "append": lambda l: lmo.lmo_kv_append_quant(caches[l], kns[l], vns[l], L - 1, abi=abis[l], stream=st),
    }
    res = {}
    for name, fn in variants.items():
        with torch.cuda.stream(st):
            for l in range(nl):
                fn(l)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for l in range(nl):
                fn(l)
        for _ in range(2):
            g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 5
        with torch.cuda.stream(st):
            e0.record(st)
            for _ in range(reps):
                g.replay()
            e1.record(st)
        torch.cuda.synchronize()
        res[name] = e0.elapsed_time(e1) * 1e3 / (reps * nl)
    print(key, f"L={L} layers={nl}", "  ".join(f"{k} {v:.1f}us" for k, v in res.items()), flush=True)
