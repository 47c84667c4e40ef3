"""Driver run under compute-sanitizer by tests/test_gpu_sanitizers.py: every
library entry point once at small shapes (several tiles, ragged tails), each
attention schedule, the fused step with and without LMO_STEP_CACHE_STABLE, and
both W4A16 paths with shallow and deep rings of steps.  Prints OK at the end."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_wurypgll25_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_wurypgll25_b200 import lmo  # noqa: E402

part = sys.argv[1] if len(sys.argv) > 1 else "all"
dev = "cuda"
if part in ("all", "attn"):
    for (B, Hkv, G, d, L) in ((3, 2, 1, 128, 77), (2, 2, 8, 128, 45), (2, 3, 2, 64, 33)):
        cache = lmo.KVCache.empty(B, Hkv, L + 5, d, zero=True)
        kf = torch.empty((B, Hkv, L, d), dtype=torch.float16, device=dev)
        vf = torch.empty_like(kf)
        lmo.lmo_gen_fill_f16(kf, 5, I.STREAM_K, 0, 0, 0, 0)
        lmo.lmo_gen_fill_f16(vf, 5, I.STREAM_V, 0, 0, 0, 0)
        lmo.lmo_kv_append_quant(cache, kf[:, :, :L - 1].contiguous(), vf[:, :, :L - 1].contiguous(), 0)
        q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device=dev)
        lmo.lmo_gen_fill_f16(q, 5, I.STREAM_Q, 0, 0, 0, 0, group=G)
        q = q.view(B, Hkv * G, d)
        for ns in (0, 1, 2, 3, lmo.LMO_SPLITS_STREAMK, lmo.LMO_SPLITS_SMTEAM):
            lmo.lmo_decode_attention_q4(cache, q, L - 1, num_splits=ns)
        for flags in (0, lmo.LMO_STEP_CACHE_STABLE):
            lmo.lmo_decode_step_q4(cache, kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous(), q, L,
                                   flags=flags)
        lens = torch.tensor([L, 1, 0][:B], dtype=torch.int32, device=dev)
        lmo.lmo_decode_step_q4(cache, kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous(), q, 0,
                               seq_lens=lens)
    torch.cuda.synchronize()
if part in ("all", "quant"):
    x = torch.randn(37, 200, 3, device=dev).half()
    c, m = lmo.lmo_quantize_groupwise(x, 37, 200, 3)
    lmo.lmo_dequantize_groupwise(c, m, 37, 200, 3)
    torch.cuda.synchronize()
if part in ("all", "w4a16"):
    g = torch.Generator(device=dev)
    g.manual_seed(1)
    for (N, K, B, ks) in ((256, 1024, 64, 1), (384, 640, 5, 2), (128, 512, 100, 0)):
        W = (torch.randn(N, K, generator=g, device=dev) * 0.05).half()
        c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
        c, m = c.view(N, K // 2), m.view(N, K // 64)
        xa = torch.randn(B, K, generator=g, device=dev).half()
        lmo.lmo_w4a16_linear(c, m, N, K, xa, k_split=ks)
        lmo.lmo_w4a16_linear_packed(lmo.lmo_w4a16_pack(c, m, N, K), N, K, xa, k_split=ks)
    torch.cuda.synchronize()
print("OK")
