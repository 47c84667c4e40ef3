"""Needs a build with -DLMO_ATTN_PROFILE=1. Per-warp wait/total cycles."""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS
splits = int(os.environ.get("SPLITS", "0"))
for key in sys.argv[1:] or ["c2"]:
    w = CONFIGS[key]
    c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
    c.kv.random_(0, 256)
    for nm in ("k_meta", "v_meta"): c.field(nm).view(torch.int32).fill_(0x2C00BC00)
    q = torch.randn(w.batch, w.q_heads, w.head_dim, device='cuda').half()
    buf = torch.zeros(148 * 64 * 4, dtype=torch.int64, device='cuda')
    lmo._lib.lmo_debug_attn_profile(ctypes.c_void_p(buf.data_ptr()))
    for i in range(3):
        buf.zero_()
        out = lmo.lmo_decode_attention_q4(c, q, w.max_len, num_splits=splits)
        torch.cuda.synchronize()
    b = buf.view(-1, 4).cpu()
    act = b[:, 2] > 0
    b = b[act].double()
    print(f"{key} splits={splits}: warps {int(act.sum())}  total cyc mean {b[:,1].mean():.0f} max {b[:,1].max():.0f} | wait mean {b[:,0].mean():.0f} ({100*b[:,0].sum()/b[:,1].sum():.0f}%) | stages/warp {b[:,2].mean():.1f} segs {b[:,3].mean():.2f} | cyc/stage excl wait {((b[:,1]-b[:,0])/b[:,2]).mean():.0f}")
