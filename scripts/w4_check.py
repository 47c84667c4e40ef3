"""W4A16 row-major vs packed path on one shape (the packed path is exact at every
ring depth): counts corrupted 128-row tiles.  usage: w4_check.py [N K B reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_wurypgll25_b200 import lmo
N, K, B, reps = [int(v) for v in (sys.argv[1:5] if len(sys.argv) > 4 else (28672, 7168, 64, 3))]
g = torch.Generator(device="cuda"); g.manual_seed(3)
W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
x = torch.randn(B, K, generator=g, device="cuda").half()
c, m = c.view(N, K // 2), m.view(N, K // 64)
ref = lmo.lmo_w4a16_linear_packed(lmo.lmo_w4a16_pack(c, m, N, K), N, K, x, k_split=1).cpu().numpy()
for r in range(reps):
    y = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1).cpu().numpy()
    bad = np.abs(y - ref) > 1e-3 * (np.abs(ref) + 1e-3)
    tiles = np.unique(np.nonzero(bad)[1] // 128) if bad.any() else []
    print(f"rep {r}: bad elements {int(bad.sum())} of {bad.size}, bad tiles {len(tiles)} {list(tiles)[:12]}", flush=True)
if bad.any():
    rows = np.nonzero(bad.any(axis=0))[0]
    t0 = rows[0] // 128
    in_t = rows[rows // 128 == t0] % 128
    print("first bad tile", t0, "bad rows within it:", list(in_t))
    print("bad cols per bad row (first 10):", [int(bad[:, r].sum()) for r in rows[:10]])
    hist = np.bincount(rows % 128, minlength=128)
    print("row-in-tile histogram of bad rows (by 16):", [int(hist[i:i + 16].sum()) for i in range(0, 128, 16)])
