"""Compare lmo_w4a16_linear between two builds (LMO_LIB_A / LMO_LIB_B) on one shape."""
import os, sys, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
N, K, B = [int(v) for v in (sys.argv[1:4] if len(sys.argv) > 3 else (28672, 7168, 64))]
res = {}
for tag in ("A", "B"):
    os.environ["LMO_LIB"] = os.environ["LMO_LIB_" + tag]
    for m in [k for k in list(sys.modules) if k.startswith("paper_conf")]:
        del sys.modules[m]
    from paper_conf_ipps_wurypgll25_b200 import lmo
    g = torch.Generator(device="cuda"); g.manual_seed(3)
    W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
    c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
    x = torch.randn(B, K, generator=g, device="cuda").half()
    c, m = c.view(N, K // 2), m.view(N, K // 64)
    if os.environ.get("PACKED") == "1":
        res[tag] = lmo.lmo_w4a16_linear_packed(lmo.lmo_w4a16_pack(c, m, N, K), N, K, x, k_split=1).cpu().numpy()
    else:
        res[tag] = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1).cpu().numpy()
d = np.abs(res["A"] - res["B"])
bad = d > 1e-3 * (np.abs(res["A"]) + 1e-3)
print("max diff", d.max(), "bad elements", int(bad.sum()), "of", d.size)
if bad.any():
    rows = np.unique(np.nonzero(bad)[1]); cols = np.unique(np.nonzero(bad)[0])
    print("bad output features (n):", len(rows), rows[:20], "tiles", np.unique(rows // 128)[:20])
    print("bad batch cols:", cols[:20])
