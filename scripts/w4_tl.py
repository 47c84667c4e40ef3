"""Per-step clock timeline of CTA (0,0) of the two-group W4A16 kernel (LMO_W4_EXP_TL build).
usage: LMO_LIB=build/variants/tl.so w4_tl.py N K B"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_wurypgll25_b200 import lmo
N, K, B = (int(a) for a in sys.argv[1:4])
g = torch.Generator(device="cuda"); g.manual_seed(1)
W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
x = torch.randn(B, K, generator=g, device="cuda").half()
y = torch.empty(B, N, device="cuda")
for _ in range(4):
    lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y)
torch.cuda.synchronize()
L = ctypes.CDLL(os.environ["LMO_LIB"])
buf = (ctypes.c_uint * (16 * 512))()
assert L.lmo_exp_w4_timeline(buf) == 0
t = np.frombuffer(buf, dtype=np.uint32).reshape(16, 512).astype(np.int64)
nst = K // 128
t = t[:, :nst]
t0 = t[2, 0]
t = (t - t0) & 0xFFFFFFFF
t[t > 2**31] -= 2**32
names = ["code_issue", "x_issue", "dq_start", "dq_cfull", "dq_abempty", "dq_afull_arr", "mma_xfull", "mma_afull"]
print("step " + " ".join(f"{n:>12}" for n in names))
for j in range(min(nst, 40)):
    print(f"{j:4d} " + " ".join(f"{v:12d}" for v in t[:, j]))
d = np.diff(t[5, :nst])
print("per-step dq period (cycles): median", np.median(d[4:]), "mean", d[4:].mean())
print("dq wait c_full", np.median(t[3, 4:] - t[2, 4:]), " wait ab_empty", np.median(t[4, 4:] - t[3, 4:]),
      " dequant+st", np.median(t[5, 4:] - t[4, 4:]), " mma waits a_full after x", np.median(t[7, 4:] - t[6, 4:]),
      " mma a_full seen - dq arrive", np.median(t[7, 4:] - t[5, 4:]))
print("g0: lds->", np.median(t[8, 4:] - t[4, 4:]), " deq+st g0", np.median(t[9, 4:] - t[8, 4:]),
      " lds g1", np.median(t[11, 4:] - t[9, 4:]), " deq+st g1", np.median(t[12, 4:] - t[11, 4:]),
      " fence+arrive", np.median(t[14, 4:] - t[12, 4:]), " wait::st", np.median(t[15, 4:] - t[14, 4:]),
      " fence+afull arrive", np.median(t[5, 4:] - t[15, 4:]))
