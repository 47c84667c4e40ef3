"""Needs a build with -DLMO_ATTN_PROFILE=1.  Per-warp globaltimer timeline of one
attention launch inside a graph of back-to-back layer launches (like the bench):
entry skew, entry -> loop start, loop start -> first data, end distribution, and
the gap to the next launch.  usage: attn_timeline.py B H G L [early]"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
B, H, G, L = [int(x) for x in sys.argv[1:5]]
STEP = len(sys.argv) > 5 and sys.argv[5] == "step"     # fused append + attention, CACHE_STABLE
NS = int(os.environ.get("SPLITS", "0"))                 # num_splits (1/2/4 = explicit team size)
d = 128
nl = max(3, int(2e9 // (B * H * (L + 16) * 144)))
caches = [lmo.KVCache.empty(B, H, (L + 15) // 16 * 16, d) for _ in range(nl)]
for c in caches:
    c.kv.random_(0, 256)
    for nm in ("k_meta", "v_meta"): c.field(nm).view(torch.int32).fill_(0x2C00BC00)
q = torch.randn(B, H * G, d, device='cuda').half()
out = torch.empty(B, H * G, d, device='cuda')
ws = lmo.attention_workspace(B, H, H * G, d)
kn = torch.randn(B, H, d, device='cuda').half(); vn = torch.randn_like(kn)
def launch(c):
    if STEP:
        lmo.lmo_decode_step_q4(c, kn, vn, q, L, out=out, workspace=ws, flags=lmo.LMO_STEP_CACHE_STABLE, num_splits=NS)
    else:
        lmo.lmo_decode_attention_q4(c, q, L, out=out, workspace=ws, num_splits=NS)
nl = min(nl, 16)
buf = torch.zeros(16 * 148 * 64 * 16, dtype=torch.int64, device='cuda')
lmo._lib.lmo_debug_attn_profile(ctypes.c_void_p(buf.data_ptr()))
for l in range(nl):                       # eager warm-up (slots 0..nl-1)
    launch(caches[l])
torch.cuda.synchronize()
for _ in range(16 - nl):                  # align the slot counter to 0 again
    launch(caches[0])
st = torch.cuda.Stream()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=st):      # captured launch l keeps slot l
    for l in range(nl):
        launch(caches[l])
for _ in range(3): g.replay()
torch.cuda.synchronize()
buf.zero_()
g.replay()
torch.cuda.synchronize()
T = []
for l in range(nl):
    b = buf.view(16, -1, 16)[l].cpu()
    b = b[b[:, 2] > 0].double()
    T.append(b)
base = T[1][:, 4].min()
for l in range(1, min(nl, 5)):
    b = T[l]
    e, s0, f, z = [(b[:, i] - base) / 1e3 for i in (4, 5, 6, 7)]
    q_ = lambda x: f"{x.min():6.2f}/{x.median():6.2f}/{x.max():6.2f}"
    print(f"launch {l}: warps {b.shape[0]} entry {q_(e)} | loopstart {q_(s0)} | first data {q_(f)} | end {q_(z)} us  (min/med/max)")
    rel = lambda i: (b[:, i] - b[:, 4]) / 1e3
    print("          from entry: " + "  ".join(f"{nm} {q_(rel(i))}" for nm, i in
          (("wait", 8), ("workmap", 9), ("mbfence", 13), ("begin", 14), ("prologue", 10), ("append", 11), ("loop", 5), ("qfrags", 12))))
    print(f"          entry->loop {q_(s0 - e)}  loop->data {q_(f - s0)}  data->end {q_(z - f)}  stages/warp {b[:,2].mean():.1f}")

# SM / SMSP placement of the busy warps (launch 2) and its effect on warp end times
import collections
b = T[2]
sm = (b[:, 3].long() >> 32)
wid = (b[:, 3].long() >> 16) & 0xffff
sp = wid % 4
end = (b[:, 7] - b[:, 4].min()) / 1e3
cnt_sm = collections.Counter(sm.tolist())
cnt_sp = collections.Counter(zip(sm.tolist(), sp.tolist()))
print("busy warps per SM: ", sorted(collections.Counter(cnt_sm.values()).items()))
print("busy warps per SMSP:", sorted(collections.Counter(cnt_sp.values()).items()),
      " SMSPs used:", len(cnt_sp), "of", 4 * len(cnt_sm))
print("smsp index histogram:", sorted(collections.Counter(sp.tolist()).items()))
for k in sorted(set(cnt_sp.values())):
    m = torch.tensor([cnt_sp[(a, c)] == k for a, c in zip(sm.tolist(), sp.tolist())])
    print(f"  warps on SMSPs holding {k} busy warps: {int(m.sum())}, end median {end[m].median():.2f} max {end[m].max():.2f} us")

# per-warp breakdown (launch 2): data->end vs segments, mbarrier wait share
segs = (b[:, 3].long() & 0xffff)
dte = (b[:, 7] - b[:, 6]) / 1e3
wait_us = b[:, 0] / 1.965e3
print("data->end by segments/warp:")
for k in sorted(set(segs.tolist())):
    m = segs == k
    print(f"  segs={k}: warps {int(m.sum())}, data->end median {dte[m].median():.2f} max {dte[m].max():.2f} us, "
          f"mbar wait median {wait_us[m].median():.2f} us")
slow = dte > dte.median() + 5
print(f"slow warps (>median+5us): {int(slow.sum())}, their wait median {wait_us[slow].median() if slow.any() else 0:.2f} us, "
      f"end-1st-data median {dte[slow].median() if slow.any() else 0:.2f}")
cs = (b[:, 15].long() & 0xffffffff).double() / 1.965e3
ce = (b[:, 15].long() >> 32).double() / 1.965e3
for k in sorted(set(segs.tolist())):
    m = segs == k
    print(f"  segs={k}: seg-start section median {cs[m].median():.2f} us, seg-end section median {ce[m].median():.2f} max {ce[m].max():.2f} us")
le = (b[:, 13] - b[:, 4].min()) / 1e3
z2 = (b[:, 7] - b[:, 4].min()) / 1e3
print(f"launch 2 (rel. to first entry): loop end {le.min():.2f}/{le.median():.2f}/{le.max():.2f}  kernel exit {z2.min():.2f}/{z2.median():.2f}/{z2.max():.2f} us")
# segments (pairs) per SMSP: is the extra work concentrated on some SMSP indices?
seg_sp = collections.Counter()
for a, c, k in zip(sm.tolist(), sp.tolist(), segs.tolist()):
    seg_sp[(a, c)] += k
print("segments per SMSP:", sorted(collections.Counter(seg_sp.values()).items()))
by_idx = collections.defaultdict(list)
for (a, c), k in seg_sp.items():
    by_idx[c].append(k)
print("mean segments per SMSP index:", {c: round(sum(v) / len(v), 2) for c, v in sorted(by_idx.items())})
# CTA -> SM placement: which CTA ids share an SM (first 8 SMs)
cta = b[:, 3].long() & 0  # (CTA id is not recorded; warp id within SM is)
