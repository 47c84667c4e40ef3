"""Host-launch vs CUDA-graph time of the packed W4A16 GEMMs of a config's layer
(is a small GEMM bound by the host's launch path?).  usage: w4_graph.py [config]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo, configs as C
w = C.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c2"]
h = w.hidden
shapes = [(3 * h, h), (h, h), (4 * h, h), (h, 4 * h)]
g = torch.Generator(device="cuda"); g.manual_seed(1)
mats = []
for N, K in shapes:
    W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
    c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
    pk = lmo.lmo_w4a16_pack(c.view(N, K // 2), m.view(N, K // 64), N, K)
    x = torch.randn(w.batch, K, generator=g, device="cuda").half()
    mats.append((N, K, pk, x, torch.empty(w.batch, N, device="cuda")))
st = torch.cuda.Stream()
def layer():
    for N, K, pk, x, y in mats:
        lmo.lmo_w4a16_linear_packed(pk, N, K, x, y=y, stream=st)
with torch.cuda.stream(st):
    for _ in range(3): layer()
torch.cuda.synchronize()
R = 50
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
t0 = time.perf_counter()
e0.record(st)
for _ in range(R): layer()
e1.record(st)
t1 = time.perf_counter()
torch.cuda.synchronize()
eager = e0.elapsed_time(e1) * 1e3 / R
host = (t1 - t0) * 1e6 / R
gr = torch.cuda.CUDAGraph()
with torch.cuda.graph(gr, stream=st):
    layer()
for _ in range(3): gr.replay()
torch.cuda.synchronize()
e0.record(st)
for _ in range(R): gr.replay()
e1.record(st)
torch.cuda.synchronize()
graph = e0.elapsed_time(e1) * 1e3 / R
print(f"{w.name}: layer eager {eager:.1f} us (host enqueue {host:.1f} us), graph {graph:.1f} us")
