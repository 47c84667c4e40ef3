"""Is a sustained c4 attention stream slower than a short burst after idle (power cap)?
Replays one 64-layer attention graph: a burst after 2 s idle, then back-to-back for ~1.5 s,
timing each replay; samples nvidia-smi clocks/power meanwhile."""
import os, sys, time, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo, inputs as I
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS
w = CONFIGS["c4"]; L = 528; nl = 64
caches = []
for l in range(nl):
    c = lmo.KVCache.empty(w.batch, w.kv_heads, w.capacity, w.head_dim)
    c.kv.random_(0, 256)
    for nm in ("k_meta", "v_meta"): c.field(nm).view(torch.int32).fill_(0x2C00BC00)
    caches.append(c)
qs = [torch.randn(w.batch, w.q_heads, w.head_dim, device="cuda").half() for _ in range(nl)]
outs = [torch.empty(w.batch, w.q_heads, w.head_dim, device="cuda") for _ in range(nl)]
ws = lmo.attention_workspace(w.batch, w.kv_heads, w.q_heads, w.head_dim)
abis = [c.abi() for c in caches]
st = torch.cuda.Stream()
def run():
    for l in range(nl):
        lmo.lmo_decode_attention_q4(caches[l], qs[l], L, out=outs[l], workspace=ws, abi=abis[l], stream=st)
with torch.cuda.stream(st): run()
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=st): run()
g.replay(); torch.cuda.synchronize()
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.mem,power.draw,clocks_event_reasons.sw_power_cap",
                        "--format=csv,noheader", "-lms", "100"], stdout=subprocess.PIPE, text=True)
time.sleep(2.0)
evs = []
with torch.cuda.stream(st):
    for i in range(400):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); g.replay(); e1.record(st)
        evs.append((e0, e1))
torch.cuda.synchronize()
smi.terminate(); out = smi.communicate()[0]
t = [a.elapsed_time(b) * 1e3 / nl for a, b in evs]
for i in (0, 1, 2, 5, 10, 20, 50, 100, 200, 399):
    print(f"replay {i:3d}: {t[i]:.1f} us/launch")
print("smi samples (clock sm, mem, power, pcap):")
print("\n".join(out.splitlines()[::4][:20]))
