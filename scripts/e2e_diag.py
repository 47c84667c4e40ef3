"""Does a concurrent pinned H2D slow an HBM-bound kernel (or vice versa)?
Per step: H2D of `mb` MB on a copy stream || `gb` GB read-stream on the compute
stream; prints each alone and both overlapped.  usage: e2e_diag.py [mb gb steps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wurypgll25_b200 import lmo
mb, gb, steps = (float(a) for a in (sys.argv[1:4] if len(sys.argv) > 3 else (25, 4, 20)))
steps = int(steps)
dev = torch.device("cuda")
h = torch.empty(int(mb * 2 ** 20), dtype=torch.uint8).pin_memory()
dbuf = [torch.empty_like(h, device=dev) for _ in range(2)]
big = torch.empty(int(gb * 2 ** 30), dtype=torch.uint8, device=dev)
sink = torch.zeros(1024, device=dev)
cs, ms = torch.cuda.Stream(), torch.cuda.Stream()


def run(h2d, comp):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(ms)
    cs.wait_event(e0)
    for i in range(steps):
        if h2d:
            with torch.cuda.stream(cs):
                dbuf[i % 2].copy_(h, non_blocking=True)
        if comp:
            lmo.lmo_probe_read_stream(big, sink, stream=ms)
    ms.wait_stream(cs)
    e1.record(ms)
    e1.synchronize()
    return e0.elapsed_time(e1) / steps


for _ in range(2):
    run(True, True)
a, b, c = run(True, False), run(False, True), run(True, True)
print(f"H2D {mb:.0f} MB alone {a:.3f} ms ({mb * 2**20 / a / 1e6:.1f} GB/s)  read {gb:.1f} GB alone {b:.3f} ms "
      f"({gb * 2**30 / b / 1e6:.0f} GB/s)  both {c:.3f} ms")
