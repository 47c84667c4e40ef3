#!/usr/bin/env python3
"""bench.py -- q4-KV decode throughput on B200 (BASELINE.json metric).

A "step" is one decode step of the whole hot path over all layers of the
workload: for every layer, append-quantize the new token's K/V (A2) and run
decode attention over the q4 cache (A3+A4).  Inputs are seeded synthetic
tensors shaped like the paper's OPT/LLaMA workloads, resident in HBM before
the timed region (value) or copied from pinned host memory inside it (e2e).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl ours|reference]

Multi-GPU (torchrun, one rank per GPU, NCCL): the batch is sharded by
sequence -- weak scaling, each rank owns a full config-sized batch at its own
global batch offset; no collective in the hot path (timing reduce only).
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_wurypgll25_b200 import configs as C  # noqa: E402
from paper_conf_ipps_wurypgll25_b200 import inputs as I  # noqa: E402

METRIC = "q4-KV decode-attention tokens/s & achieved HBM GB/s at 1/2/4/8 B200"
FALLBACK_HBM = 6650.0


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="c2", choices=sorted(C.CONFIGS))
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--splits", type=int, default=0, help="num_splits (0 = stream-K auto)")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-stream", action="store_true", help="skip the A1/A5 weight streaming leg")
    p.add_argument("--no-offload", action="store_true", help="skip the host-offloaded KV leg")
    p.add_argument("--no-early", action="store_true", help="disable LMO_STEP_CACHE_STABLE")
    p.add_argument("--cpu-sample-seconds", type=float, default=10.0)
    return p.parse_args()


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md 6.65 TB/s)"


def workload_config(w: C.Workload, n: int, extra=None):
    d = {
        "workload": f"{w.key}: {w.name}",
        "batch_per_gpu": w.batch, "global_batch": w.batch * n, "q_heads": w.q_heads,
        "kv_heads": w.kv_heads, "head_dim": w.head_dim, "layers": w.layers,
        "prompt": w.prompt, "gen": w.gen, "kv_format": "4-bit group-wise min/scale, G=64",
        "parallelism": f"batch-sharded dp{n} (weak scaling)",
    }
    if extra:
        d.update(extra)
    return d


# ------------------------------------------------------------- clocks ------

class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.6)          # nvidia-smi start-up: samples begin before the timed region
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.lines = []
        if self.proc is not None:
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [ln for ln in out.splitlines() if ln.strip()]

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in getattr(self, "lines", []):
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = max(mx, float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# -------------------------------------------------------- CPU oracle -------

def cpu_oracle_rate(w: C.Workload, target_s: float, nthreads: int):
    """Time the oracle (as it stands) on a bounded sample of decode work at the
    mean decode length: whole layers' worth of (sequence, kv-head) pairs (one
    append + one attention each), repeated over layers until ~target_s of CPU
    wall time; extrapolated linearly to tokens/s of the whole workload."""
    import numpy as np
    import oracle
    seed = I.seed_for_config(w.index)
    L = w.prompt + w.gen // 2
    d, G = w.head_dim, w.group_ratio
    pairs_total = w.batch * w.kv_heads
    units = [(l, b, h) for l in range(w.layers) for b in range(w.batch) for h in range(w.kv_heads)]
    done, elapsed, npairs = 0, 0.0, max(1, nthreads)
    while elapsed < target_s and done < len(units):
        chunk = units[done:done + npairs]
        B = len(chunk)
        cache = oracle.new_cache(B, 1, L + 1, d)
        ks = np.stack([I.gen_f16(seed, I.STREAM_K, l, b, 1, h, 1, 0, L + 1, d)[0] for l, b, h in chunk])
        vs = np.stack([I.gen_f16(seed, I.STREAM_V, l, b, 1, h, 1, 0, L + 1, d)[0] for l, b, h in chunk])
        qs = np.stack([I.gen_f16(seed, I.STREAM_Q, l, b, 1, h * G, G, 0, 1, d, group=G)[0, :, 0]
                       for l, b, h in chunk])
        oracle.kv_append_quant(cache, ks[:, :, :L], vs[:, :, :L], 0)   # resident cache (untimed)
        t0 = time.perf_counter()
        oracle.kv_append_quant(cache, ks[:, :, L:], vs[:, :, L:], L)    # A2 (timed)
        oracle.decode_attention_q4(cache, qs, L + 1, nthreads=nthreads)  # A3 (timed)
        elapsed += time.perf_counter() - t0
        done += B
        npairs = min(len(units) - done, npairs * 2)
    t_unit = elapsed / done
    t_step = t_unit * pairs_total * w.layers
    tokens_per_s = w.batch / t_step
    by = C.layer_step_bytes(w, L + 1) * w.layers
    return {
        "value": tokens_per_s, "unit": "tokens/s", "cores": nthreads, "kind": "oracle",
        "sample": (f"{done} (layer, sequence, kv-head) units of one decode step at L={L + 1} "
                   f"(append + attention of {G} q head(s) each) = {elapsed:.1f} s CPU wall on "
                   f"{nthreads} threads; extrapolated x{pairs_total * w.layers / done:.1f} to the "
                   f"{pairs_total} x {w.layers} units of a step (work is linear in units)"),
        "gbs_equiv": by / t_step / 1e9,
    }


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    w = C.CONFIGS[args.config]
    nthreads = len(os.sched_getaffinity(0))
    vals = []
    base = None
    per = max(1.0, min(3.0, args.cpu_sample_seconds / 3))
    for i in range(args.warmup + args.steps):
        r = cpu_oracle_rate(w, per if i >= args.warmup else 0.5, nthreads)
        if i >= args.warmup:
            vals.append(r["value"])
            base = r
    v = statistics.median(vals)
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "tokens/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * w.batch / v, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded counter-based generator)",
        "config": workload_config(w, 1),
        "cpu_baseline": {"value": v, "unit": "tokens/s", "cores": nthreads, "kind": "oracle",
                         "sample": base["sample"]},
        "e2e": {"value": v, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------- our arm -------

def run_ours(args):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_wurypgll25_b200 import lmo

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    w = C.CONFIGS[args.config]
    seed = I.seed_for_config(w.index)
    B, Hkv, Hq, d, G, s = w.batch, w.kv_heads, w.q_heads, w.head_dim, w.group_ratio, w.prompt
    from paper_conf_ipps_wurypgll25_b200 import dist as D
    b_off, _ = D.shard(rank, world, B)    # global batch offset (weak scaling, no hot-path collective)
    nl = w.layers
    steps_total = args.warmup + args.steps
    # Timed decode steps are spread evenly over the whole generation t = 1..n-1
    # (L = s+t), so the measured throughput covers the workload's length mix;
    # warm-up steps replay the same positions.  The cache is prefilled with the
    # K/V of every position up to s+n-2 (what a real decode would have written),
    # so any step t can run in any order; each step re-appends slot s+t-1.
    K_ = args.steps
    timed_t = [1 + (j * (w.steps - 1)) // max(1, K_ - 1) for j in range(K_)] if K_ > 1 else [w.steps]
    t_of = [timed_t[j % len(timed_t)] for j in range(args.warmup)] + timed_t
    distinct_t = sorted(set(t_of))

    # ---- caches + prefill (A1 through the append entry; timed separately)
    caches = [lmo.KVCache.empty(B, Hkv, w.capacity, d, device=dev) for _ in range(nl)]
    abis = [c.abi() for c in caches]
    stream = torch.cuda.Stream(device=dev)
    pre_ms = 0.0
    with torch.cuda.stream(stream):
        P_ = w.max_len - 1                    # positions 0 .. s+n-2
        kp = torch.empty((B, Hkv, P_, d), dtype=torch.float16, device=dev)
        vp = torch.empty_like(kp)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for l in range(nl):
            lmo.lmo_gen_fill_f16(kp, seed, I.STREAM_K, l, b_off, 0, 0)
            lmo.lmo_gen_fill_f16(vp, seed, I.STREAM_V, l, b_off, 0, 0)
            e0.record()       # prefill quantize (A1 through the append entry), prompt part timed
            lmo.lmo_kv_append_quant(caches[l], kp[:, :, :s].contiguous(), vp[:, :, :s].contiguous(),
                                    pos0=0, abi=abis[l])
            e1.record()
            e1.synchronize()
            pre_ms += e0.elapsed_time(e1)
            if P_ > s:        # generated-token positions (what earlier decode steps appended)
                lmo.lmo_kv_append_quant(caches[l], kp[:, :, s:].contiguous(), vp[:, :, s:].contiguous(),
                                        pos0=s, abi=abis[l])
        del kp, vp
        # ---- per-step inputs (device-resident) and outputs
        qbuf, kbuf, vbuf = {}, {}, {}
        for t in distinct_t:
            qbuf[t] = torch.empty((nl, B, Hq, 1, d), dtype=torch.float16, device=dev)
            kbuf[t] = torch.empty((nl, B, Hkv, 1, d), dtype=torch.float16, device=dev)
            vbuf[t] = torch.empty_like(kbuf[t])
            for l in range(nl):
                lmo.lmo_gen_fill_f16(qbuf[t][l], seed, I.STREAM_Q, l, b_off, 0, t - 1, group=G)
                lmo.lmo_gen_fill_f16(kbuf[t][l], seed, I.STREAM_K, l, b_off, 0, s + t - 1)
                lmo.lmo_gen_fill_f16(vbuf[t][l], seed, I.STREAM_V, l, b_off, 0, s + t - 1)
        out = torch.empty((nl, B, Hq, d), dtype=torch.float32, device=dev)
        ws = lmo.attention_workspace(B, Hkv, Hq, d, args.splits, device=dev)
    stream.synchronize()
    sigma = 1.0 / math.sqrt(d)

    def step(t, attn=True, append=True):
        """One decode step: for every layer, A2 append of the new token at slot
        s+t-1 and A3/A4 attention over L = s+t -- one fused launch per layer
        (lmo_decode_step_q4); attn-only variant for the roofline leg."""
        for l in range(nl):
            if append and attn:
                lmo.lmo_decode_step_q4(caches[l], kbuf[t][l], vbuf[t][l], qbuf[t][l].view(B, Hq, d),
                                       s + t, softmax_scale=sigma, num_splits=args.splits,
                                       out=out[l], workspace=ws, abi=abis[l],
                                       flags=0 if args.no_early else lmo.LMO_STEP_CACHE_STABLE)
            elif attn:
                lmo.lmo_decode_attention_q4(caches[l], qbuf[t][l].view(B, Hq, d), s + t,
                                            softmax_scale=sigma, num_splits=args.splits,
                                            out=out[l], workspace=ws, abi=abis[l])
            else:
                lmo.lmo_kv_append_quant(caches[l], kbuf[t][l], vbuf[t][l], pos0=s + t - 1,
                                        abi=abis[l])

    # ---- capture one CUDA graph per distinct step
    graphs = {}
    n0 = lmo.launch_count()
    for t in distinct_t:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            step(t)
        graphs[t] = g
    launches_per_step = (lmo.launch_count() - n0) // len(distinct_t)
    # attention-only graph (roofline leg) at the middle length
    t_mid = distinct_t[len(distinct_t) // 2]
    g_attn = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g_attn, stream=stream):
        step(t_mid, append=False)
    torch.cuda.synchronize()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def reduce_max(x: float) -> float:
        return D.max_over_ranks(x, device=dev)

    # ---- warm-up + timed steps (device-resident inputs).  The clock sampler runs
    # across a ~0.5 s load window that ends with the timed region (warm-up steps
    # are replayed until the window is full, so clocks are sampled under load).
    with torch.cuda.stream(stream):
        for j in range(args.warmup):
            graphs[t_of[j]].replay()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        with torch.cuda.stream(stream):
            t_end = time.perf_counter() + 0.5
            while time.perf_counter() < t_end:
                for j in range(args.warmup):
                    graphs[t_of[j]].replay()
                torch.cuda.current_stream().synchronize()
            ev0.record(stream)
            for j in range(args.warmup, steps_total):
                graphs[t_of[j]].replay()
            ev1.record(stream)
            # keep the GPU loaded while the sampler catches the tail of the window
            for j in range(args.warmup):
                graphs[t_of[j]].replay()
        ev1.synchronize()
        torch.cuda.synchronize()
    barrier()
    ms = reduce_max(ev0.elapsed_time(ev1))
    clocks = clk.summary()
    tokens = world * B * args.steps
    value = tokens / (ms / 1e3)
    step_bytes = sum(C.layer_step_bytes(w, s + t_of[j], B) * nl for j in range(args.warmup, steps_total))
    gbs = world * step_bytes / (ms / 1e3) / 1e9

    # ---- roofline leg: attention-only launches, CUDA events on the launching stream
    reps = 5
    with torch.cuda.stream(stream):
        g_attn.replay()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(reps):
            g_attn.replay()
        a1.record(stream)
    a1.synchronize()
    attn_ms = reduce_max(a0.elapsed_time(a1)) / (reps * nl)
    attn_bytes = C.attention_launch_bytes(w, s + t_mid, B)
    peak, peak_src = peaks()
    achieved = attn_bytes / (attn_ms / 1e3) / 1e9
    traffic = None
    prof = os.path.join(ROOT, "profiles", f"ncu_{w.key}.json")
    if os.path.exists(prof):
        try:
            traffic = json.load(open(prof)).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    # ---- streaming legs (A1 quantize, A5 dequantize) on one layer's weights, 12 h1^2
    # elements (QKV/O + FFN), groups of 64 along the contiguous dim: the
    # "q4 weight dequant" of BASELINE config 3 (Eq 4).  > L2; CUDA events.
    streaming = None
    if not args.no_stream and w.hidden > 0:
        nel = 12 * w.hidden * w.hidden
        rows, n = nel // w.hidden, w.hidden
        with torch.cuda.stream(stream):
            gen = torch.Generator(device=dev)
            gen.manual_seed(seed)
            xw = (torch.randn((rows, n), generator=gen, device=dev) * 0.02).half()   # weight-like N(0, 0.02)
            codes = torch.empty((rows, n // 2), dtype=torch.uint8, device=dev)
            meta = torch.empty((rows, n // 64), dtype=torch.int32, device=dev)
            yw = torch.empty_like(xw)
            res = {}
            for name, fn, by in (
                    ("quantize_A1", lambda: lmo.lmo_quantize_groupwise(xw, rows, n, 1, codes=codes, meta=meta,
                                                                      stream=stream), nel * (2 + 0.5625)),
                    ("dequantize_A5", lambda: lmo.lmo_dequantize_groupwise(codes, meta, rows, n, 1, y=yw,
                                                                          stream=stream), nel * (0.5625 + 2))):
                fn()
                q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                q0.record(stream)
                for _ in range(5):
                    fn()
                q1.record(stream)
                q1.synchronize()
                t_ms = reduce_max(q0.elapsed_time(q1)) / 5
                res[name] = {"GB/s": by / (t_ms / 1e3) / 1e9, "frac": by / (t_ms / 1e3) / 1e9 / peak,
                             "us_per_launch": t_ms * 1e3, "algorithmic_bytes": by}
            streaming = {"elements": nel, "shape": f"({rows}, {n}) fp16 = 12 h1^2 weights of one layer",
                         "peak": peak, **res}
            del xw, codes, meta, yw

    # ---- NEXT-3 leg: one layer's linear layers over q4 weights (QKV 3h x h, O h x h,
    # FFN1 4h x h, FFN2 h x 4h: the paper's 4 h1^2 + 2 h1 h2) at this GPU's
    # batch through lmo_w4a16_linear (dequantization fused into the tcgen05 GEMM), vs the
    # paper's path -- dequantize (A5) then an fp16 cuBLAS matmul (Eq 4).
    w4a16 = None
    if not args.no_stream and w.hidden > 0 and B <= 128:
        h = w.hidden
        shapes = [("qkv", 3 * h, h), ("o", h, h), ("ffn1", 4 * h, h), ("ffn2", h, 4 * h)]
        with torch.cuda.stream(stream):
            gen = torch.Generator(device=dev)
            gen.manual_seed(seed + 1)
            mats = []
            for name, N_, K_ in shapes:
                wt = (torch.randn((N_, K_), generator=gen, device=dev) * 0.02).half()
                c_, m_ = lmo.lmo_quantize_groupwise(wt, N_, K_, 1, stream=stream)
                xa = torch.randn((B, K_), generator=gen, device=dev).half()
                c_, m_ = c_.view(N_, K_ // 2), m_.view(N_, K_ // 64)
                pk = lmo.lmo_w4a16_pack(c_, m_, N_, K_, stream=stream)   # once, at weight-load time
                mats.append((name, N_, K_, c_, m_, xa, torch.empty((B, N_), device=dev), pk))
                del wt
            wd = torch.empty((max(N_ * K_ for _, N_, K_ in shapes),), dtype=torch.float16, device=dev)

            def fused():
                for _, N_, K_, c_, m_, xa, ya, pk in mats:
                    lmo.lmo_w4a16_linear_packed(pk, N_, K_, xa, y=ya, stream=stream)

            def dq_cublas():
                for _, N_, K_, c_, m_, xa, ya, pk in mats:
                    wv = wd[:N_ * K_].view(N_, K_)
                    lmo.lmo_dequantize_groupwise(c_, m_, N_, K_, 1, y=wv.view(N_, K_, 1), stream=stream)
                    torch.matmul(xa, wv.t())

            def timeit(fn, reps=10):
                fn()
                q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                q0.record(stream)
                for _ in range(reps):
                    fn()
                q1.record(stream)
                q1.synchronize()
                return reduce_max(q0.elapsed_time(q1)) / reps

            t_f, t_b = timeit(fused), timeit(dq_cublas)
            by = sum(N_ * K_ * 0.5625 + B * K_ * 2 + B * N_ * 4 for _, N_, K_ in shapes)
            fl = sum(2.0 * B * N_ * K_ for _, N_, K_ in shapes)
            w4a16 = {"kernel": "w4a16_kernel (lmo_w4a16_linear_packed; tcgen05, A = dequantized weights in TMEM)",
                     "shapes": {n_: [N_, K_] for n_, N_, K_ in shapes}, "batch": B,
                     "us_per_layer": t_f * 1e3, "GB/s": by / (t_f / 1e3) / 1e9,
                     "frac": by / (t_f / 1e3) / 1e9 / peak, "TFLOP/s": fl / (t_f / 1e3) / 1e12,
                     "algorithmic_bytes": by,
                     "dequant_then_cublas_us_per_layer": t_b * 1e3, "speedup_vs_dequant_then_cublas": t_b / t_f}
            del mats, wd

    # ---- NEXT-4 leg: the same decode step with every layer's q4 cache offloaded to pinned
    # host memory (the paper's setting, Alg 1): per layer a strided H2D of the old rows
    # into a 3-slot device ring, the fused step, a D2H of the new row (lmo_offload_*).
    offload = None
    host_bytes = nl * caches[0].nbytes()
    if not args.no_offload and host_bytes <= 8e9:
        ox = lmo.OffloadKV(nl, B, Hkv, w.capacity, d, slots=3, device=dev)
        for l in range(nl):
            ox.host_layer(l).copy_(caches[l].kv.cpu())
        t = t_mid
        L = s + t
        oout = torch.empty((nl, B, Hq, d), dtype=torch.float32, device=dev)
        kq = qbuf[t].view(nl, B, Hq, d)
        with torch.cuda.stream(stream):
            ox.decode_step(kbuf[t], vbuf[t], kq, L, softmax_scale=sigma, num_splits=args.splits,
                           out=oout, workspace=ws, stream=stream)
            o0, o1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            o0.record(stream)
            nrep = 3
            for _ in range(nrep):
                ox.decode_step(kbuf[t], vbuf[t], kq, L, softmax_scale=sigma, num_splits=args.splits,
                               out=oout, workspace=ws, stream=stream)
            o1.record(stream)
        o1.synchronize()
        off_ms = reduce_max(o0.elapsed_time(o1)) / nrep
        # raw pinned H2D bandwidth of this box (one 1 GiB copy) for the fraction
        hb = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
        db = torch.empty(1 << 30, dtype=torch.uint8, device=dev)
        db.copy_(hb, non_blocking=True)
        torch.cuda.synchronize()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record()
        db.copy_(hb, non_blocking=True)
        p1.record()
        p1.synchronize()
        pcie = (1 << 30) / (p0.elapsed_time(p1) / 1e3) / 1e9
        del hb, db
        h2d_step = nl * B * Hkv * (L - 1) * lmo.row_bytes(d)
        offload = {"value": world * B / (off_ms / 1e3), "unit": "tokens/s", "ms_per_step": off_ms,
                   "L": L, "ring_slots": 3, "host_bytes": host_bytes,
                   "h2d_bytes_per_step": h2d_step,
                   "d2h_bytes_per_step": nl * B * Hkv * lmo.row_bytes(d),
                   "h2d_gbs": h2d_step / (off_ms / 1e3) / 1e9, "h2d_peak_gbs_measured": pcie,
                   "frac_of_h2d_peak": h2d_step / (off_ms / 1e3) / 1e9 / pcie,
                   "path": "pinned host q4 caches -> strided H2D (copy stream) -> fused step on a ring slot -> D2H of the new row"}
        ox.close()
        del ox, oout

    # ---- e2e: host buffers, H2D of each step's inputs + D2H of its result in the region
    e2e = None
    if not args.no_e2e:
        hq = {t: qbuf[t].cpu().pin_memory() for t in distinct_t}
        hk = {t: kbuf[t].cpu().pin_memory() for t in distinct_t}
        hv = {t: vbuf[t].cpu().pin_memory() for t in distinct_t}
        hout = torch.empty((B, Hq, d), dtype=torch.float32).pin_memory()
        h2d = (hq[t_mid].numel() + hk[t_mid].numel() + hv[t_mid].numel()) * 2
        d2h = hout.numel() * 4
        barrier()
        # Copy engine and SMs overlap: step j+1's H2D (copy stream) runs while step
        # j's graph computes; each graph waits for its own inputs' event, each D2H
        # for its graph.  Every step's inputs still cross PCIe inside the region.
        cstream = torch.cuda.Stream(device=dev)
        timed = list(range(args.warmup, steps_total))
        with torch.cuda.stream(stream):
            x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            x0.record(stream)
        cstream.wait_event(x0)

        def h2d_of(j):
            t = t_of[j]
            with torch.cuda.stream(cstream):
                qbuf[t].copy_(hq[t], non_blocking=True)
                kbuf[t].copy_(hk[t], non_blocking=True)
                vbuf[t].copy_(hv[t], non_blocking=True)
                ev = torch.cuda.Event()
                ev.record(cstream)
            return ev

        ready = h2d_of(timed[0])
        read_out = None
        for i, j in enumerate(timed):
            nxt = h2d_of(timed[i + 1]) if i + 1 < len(timed) else None
            with torch.cuda.stream(stream):
                stream.wait_event(ready)
                if read_out is not None:      # out[] is rewritten: previous D2H first
                    stream.wait_event(read_out)
                graphs[t_of[j]].replay()
                done = torch.cuda.Event()
                done.record(stream)
            with torch.cuda.stream(cstream):
                cstream.wait_event(done)
                hout.copy_(out[nl - 1], non_blocking=True)
                read_out = torch.cuda.Event()
                read_out.record(cstream)
            ready = nxt
        with torch.cuda.stream(stream):
            stream.wait_stream(cstream)
            x1.record(stream)
        x1.synchronize()
        barrier()
        e2e_ms = reduce_max(x0.elapsed_time(x1))
        e2e = {"value": tokens / (e2e_ms / 1e3), "unit": "tokens/s", "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "ms_per_step": e2e_ms / args.steps,
               "path": "pinned host inputs -> H2D (copy stream, overlapped with the previous step) -> liblmo C-ABI step graph -> D2H last-layer output"}

    cpu = None
    if rank == 0 and world == 1:
        try:
            cpu = cpu_oracle_rate(w, args.cpu_sample_seconds, len(os.sched_getaffinity(0)))
            cpu.pop("gbs_equiv", None)
        except Exception as ex:  # never fail the bench line on the baseline leg
            cpu = {"value": None, "error": str(ex)[:200]}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u4+f16/f32",
            "data": "synthetic (seeded counter-based generator; OPT/LLaMA-shaped K/V/q)",
            "config": workload_config(w, world, {
                "l2": f"inputs larger than L2: per-step q4 KV footprint "
                      f"{sum(c.nbytes() for c in caches) / 1e9:.2f} GB per GPU cycles through 126 MB L2",
                "num_splits": args.splits,
                "timed_decode_steps_t": timed_t, "attention_len": f"L = s + t ({w.prompt + timed_t[0]}..{w.prompt + timed_t[-1]})"}),
            "achieved_gbs": gbs, "frac_of_peak": gbs / peak,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel": "decode_attn_q4_kernel (attention-only launches, L=s+t_mid)",
                         "peak_source": peak_src,
                         "per_launch_us": attn_ms * 1e3, "algorithmic_bytes_per_launch": attn_bytes},
            "prefill_ms_all_layers": pre_ms,
            "streaming": streaming,
            "w4a16": w4a16,
            "offload": offload,
            "gpu_launches": launches_per_step * args.steps,
            "clocks": clocks,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
