"""NEXT-4: LM-Offload's performance model (§3.2, Eq 1-24) re-parameterised
for one B200, as a host-side validation tool for the resident and the
host-offloaded decode steps of this library.  No method arithmetic.

The paper models one decode step of one layer as the max of six overlapped tasks
(Eq 2), adds the (de)quantization overheads to the load/store tasks
(Eq 3-7) and sizes them from the tensor shapes (Eq 17-19)
and hardware rates (Eq 13-16, 21-24).  Two readings are provided:

* ``paper``: the equations as printed -- dequantization and quantization are
  separate passes costed as FLOP / gpu_flops + elements / gpu_mem_bw (Eq 22-24,
  the FlexGen torch-op implementation the paper profiles);
* ``fused`` (this library): the old cache is dequantized inside the attention
  kernel and the new token is quantized inside the same launch (NEXT-1), so
  Eq 6/7's dequan/quan terms cost no extra pass; the compute task is the q4
  attention kernel, modelled from measured B200 rates -- HBM bandwidth and the
  per-SMSP stage cost at the kernel's warps per SMSP plus a
  measured per-launch head.

Readings of the garbled equations (reading 18): Eq 18's "x n" makes
the "average" old cache a sum over the generation -- we use the per-step
average 2 (s + n/2) h1 bls; Eq 17's (s+1) is taken as printed for the prefill;
``num_pre_cache`` in Eq 24 is Eq 18's old_kv_cache; "qpu mem bw" is gpu_mem_bw.
Element counts are converted to bytes with the format's 0.5625 B/element (q4)
or 2 B (fp16).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

from . import configs as C

Q4_BYTES = 0.5625     # bytes per element of the group-wise 4-bit format (codes + fp16 min/scale per 64)
F16_BYTES = 2.0


@dataclass(frozen=True)
class Hardware:
    """B200 rates (GB/s, GFLOP/s, MHz, counts); every value is a measurement cited in
    DESIGN.md §6 / MEASURED_PEAKS.json, not a fit to the steps being predicted."""
    gpu_mem_bw: float = 6554.6          # GB/s, copy (MEASURED_PEAKS.json hbm_gbs)
    pcie_h2d: float = 55.58             # GB/s, pinned host -> device (bench offload leg, round 1)
    pcie_d2h: float = 55.58             # GB/s, taken equal to H2D (Gen5 x16 is symmetric)
    gpu_flops: float = 74.4e3           # GFLOP/s fp32 FMA peak: 148 SMs x 128 lanes x 1.965 GHz x 2
    gpu_freq_mhz: float = 1965.0        # SM clock under the bench (clocks line)
    smsp: int = 592                     # 148 SMs x 4 SMSPs
    warps_per_smsp: int = 4             # resident attention warps (4 CTAs of 4 warps per SM)
    # q4 attention kernel: cycles per 32-token stage per SMSP vs busy warps per SMSP (1..4)
    # and the per-launch head, MHA and GQA-8 (scripts/smsp_probe.py, profiles/smsp_probe_r2.txt:
    # the slope / intercept between L = 256 and 768 at 592*k pairs)
    stage_cycles_mha: tuple = (1275.0, 872.0, 773.0, 777.0)
    stage_cycles_gqa: tuple = (1603.0, 1044.0, 914.0, 867.0)
    launch_head_us_mha: float = 4.1
    launch_head_us_gqa: float = 4.7
    cpu_freq_mhz: float = 2000.0        # host (weights quantized on CPU, Eq 13)
    cpu_flops: float = 500.0            # GFLOP/s host
    cpu_mem_bw: float = 100.0           # GB/s host


@dataclass(frozen=True)
class Model:
    """Shape parameters of Table 2: h1 (hidden), h2 (FFN), s, n, bls (block = batch), l."""
    h1: int
    h2: int
    s: int
    n: int
    bls: int
    l: int
    kv_heads: int = 0
    head_dim: int = 128
    group_ratio: int = 1

    @staticmethod
    def from_workload(w: C.Workload, batch: int | None = None) -> "Model":
        return Model(h1=w.kv_heads * w.head_dim, h2=4 * w.hidden, s=w.prompt, n=w.gen,
                     bls=w.batch if batch is None else batch, l=w.layers, kv_heads=w.kv_heads,
                     head_dim=w.head_dim, group_ratio=w.group_ratio)


# ------------------------------------------------------------ sizes (Eq 17-19)

def num_weights(m: Model) -> int:
    """4 h1^2 + 2 h1 h2."""
    return 4 * m.h1 * m.h1 + 2 * m.h1 * m.h2


def pf_kv_cache(m: Model) -> float:
    """Eq 17: 2 (s+1) h1 bls elements (K and V of the prompt)."""
    return 2 * (m.s + 1) * m.h1 * m.bls


def old_kv_cache(m: Model) -> float:
    """Eq 18 per decode step (reading 18): 2 (s + n/2) h1 bls elements."""
    return 2 * (m.s + m.n / 2) * m.h1 * m.bls


def new_kv_cache(m: Model) -> float:
    """Eq 19 per decode step: 2 h1 bls elements (the new token's K and V)."""
    return 2 * m.h1 * m.bls


# ------------------------------------------------------ (de)quantization terms

def quan_gpu(m: Model, elements: float, hw: Hardware) -> float:
    """Eq 20-23 for a tensor quantized on the GPU (seconds): minmax (Eq 21) + norm
    (Eq 22, 3 FLOP/element) + postprocess (Eq 23, a memory pass)."""
    minmax = elements / (hw.gpu_freq_mhz * 1e6) / hw.smsp / 32       # one element per lane-cycle
    norm = elements * 3 / (hw.gpu_flops * 1e9)
    post = elements * F16_BYTES / (hw.gpu_mem_bw * 1e9)
    return minmax + norm + post


def dequan_gpu(m: Model, elements: float, hw: Hardware) -> float:
    """Eq 24 (and Eq 16 on the GPU): de_norm + de_postprocess, no min/max."""
    return elements * 3 / (hw.gpu_flops * 1e9) + elements * F16_BYTES / (hw.gpu_mem_bw * 1e9)


def quan_pf_wgt(m: Model, wc: float, hw: Hardware) -> float:
    """Eq 12-15: weights quantized once on the CPU (wc = fraction on CPU)."""
    nw = num_weights(m) * wc
    return nw / (hw.cpu_freq_mhz * 1e6) + nw * 3 / (hw.cpu_flops * 1e9) + nw * F16_BYTES / (hw.cpu_mem_bw * 1e9)


def dequan_wgt(m: Model, hw: Hardware) -> float:
    """Eq 16 on the GPU per decode step (every layer's weights are dequantized)."""
    return dequan_gpu(m, num_weights(m), hw)


# ------------------------------------------------------------ attention kernel

def attention_team_size(pairs: int, hw: Hardware) -> int:
    """The library's default team size (decode_attn.cu choose_team): the smallest
    T in 1, 2, 4 with pairs * T >= 0.35 of the resident warps."""
    warps = hw.smsp * hw.warps_per_smsp
    for T in (1, 2):
        if pairs * T >= 0.35 * warps:
            return T
    return 4


def attention_kernel_s(m: Model, L: int, hw: Hardware, batch: int | None = None) -> float:
    """The fused q4 attention launch of one layer at length L (seconds): the slower of
    the HBM stream (q4 K+V rows, q, fp32 out) and the per-SMSP issue bound, plus the
    head.  Work placement follows the library: each (sequence, kv head) pair is
    split over a team of T warps (attention_team_size), each warp taking
    ceil(stages / T) 32-token stages; the busiest SMSP runs ceil(pieces / SMSPs)
    pieces at the measured stage cost for that many busy warps."""
    b = m.bls if batch is None else batch
    pairs = b * m.kv_heads
    stages = math.ceil(L / 32)
    by = pairs * L * 2 * m.head_dim * Q4_BYTES + b * m.kv_heads * m.group_ratio * m.head_dim * 6
    t_hbm = by / (hw.gpu_mem_bw * 1e9)
    T = attention_team_size(pairs, hw)
    per_smsp = math.ceil(pairs * T / hw.smsp)              # pieces on the busiest SMSP
    busy = min(4, per_smsp)
    cyc = (hw.stage_cycles_mha if m.group_ratio == 1 else hw.stage_cycles_gqa)[busy - 1]
    t_issue = per_smsp * math.ceil(stages / T) * cyc / (hw.gpu_freq_mhz * 1e6)
    head = hw.launch_head_us_mha if m.group_ratio == 1 else hw.launch_head_us_gqa
    return max(t_hbm, t_issue) + head * 1e-6


def strong_scaling_attention_s(w: C.Workload, n_gpus: int, L: int | None = None,
                               hw: Hardware | None = None) -> float:
    """One rank's attention launch when the global batch is split over n_gpus
    (dist.shard 'strong': the largest shard is ceil(B / N) sequences)."""
    hw = hw or Hardware()
    L = w.prompt + w.gen // 2 if L is None else L
    return attention_kernel_s(Model.from_workload(w), L, hw, batch=-(-w.batch // n_gpus))


# ------------------------------------------------------------------ Eq 1-7

@dataclass
class StepBreakdown:
    load_weight: float = 0.0
    load_cache: float = 0.0
    load_activation: float = 0.0
    store_cache: float = 0.0
    store_activation: float = 0.0
    compute: float = 0.0
    terms: dict = field(default_factory=dict)

    def t_gen(self) -> float:
        """Eq 2: the six tasks overlap; the step of one layer takes the slowest."""
        return max(self.load_weight, self.load_cache, self.load_activation, self.store_cache,
                   self.store_activation, self.compute)


def decode_layer(m: Model, L: int, hw: Hardware, offload_kv: bool, reading: str = "fused",
                 kv_q4: bool = True) -> StepBreakdown:
    """T_gen of one layer at attention length L (Eq 2 with Eq 6-7 folded in).
    offload_kv: the KV cache lives in pinned host memory (the paper's setting, Alg 1);
    otherwise it is resident in HBM (load_cache = store_cache = 0, as with attention
    offloading in the paper's terms: the cache never crosses PCIe)."""
    bpe = Q4_BYTES if kv_q4 else F16_BYTES
    old_el = 2 * (L - 1) * m.h1 * m.bls            # rows [0, L-1) of every (b, kv head)
    new_el = new_kv_cache(m)
    st = StepBreakdown()
    st.compute = attention_kernel_s(m, L, hw)
    if reading == "paper" and kv_q4:               # separate (de)quantization passes
        st.terms["dequan_old_cache"] = dequan_gpu(m, old_el, hw)
        st.terms["quan_new_cache"] = quan_gpu(m, new_el, hw)
    else:                                          # fused into the attention launch
        st.terms["dequan_old_cache"] = 0.0
        st.terms["quan_new_cache"] = 0.0
    if offload_kv:
        st.load_cache = old_el * bpe / (hw.pcie_h2d * 1e9) + st.terms["dequan_old_cache"]   # Eq 6
        st.store_cache = new_el * bpe / (hw.pcie_d2h * 1e9) + st.terms["quan_new_cache"]    # Eq 7
    else:
        st.compute += st.terms["dequan_old_cache"] + st.terms["quan_new_cache"]
    return st


def decode_step_s(w: C.Workload, t: int, hw: Hardware | None = None, offload_kv: bool = False,
                  reading: str = "fused", batch: int | None = None) -> float:
    """One decode step (all layers) at step t (L = s + t): T_gen * l (Eq 1's decode term)."""
    hw = hw or Hardware()
    m = Model.from_workload(w, batch)
    return decode_layer(m, w.prompt + t, hw, offload_kv, reading).t_gen() * m.l


def total_time_s(w: C.Workload, hw: Hardware | None = None, offload_kv: bool = False,
                 reading: str = "fused", t_init: float = 0.0, t_pf_layer: float | None = None) -> float:
    """Eq 1: T = T_init + T_pf * l + sum over the n-1 decode steps of T_gen * l (the
    per-step length is exact here instead of Eq 18's average)."""
    hw = hw or Hardware()
    m = Model.from_workload(w)
    if t_pf_layer is None:                         # Eq 5: prefill quantization of the prompt cache
        t_pf_layer = quan_gpu(m, pf_kv_cache(m), hw)
    dec = sum(decode_step_s(w, t, hw, offload_kv, reading) for t in range(1, w.gen))
    return t_init + t_pf_layer * m.l + dec


def kv_quantization_beneficial(w: C.Workload, t: int, hw: Hardware | None = None,
                               reading: str = "paper") -> dict:
    """The paper's use case 2: compare load_cache + store_cache of the
    fp16 cache with Eq 6 + Eq 7 of the q4 cache, for the offloaded setting."""
    hw = hw or Hardware()
    m = Model.from_workload(w)
    L = w.prompt + t
    f16 = decode_layer(m, L, hw, True, reading, kv_q4=False)
    q4 = decode_layer(m, L, hw, True, reading, kv_q4=True)
    a, b = f16.load_cache + f16.store_cache, q4.load_cache + q4.store_cache
    return {"fp16_s": a, "q4_s": b, "beneficial": b < a, "speedup": a / b}
