"""Workload shapes (BASELINE.json ``configs``) and algorithmic byte accounting.

Host logic only; no kernel arithmetic.  Byte formulas follow SURVEY.md §8(d)
and are pinned in ``tests/test_configs.py`` against the sizes the paper
prints (PAPER.md P:29 / P:99 "KV cache ... 157GB ... weights ... 55GB" for
OPT-30B, s=64, n=128, block 640; Table 1 P:121 "KV cache (new) 0.8 GB").

Storage of the 4-bit group-wise format (Alg 2):
``d/2`` code bytes + ``d/64`` groups x 4 B (fp16 min, fp16 scale) per row of
``d`` elements, i.e. 0.5625 B/element.
"""
from __future__ import annotations

from dataclasses import dataclass, asdict

GROUP = 64
BITS = 4
CAP_ALIGN = 16  # cache capacity is rounded up to a multiple of the 16-token block


@dataclass(frozen=True)
class Workload:
    key: str
    name: str
    layers: int
    batch: int
    q_heads: int
    kv_heads: int
    head_dim: int
    prompt: int          # s
    gen: int             # n (generation length)
    hidden: int = 0      # h1, for the weight-dequant leg (c3)
    index: int = 0       # position in BASELINE.json configs (seed)

    @property
    def group_ratio(self) -> int:
        return self.q_heads // self.kv_heads

    @property
    def steps(self) -> int:
        """Decode steps per sequence: n-1 (Eq 1)."""
        return self.gen - 1

    @property
    def max_len(self) -> int:
        """Cache capacity s+n-1 (pinned by the 157 GB figure)."""
        return self.prompt + self.gen - 1

    @property
    def capacity(self) -> int:
        return round_up(self.max_len, CAP_ALIGN)

    def len_at_step(self, t: int) -> int:
        """Attention length at decode step t = 1..n-1: L = s + t."""
        return self.prompt + t

    def as_dict(self):
        return asdict(self)


def round_up(x: int, m: int) -> int:
    return (x + m - 1) // m * m


CONFIGS = {
    "c1": Workload("c1", "OPT-125M-shaped tiny", layers=1, batch=4, q_heads=12, kv_heads=12,
                   head_dim=64, prompt=64, gen=8, hidden=768, index=0),
    "c2": Workload("c2", "OPT-6.7B-shaped", layers=32, batch=32, q_heads=32, kv_heads=32,
                   head_dim=128, prompt=512, gen=32, hidden=4096, index=1),
    "c3": Workload("c3", "OPT-30B-shaped (paper workload)", layers=48, batch=64, q_heads=56,
                   kv_heads=56, head_dim=128, prompt=64, gen=128, hidden=7168, index=2),
    "c4": Workload("c4", "OPT-66B-shaped", layers=64, batch=64, q_heads=72, kv_heads=72,
                   head_dim=128, prompt=512, gen=32, hidden=9216, index=3),
    "c5": Workload("c5", "LLaMA-2-70B-shaped GQA", layers=80, batch=128, q_heads=64, kv_heads=8,
                   head_dim=128, prompt=1024, gen=128, hidden=8192, index=4),
}


# ---------------------------------------------------------------- bytes ----

def q4_row_bytes(d: int) -> float:
    """Packed bytes of one d-element row: codes + (min, scale) fp16 per group."""
    ngroups = (d + GROUP - 1) // GROUP
    return d / 2 + 4 * ngroups


def kv_cache_bytes_fp16(layers: int, hidden: int, max_len: int, block: int) -> int:
    """Unquantized fp16 K+V cache: 2 (K,V) x l x (s+n-1) x h1 x bls x 2 B."""
    return 2 * layers * max_len * hidden * block * 2


def weight_bytes_fp16(layers: int, hidden: int, vocab: int) -> int:
    """fp16 weights: l x (4 h1^2 + 2 h1 h2) with h2 = 4 h1, plus
    the token embedding vocab x h1."""
    per_layer = 4 * hidden * hidden + 2 * hidden * (4 * hidden)
    return 2 * (layers * per_layer + vocab * hidden)


def new_kv_bytes_fp16_per_token(layers: int, hidden: int, block: int) -> int:
    """New K+V per generated token over all layers: 2 x h1 x bls x 2 B x l."""
    return 2 * hidden * block * 2 * layers


def attention_kv_bytes(w: Workload, L: int, batch: int | None = None) -> float:
    """q4 K+V bytes one decode-attention launch reads at length L."""
    b = w.batch if batch is None else batch
    return 2 * b * w.kv_heads * L * q4_row_bytes(w.head_dim)


def attention_launch_bytes(w: Workload, L: int, batch: int | None = None, out_bytes: int = 4) -> float:
    """Algorithmic bytes of one decode-attention launch: q4 KV + q read + out write."""
    b = w.batch if batch is None else batch
    return attention_kv_bytes(w, L, b) + b * w.q_heads * w.head_dim * (2 + out_bytes)


def append_launch_bytes(w: Workload, batch: int | None = None, n_new: int = 1) -> float:
    """Append-quantize of n_new tokens: read fp16 K,V; write q4 K,V."""
    b = w.batch if batch is None else batch
    rows = 2 * b * w.kv_heads * n_new
    return rows * (2 * w.head_dim + q4_row_bytes(w.head_dim))


def layer_step_bytes(w: Workload, L: int, batch: int | None = None, out_bytes: int = 4) -> float:
    return attention_launch_bytes(w, L, batch, out_bytes) + append_launch_bytes(w, batch)


def weight_dequant_bytes_per_layer(w: Workload) -> float:
    """c3 weight leg: read q4 weights (0.5625 B/el), write fp16 (2 B/el)."""
    n = 4 * w.hidden * w.hidden + 2 * w.hidden * (4 * w.hidden)
    return n * (0.5625 + 2.0)
