"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no quantization, no
attention): it only defines the counter-based random generator that both
sides use to produce bit-identical fp16 K/V/q values, so that the oracle
(``oracle/``) and the CUDA path never have to exchange data.  The device
twin of this generator lives in ``csrc/gen.cu`` (``lmo_gen_fill_f16``); a GPU
test checks that the two agree bit for bit.

Recipe (DESIGN.md §"Input recipe"; SURVEY.md §8(d) "Concrete synthetic
inputs"):

* ``h = splitmix64(seed ^ (stream << 56) ^ idx)`` where ``idx`` packs the
  *global* logical coordinates ``(layer, b, head, pos, i)`` into bit fields
  (layer<<44 | b<<32 | head<<24 | pos<<12 | i), so every value is a function
  of where it sits in the full workload and not of how a rank or a test
  slices it.
* Irwin-Hall(4): ``s = sum of the four 16-bit lanes of h - 131070``; the
  value ``s * 2**-15`` lies in [-4, 4] with std ~1.155 (~N(0, 1.15^2)).
* Outlier channels (the "massive activation" feature dims of OPT/LLaMA K and
  q): channel ``i`` of (layer, kv-head) is an outlier with probability ~1/100
  (``splitmix64(seed ^ 0xA5<<56 ^ layer<<32 ^ kvh<<16 ^ i) % 100 == 0``) and
  is multiplied by 8 for the K and q streams.  V has no outliers.
* Finally rounded to fp16 (round-to-nearest-even).  ``s * 2**-15 * 8`` is
  exact in fp32, so one correctly rounded conversion gives identical bits
  on host (numpy) and device (``__float2half_rn``).

Streams: ``STREAM_K`` (prompt and generated keys share it: position is a
coordinate), ``STREAM_V``, ``STREAM_Q`` (pos field = decode step index).
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1
STREAM_K = 1
STREAM_V = 2
STREAM_Q = 3
OUTLIER_STREAM = 0xA5
OUTLIER_SCALE = 8.0

_U = np.uint64


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser over uint64 arrays (wraps mod 2**64)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + _U(0x9E3779B97F4A7C15)
        z = (z ^ (z >> _U(30))) * _U(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> _U(27))) * _U(0x94D049BB133111EB)
    return z ^ (z >> _U(31))


def pack_index(layer, b, head, pos, i) -> np.ndarray:
    """Bit-field index of a global coordinate (limits asserted)."""
    layer = np.asarray(layer, dtype=np.uint64)
    b = np.asarray(b, dtype=np.uint64)
    head = np.asarray(head, dtype=np.uint64)
    pos = np.asarray(pos, dtype=np.uint64)
    i = np.asarray(i, dtype=np.uint64)
    return (layer << _U(44)) | (b << _U(32)) | (head << _U(24)) | (pos << _U(12)) | i


def check_limits(layer: int, b_max: int, head_max: int, pos_max: int, dim: int) -> None:
    if not (0 <= layer < 256 and b_max <= 4096 and head_max <= 256 and pos_max <= 4096 and dim <= 4096):
        raise ValueError("coordinate outside the generator's bit fields")


def outlier_mask(seed: int, layer: int, kvh, i) -> np.ndarray:
    """True where channel i of (layer, kv-head kvh) is an outlier channel."""
    kvh = np.asarray(kvh, dtype=np.uint64)
    i = np.asarray(i, dtype=np.uint64)
    key = (_U(seed) ^ (_U(OUTLIER_STREAM) << _U(56)) ^ (_U(layer) << _U(32))
           ^ (kvh << _U(16)) ^ i)
    return (splitmix64(key) % _U(100)) == _U(0)


def irwin_hall4(h: np.ndarray) -> np.ndarray:
    """Centred sum of the four 16-bit lanes of h, as float64 times 2**-15."""
    m = _U(0xFFFF)
    s = ((h & m).astype(np.int64) + ((h >> _U(16)) & m).astype(np.int64)
         + ((h >> _U(32)) & m).astype(np.int64) + ((h >> _U(48)) & m).astype(np.int64))
    return (s - 131070).astype(np.float64) * (2.0 ** -15)


def gen_f16(seed: int, stream: int, layer: int, b0: int, nb: int, h0: int, nh: int,
            p0: int, npos: int, dim: int, group: int = 1) -> np.ndarray:
    """fp16 array [nb][nh][npos][dim] of the logical tensor box starting at
    (b0, h0, p0).  ``group`` maps a head to its kv-head for the outlier mask
    (q heads: group = Hq/Hkv; K/V: 1)."""
    check_limits(layer, b0 + nb, h0 + nh, p0 + npos, dim)
    b = np.arange(b0, b0 + nb, dtype=np.uint64)[:, None, None, None]
    h = np.arange(h0, h0 + nh, dtype=np.uint64)[None, :, None, None]
    p = np.arange(p0, p0 + npos, dtype=np.uint64)[None, None, :, None]
    i = np.arange(dim, dtype=np.uint64)[None, None, None, :]
    idx = pack_index(layer, b, h, p, i)
    hsh = splitmix64(_U(seed) ^ (_U(stream) << _U(56)) ^ idx)
    val = irwin_hall4(hsh)
    if stream in (STREAM_K, STREAM_Q):
        kvh = h // _U(group)
        val = np.where(outlier_mask(seed, layer, kvh, i), val * OUTLIER_SCALE, val)
    # val is exact in float32 (<= 18 significant bits), so float32 -> float16
    # is one correctly rounded (RN-even) conversion, as on the device.
    return val.astype(np.float32).astype(np.float16)


def seed_for_config(index: int) -> int:
    """One seed per BASELINE.json config."""
    return 0x4C4D4F00 + index


def uniform_f16(rng: np.random.Generator, shape, lo: float, hi: float) -> np.ndarray:
    """Plain numpy helper for test fixtures (edge-case groups)."""
    return rng.uniform(lo, hi, size=shape).astype(np.float16)
