"""TEST INFRASTRUCTURE: numpy-facing ctypes wrapper of ``liblmo_oracle.so``.

Each function restates the paper passage it follows; the arithmetic itself is
in ``lmo_oracle.c`` (plain C, fp64).  Parity unpinned: none -- every function
here is pinned by tests/test_oracle_pins.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "lmo_oracle.c")
LIB = os.path.join(HERE, "liblmo_oracle.so")
CFLAGS = ["-O2", "-std=c11", "-fno-fast-math", "-ffp-contract=off", "-shared", "-fPIC",
          "-Wall", "-Wextra", "-pthread"]

__all__ = ["build", "lib", "h2d", "rn16", "ru16", "quantize_groupwise", "dequantize_groupwise",
           "kv_append_quant", "decode_attention_q4", "new_cache", "w4a16_linear"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (idempotent)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + ".tmp"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, SRC, "-lm"])
        os.replace(tmp, LIB)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        P = ctypes.c_void_p
        i64, i32 = ctypes.c_int64, ctypes.c_int
        L.lmo_oracle_h2d.argtypes = [ctypes.c_uint16]
        L.lmo_oracle_h2d.restype = ctypes.c_double
        L.lmo_oracle_rn16.argtypes = [ctypes.c_double]
        L.lmo_oracle_rn16.restype = ctypes.c_uint16
        L.lmo_oracle_ru16.argtypes = [ctypes.c_double]
        L.lmo_oracle_ru16.restype = ctypes.c_uint16
        L.lmo_oracle_quantize_groupwise.argtypes = [P, i64, i64, i64, i32, i32, P, P]
        L.lmo_oracle_dequantize_groupwise.argtypes = [P, P, i64, i64, i64, i32, i32, P]
        L.lmo_oracle_kv_append_quant.argtypes = [P, P, P, P, i32, i32, i32, i32, P, P, i32, P]
        L.lmo_oracle_decode_attention_q4_mt.argtypes = [P, P, P, P, i32, i32, i32, i32, P, i32, P,
                                                        ctypes.c_double, P, i32]
        L.lmo_oracle_w4a16_linear.argtypes = [P, P, i64, i64, i32, P, i64, P]
        L.lmo_oracle_decode_attention_q4_ext.argtypes = [P, P, P, P, i32, i32, i32, i32, P, i32, P, P, P,
                                                         ctypes.c_double, P, i32]
        for f in ("lmo_oracle_quantize_groupwise", "lmo_oracle_dequantize_groupwise", "lmo_oracle_w4a16_linear",
                  "lmo_oracle_kv_append_quant", "lmo_oracle_decode_attention_q4_mt",
                  "lmo_oracle_decode_attention_q4_ext"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.c_void_p)


def _bits(x: np.ndarray) -> np.ndarray:
    """fp16 array (or uint16 bit patterns) -> contiguous uint16 bits."""
    x = np.ascontiguousarray(x)
    if x.dtype == np.float16:
        return x.view(np.uint16)
    assert x.dtype == np.uint16
    return x


def h2d(bits: int) -> float:
    return lib().lmo_oracle_h2d(int(bits))


def rn16(x: float) -> int:
    return int(lib().lmo_oracle_rn16(float(x)))


def ru16(x: float) -> int:
    return int(lib().lmo_oracle_ru16(float(x)))


def quantize_groupwise(x: np.ndarray, outer: int, n: int, inner: int, bits: int = 4,
                       group: int = 64):
    """Alg 2 "Compress(tensor, target_bits, quantize_dim)" (PAPER.md P:263-284,
    Eq 10) on x viewed as (outer, n, inner), groups along n.
    Returns (codes uint8 (outer, n_pad/2, inner), meta uint16 (outer, ngroups, inner, 2))."""
    xb = _bits(x).reshape(-1)
    assert xb.size == outer * n * inner
    ng = (n + group - 1) // group
    codes = np.zeros((outer, ng * group // 2, inner), dtype=np.uint8)
    meta = np.zeros((outer, ng, inner, 2), dtype=np.uint16)
    rc = lib().lmo_oracle_quantize_groupwise(_ptr(xb), outer, n, inner, bits, group,
                                             _ptr(codes), _ptr(meta))
    if rc:
        raise ValueError("oracle quantize: invalid arguments")
    return codes, meta


def dequantize_groupwise(codes: np.ndarray, meta: np.ndarray, outer: int, n: int, inner: int,
                         bits: int = 4, group: int = 64) -> np.ndarray:
    """Eq 11 in step form y = RN16(RN32(c*scale + min));
    returns fp16 (outer, n, inner)."""
    codes = np.ascontiguousarray(codes, dtype=np.uint8)
    meta = np.ascontiguousarray(meta, dtype=np.uint16)
    y = np.zeros((outer, n, inner), dtype=np.uint16)
    rc = lib().lmo_oracle_dequantize_groupwise(_ptr(codes), _ptr(meta), outer, n, inner, bits,
                                               group, _ptr(y))
    if rc:
        raise ValueError("oracle dequantize: invalid arguments")
    return y.view(np.float16)


def new_cache(B: int, Hkv: int, cap: int, d: int, fill: int = 0):
    """Host q4 KV cache in the library layout: dict of codes/meta arrays."""
    ng = d // 64
    mfill = fill | (fill << 8)
    return {
        "k_codes": np.full((B, Hkv, cap, d // 2), fill, dtype=np.uint8),
        "v_codes": np.full((B, Hkv, cap, d // 2), fill, dtype=np.uint8),
        "k_meta": np.full((B, Hkv, cap, ng, 2), mfill, dtype=np.uint16),
        "v_meta": np.full((B, Hkv, cap, ng, 2), mfill, dtype=np.uint16),
    }


def kv_append_quant(cache: dict, k_new: np.ndarray, v_new: np.ndarray, pos) -> None:
    """Concatenate the new tokens' K/V into the cache, quantizing them
    (Eq 7): row-wise Alg 2 along head_dim into slots pos[b]+t."""
    B, Hkv, cap, half = cache["k_codes"].shape
    d = half * 2
    n_new = k_new.shape[2]
    assert k_new.shape == (B, Hkv, n_new, d) and v_new.shape == k_new.shape
    pos = np.ascontiguousarray(np.broadcast_to(np.asarray(pos, dtype=np.int32), (B,)))
    kb, vb = _bits(k_new), _bits(v_new)
    rc = lib().lmo_oracle_kv_append_quant(_ptr(cache["k_codes"]), _ptr(cache["k_meta"]),
                                          _ptr(cache["v_codes"]), _ptr(cache["v_meta"]), B, Hkv,
                                          cap, d, _ptr(kb), _ptr(vb), n_new, _ptr(pos))
    if rc:
        raise ValueError("oracle append: invalid arguments")


def decode_attention_q4(cache: dict, q: np.ndarray, lens, sigma: float | None = None,
                        nthreads: int = 1, k_last: np.ndarray | None = None,
                        v_last: np.ndarray | None = None) -> np.ndarray:
    """softmax(sigma * q K^T) V over the exact dequantized q4 cache,
    kv head = h // (Hq/Hkv).  q: fp16 [B][Hq][d]; returns float64 [B][Hq][d].
    k_last/v_last (reading 13b, FlexGen-exact, T6): raw fp16 [B][Hkv][d] K/V used for
    token L_b-1 of every (b, kv head) instead of its quantized cache slot."""
    B, Hkv, cap, half = cache["k_codes"].shape
    d = half * 2
    Hq = q.shape[1]
    assert q.shape == (B, Hq, d)
    if sigma is None:
        sigma = 1.0 / np.sqrt(d)
    lens = np.ascontiguousarray(np.broadcast_to(np.asarray(lens, dtype=np.int32), (B,)))
    qb = _bits(q)
    out = np.zeros((B, Hq, d), dtype=np.float64)
    kl = vl = None
    if k_last is not None or v_last is not None:
        kl = _bits(np.asarray(k_last, dtype=np.float16).reshape(B, Hkv, d))
        vl = _bits(np.asarray(v_last, dtype=np.float16).reshape(B, Hkv, d))
    rc = lib().lmo_oracle_decode_attention_q4_ext(
        _ptr(cache["k_codes"]), _ptr(cache["k_meta"]), _ptr(cache["v_codes"]),
        _ptr(cache["v_meta"]), B, Hkv, cap, d, _ptr(qb), Hq, _ptr(lens),
        None if kl is None else _ptr(kl), None if vl is None else _ptr(vl), float(sigma), _ptr(out),
        int(nthreads))
    if rc:
        raise ValueError("oracle attention: invalid arguments")
    return out


def w4a16_linear(codes: np.ndarray, meta: np.ndarray, N: int, K: int, x: np.ndarray,
                 group: int = 64) -> np.ndarray:
    """A linear layer over q4 weights (NEXT-3): y = x W~^T with W~ the Eq 11 / D1
    dequantization of W [N][K] quantized along K -- the paper's per-step
    "dequan_wgt" then matmul (Eq 4).  x fp16 [B][K];
    returns float64 [B][N]."""
    codes = np.ascontiguousarray(codes, dtype=np.uint8)
    meta = np.ascontiguousarray(meta, dtype=np.uint16)
    xb = _bits(x)
    B = xb.size // K
    assert xb.size == B * K
    y = np.zeros((B, N), dtype=np.float64)
    rc = lib().lmo_oracle_w4a16_linear(_ptr(codes), _ptr(meta), N, K, group, _ptr(xb), B, _ptr(y))
    if rc:
        raise ValueError("oracle w4a16: invalid arguments")
    return y
