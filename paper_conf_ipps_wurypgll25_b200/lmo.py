"""Thin ctypes binding of liblmo.so (include/lmo.h) -- argument marshalling only.

Every step of the path runs in the library's CUDA kernels; this module only
turns torch tensors into (device pointer, size) arguments, passes the current
CUDA stream, and raises on a non-OK status.  There is no CPU fallback: if the
library is missing or cannot be loaded, importing this module raises.
"""
from __future__ import annotations

import ctypes
import math
import os
from dataclasses import dataclass

import torch

from . import build as _build

LMO_OK, LMO_ERR_NULL, LMO_ERR_SHAPE, LMO_ERR_UNSUPPORTED, LMO_ERR_ALIGN, LMO_ERR_WORKSPACE, \
    LMO_ERR_CUDA = range(7)
LMO_F16, LMO_F32 = 0, 1
LMO_STEP_CACHE_STABLE = 1
LMO_STEP_FLEXGEN_EXACT = 2  # the new token attends with its raw fp16 K/V (include/lmo.h)
LMO_SPLITS_STREAMK = -1   # num_splits value selecting the stream-K schedule
LMO_SPLITS_SMTEAM = -2    # num_splits value selecting the SM-team schedule
GROUP = 64


class LmoError(RuntimeError):
    def __init__(self, status: int, fn: str):
        super().__init__(f"{fn}: {_lib.lmo_status_string(status).decode()}")
        self.status = status


class lmo_kv_cache(ctypes.Structure):
    _fields_ = [("kv", ctypes.c_void_p), ("batch", ctypes.c_int32), ("kv_heads", ctypes.c_int32),
                ("capacity", ctypes.c_int32), ("head_dim", ctypes.c_int32)]


def _load():
    path = os.environ.get("LMO_LIB") or _build.LIB   # LMO_LIB: alternate build (experiments)
    if not os.path.exists(path):
        raise ImportError(f"liblmo.so not built ({path}); run __graft_entry__.build()")
    L = ctypes.CDLL(path)
    P, i64, i32, u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64
    sig = {
        "lmo_quantize_groupwise": [P, i64, i64, i64, ctypes.c_int, ctypes.c_int, P, P, P],
        "lmo_dequantize_groupwise": [P, P, i64, i64, i64, ctypes.c_int, ctypes.c_int, P, P],
        "lmo_kv_append_quant": [ctypes.POINTER(lmo_kv_cache), P, P, i32, i32, P, P],
        "lmo_decode_attention_q4": [ctypes.POINTER(lmo_kv_cache), P, i32, i32, P, ctypes.c_float,
                                    i32, P, ctypes.c_int, P, ctypes.c_size_t, P],
        "lmo_gen_fill_f16": [P, i32, i32, i32, i32, u64, i32, i32, i32, i32, i32, i32, P],
        "lmo_w4a16_linear": [P, P, i64, i64, P, i32, P, i32, P],
        "lmo_w4a16_pack": [P, P, i64, i64, P, P],
        "lmo_w4a16_linear_packed": [P, i64, i64, P, i32, P, i32, P],
        "lmo_probe_read_stream": [P, ctypes.c_size_t, P, P],
        "lmo_decode_step_q4": [ctypes.POINTER(lmo_kv_cache), P, P, P, i32, i32, P, ctypes.c_float,
                               i32, P, ctypes.c_int, P, ctypes.c_size_t, ctypes.c_uint32, P],
    }
    alt = bool(os.environ.get("LMO_LIB"))
    for name, args in sig.items():
        if alt and not hasattr(L, name):   # an older experimental build: skip symbols it lacks
            continue
        f = getattr(L, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    L.lmo_offload_ring_bytes.argtypes = [ctypes.POINTER(lmo_kv_cache), i32]
    L.lmo_offload_ring_bytes.restype = ctypes.c_size_t
    L.lmo_offload_create.argtypes = [ctypes.POINTER(lmo_kv_cache), i32, P, P, i32, ctypes.POINTER(P)]
    L.lmo_offload_create.restype = ctypes.c_int
    L.lmo_offload_decode_step.argtypes = [P, P, P, P, i32, i32, ctypes.c_float, i32, P, ctypes.c_int,
                                          P, ctypes.c_size_t, P]
    L.lmo_offload_decode_step.restype = ctypes.c_int
    L.lmo_offload_destroy.argtypes = [P]
    L.lmo_offload_destroy.restype = ctypes.c_int
    L.lmo_decode_attention_workspace_bytes.argtypes = [i32, i32, i32, i32, i32]
    L.lmo_decode_attention_workspace_bytes.restype = ctypes.c_size_t
    L.lmo_status_string.argtypes = [ctypes.c_int]
    L.lmo_status_string.restype = ctypes.c_char_p
    L.lmo_w4a16_packed_bytes.argtypes = [i64, i64]
    L.lmo_w4a16_packed_bytes.restype = ctypes.c_size_t
    L.lmo_kv_row_bytes.argtypes = [i32]
    L.lmo_kv_row_bytes.restype = ctypes.c_size_t
    L.lmo_launch_count.argtypes = []
    L.lmo_launch_count.restype = ctypes.c_uint64
    L.lmo_version.argtypes = []
    L.lmo_version.restype = ctypes.c_uint32
    return L


_lib = _load()
LIB_PATH = _build.LIB
EXPORTS = ["lmo_quantize_groupwise", "lmo_dequantize_groupwise", "lmo_kv_append_quant",
           "lmo_kv_row_bytes",
           "lmo_decode_attention_workspace_bytes", "lmo_decode_attention_q4", "lmo_decode_step_q4",
           "lmo_status_string",
           "lmo_gen_fill_f16", "lmo_launch_count", "lmo_version",
           "lmo_offload_ring_bytes", "lmo_offload_create", "lmo_offload_decode_step",
           "lmo_offload_destroy", "lmo_w4a16_linear", "lmo_w4a16_packed_bytes", "lmo_w4a16_pack",
           "lmo_w4a16_linear_packed", "lmo_probe_read_stream"]


def _check(status: int, fn: str) -> None:
    if status != LMO_OK:
        raise LmoError(status, fn)


def _ptr(t: torch.Tensor | None):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _need_cuda(*ts):
    for t in ts:
        if t is not None and (not t.is_cuda or not t.is_contiguous()):
            raise ValueError("liblmo expects contiguous CUDA tensors")


def launch_count() -> int:
    return int(_lib.lmo_launch_count())


# ---------------------------------------------------------------- A1 / A5

def lmo_quantize_groupwise(x: torch.Tensor, outer: int, n: int, inner: int,
                           codes: torch.Tensor | None = None, meta: torch.Tensor | None = None,
                           bits: int = 4, group_size: int = GROUP, stream=None):
    """Alg 2 / Eq 10 on x (fp16) viewed as (outer, n, inner).
    Returns (codes uint8 (outer, n_pad/2, inner), meta int32 (outer, n_pad/64, inner))."""
    ng = (n + group_size - 1) // group_size
    if codes is None:
        codes = torch.empty((outer, ng * group_size // 2, inner), dtype=torch.uint8, device=x.device)
    if meta is None:
        meta = torch.empty((outer, ng, inner), dtype=torch.int32, device=x.device)
    _need_cuda(x, codes, meta)
    assert x.dtype == torch.float16 and x.numel() == outer * n * inner
    _check(_lib.lmo_quantize_groupwise(_ptr(x), outer, n, inner, bits, group_size, _ptr(codes),
                                       _ptr(meta), _stream(stream)), "lmo_quantize_groupwise")
    return codes, meta


def lmo_dequantize_groupwise(codes: torch.Tensor, meta: torch.Tensor, outer: int, n: int,
                             inner: int, y: torch.Tensor | None = None, bits: int = 4,
                             group_size: int = GROUP, stream=None) -> torch.Tensor:
    """Eq 11 -> fp16 (outer, n, inner)."""
    if y is None:
        y = torch.empty((outer, n, inner), dtype=torch.float16, device=codes.device)
    _need_cuda(codes, meta, y)
    _check(_lib.lmo_dequantize_groupwise(_ptr(codes), _ptr(meta), outer, n, inner, bits,
                                         group_size, _ptr(y), _stream(stream)),
           "lmo_dequantize_groupwise")
    return y


def lmo_w4a16_linear(codes: torch.Tensor, meta: torch.Tensor, N: int, K: int, x: torch.Tensor,
                     y: torch.Tensor | None = None, k_split: int = 0, stream=None) -> torch.Tensor:
    """NEXT-3: y = x W~^T over q4 weights W [N][K] quantized along K (Eq 4's
    load_weight + dequan_wgt then matmul), fused on the tensor cores.
    x fp16 [batch][K]; returns fp32 [batch][N]."""
    batch = x.numel() // K
    if y is None:
        y = torch.empty((batch, N), dtype=torch.float32, device=x.device)
    _need_cuda(codes, meta, x, y)
    _check(_lib.lmo_w4a16_linear(_ptr(codes), _ptr(meta), N, K, _ptr(x), batch, _ptr(y), k_split,
                                 _stream(stream)), "lmo_w4a16_linear")
    return y


def lmo_w4a16_pack(codes: torch.Tensor, meta: torch.Tensor, N: int, K: int, stream=None) -> torch.Tensor:
    """Once-per-weight repack into the GEMM's streaming layout (include/lmo.h)."""
    nbytes = _lib.lmo_w4a16_packed_bytes(N, K)
    if nbytes == 0:
        raise LmoError(LMO_ERR_SHAPE, "lmo_w4a16_packed_bytes")
    packed = torch.empty(nbytes, dtype=torch.uint8, device=codes.device)
    _need_cuda(codes, meta, packed)
    _check(_lib.lmo_w4a16_pack(_ptr(codes), _ptr(meta), N, K, _ptr(packed), _stream(stream)), "lmo_w4a16_pack")
    return packed


def lmo_w4a16_linear_packed(packed: torch.Tensor, N: int, K: int, x: torch.Tensor,
                            y: torch.Tensor | None = None, k_split: int = 0, stream=None) -> torch.Tensor:
    """lmo_w4a16_linear on weights in the packed streaming layout."""
    batch = x.numel() // K
    if y is None:
        y = torch.empty((batch, N), dtype=torch.float32, device=x.device)
    _need_cuda(packed, x, y)
    _check(_lib.lmo_w4a16_linear_packed(_ptr(packed), N, K, _ptr(x), batch, _ptr(y), k_split, _stream(stream)),
           "lmo_w4a16_linear_packed")
    return y


# ------------------------------------------------------------ KV cache ----

def row_bytes(head_dim: int) -> int:
    """Compressed K+V token row: K codes | K meta | V codes | V meta."""
    return 2 * (head_dim // 2 + 4 * (head_dim // GROUP))


@dataclass
class KVCache:
    """One layer's q4 KV cache in the library layout (torch owns the memory):
    kv [B][Hkv][cap][row_bytes] uint8, one compressed K+V row per token slot."""
    kv: torch.Tensor
    batch: int
    kv_heads: int
    capacity: int
    head_dim: int

    @staticmethod
    def empty(batch: int, kv_heads: int, capacity: int, head_dim: int, device="cuda",
              zero: bool = False) -> "KVCache":
        cap = (capacity + 15) // 16 * 16
        alloc = torch.zeros if zero else torch.empty
        kv = alloc((batch, kv_heads, cap, row_bytes(head_dim)), dtype=torch.uint8, device=device)
        return KVCache(kv, batch, kv_heads, cap, head_dim)

    def abi(self) -> lmo_kv_cache:
        return lmo_kv_cache(self.kv.data_ptr(), self.batch, self.kv_heads, self.capacity,
                            self.head_dim)

    def nbytes(self) -> int:
        return self.kv.numel()

    # field views (strided): K codes [B][Hkv][cap][d/2] u8, meta [B][Hkv][cap][d/64] as
    # int32 bytes.  The V codes are pair-interleaved (include/lmo.h): no per-token view.
    def field(self, name: str) -> torch.Tensor:
        rb, mb = self.head_dim // 2, 4 * (self.head_dim // GROUP)
        if name == "v_codes":
            raise ValueError("V codes are stored pair-interleaved; use to_host_fields()")
        off = {"k_codes": (0, rb), "k_meta": (rb, mb), "v_meta": (2 * rb + mb, mb)}[name]
        return self.kv[..., off[0]:off[0] + off[1]]

    def to_host_fields(self):
        """Copy to host as the oracle's field arrays: codes uint8 [B][Hkv][cap][d/2],
        meta uint16 [B][Hkv][cap][d/64][2] ({min, scale} bit patterns).  The V codes are
        de-interleaved from the pair layout: the V areas of rows 2p, 2p+1 hold the 16-bit
        4-dim chunks of tokens 2p (low half of each word) and 2p+1 (high half)."""
        import numpy as np
        kv = self.kv.cpu().numpy()
        rb, ng = self.head_dim // 2, self.head_dim // GROUP
        out = {}
        for name in ("k_codes", "k_meta", "v_codes", "v_meta"):
            off = {"k_codes": 0, "k_meta": rb, "v_codes": rb + 4 * ng, "v_meta": 2 * rb + 4 * ng}[name]
            if name == "k_codes":
                out[name] = np.ascontiguousarray(kv[..., off:off + rb])
            elif name == "v_codes":
                B, H, cap = kv.shape[:3]
                area = np.ascontiguousarray(kv[..., off:off + rb]).reshape(B, H, cap // 2, 2 * rb)
                w = area.view(np.uint16)                               # [B][H][pairs][d/4 words x 2 halves]
                v = np.empty((B, H, cap // 2, 2, rb), np.uint8)
                v[:, :, :, 0] = np.ascontiguousarray(w[..., 0::2]).view(np.uint8)
                v[:, :, :, 1] = np.ascontiguousarray(w[..., 1::2]).view(np.uint8)
                out[name] = v.reshape(B, H, cap, rb)
            else:
                m = np.ascontiguousarray(kv[..., off:off + 4 * ng])
                out[name] = m.view(np.uint16).reshape(*m.shape[:-1], ng, 2)
        return out


def lmo_kv_append_quant(cache: KVCache, k_new: torch.Tensor, v_new: torch.Tensor, pos0: int = 0,
                        pos_dev: torch.Tensor | None = None, stream=None, abi=None) -> None:
    """Append-quantize k_new/v_new [B][Hkv][n_new][d] at slots pos (Eq 7)."""
    n_new = k_new.shape[2]
    _need_cuda(k_new, v_new, pos_dev)
    want = (cache.batch, cache.kv_heads, n_new, cache.head_dim)
    if k_new.dtype != torch.float16 or v_new.dtype != torch.float16 or tuple(k_new.shape) != want \
            or tuple(v_new.shape) != want:
        raise ValueError(f"k_new/v_new must be fp16 {want}")
    if pos_dev is not None and (pos_dev.dtype != torch.int32 or pos_dev.numel() != cache.batch):
        raise ValueError(f"pos_dev must be int32 [{cache.batch}]")
    c = abi if abi is not None else cache.abi()
    _check(_lib.lmo_kv_append_quant(ctypes.byref(c), _ptr(k_new), _ptr(v_new), n_new, pos0,
                                    _ptr(pos_dev), _stream(stream)), "lmo_kv_append_quant")


def lmo_decode_attention_workspace_bytes(batch: int, kv_heads: int, q_heads: int, head_dim: int,
                                         num_splits: int = 0) -> int:
    return int(_lib.lmo_decode_attention_workspace_bytes(batch, kv_heads, q_heads, head_dim,
                                                         num_splits))


def attention_workspace(batch: int, kv_heads: int, q_heads: int, head_dim: int,
                        num_splits: int = 0, device="cuda") -> torch.Tensor:
    """Zero-initialised workspace (its arrival counters must start at 0)."""
    n = lmo_decode_attention_workspace_bytes(batch, kv_heads, q_heads, head_dim, num_splits)
    if n == 0:
        raise LmoError(LMO_ERR_SHAPE, "lmo_decode_attention_workspace_bytes")
    return torch.zeros(n, dtype=torch.uint8, device=device)


def _check_step_args(cache: KVCache, q, out, seq_lens, workspace, k_new=None, v_new=None):
    """Host-side shape/dtype/device checks of the tensors handed to the C ABI (the
    library sees raw pointers; a wrong dtype or shape here would be read or written
    out of bounds)."""
    _need_cuda(q, out, seq_lens, workspace, k_new, v_new)
    B, Hkv, d = cache.batch, cache.kv_heads, cache.head_dim
    if q.dtype != torch.float16 or q.dim() != 3 or q.shape[0] != B or q.shape[2] != d or q.shape[1] % Hkv:
        raise ValueError(f"q must be fp16 [{B}][Hq][{d}] with Hq % {Hkv} == 0, got {q.dtype} {tuple(q.shape)}")
    if out.dtype not in (torch.float16, torch.float32) or tuple(out.shape) != tuple(q.shape):
        raise ValueError(f"out must be fp16/fp32 {tuple(q.shape)}, got {out.dtype} {tuple(out.shape)}")
    if seq_lens is not None and (seq_lens.dtype != torch.int32 or seq_lens.numel() != B):
        raise ValueError(f"seq_lens must be int32 [{B}]")
    for t in (k_new, v_new):
        if t is not None and (t.dtype != torch.float16 or t.numel() != B * Hkv * d):
            raise ValueError(f"k_new/v_new must be fp16 [{B}][{Hkv}](1)[{d}]")
    for t in (q, out, workspace, k_new, v_new, seq_lens):
        if t is not None and t.device != cache.kv.device:
            raise ValueError("all tensors must live on the cache's device")


def _nbytes(t: torch.Tensor) -> int:
    return t.numel() * t.element_size()


def lmo_decode_attention_q4(cache: KVCache, q: torch.Tensor, length: int = 0,
                            seq_lens: torch.Tensor | None = None, softmax_scale: float | None = None,
                            num_splits: int = 0, out: torch.Tensor | None = None,
                            out_dtype: torch.dtype = torch.float32,
                            workspace: torch.Tensor | None = None, stream=None,
                            abi=None) -> torch.Tensor:
    """softmax(scale q K^T) V over the q4 cache, dequant fused."""
    B, Hq, d = q.shape
    if softmax_scale is None:
        softmax_scale = 1.0 / math.sqrt(d)
    if out is None:
        out = torch.empty((B, Hq, d), dtype=out_dtype, device=q.device)
    if workspace is None:
        workspace = attention_workspace(cache.batch, cache.kv_heads, Hq, cache.head_dim,
                                        num_splits, q.device)
    _check_step_args(cache, q, out, seq_lens, workspace)
    dt = LMO_F16 if out.dtype == torch.float16 else LMO_F32
    c = abi if abi is not None else cache.abi()
    _check(_lib.lmo_decode_attention_q4(ctypes.byref(c), _ptr(q), Hq, length, _ptr(seq_lens),
                                        float(softmax_scale), num_splits, _ptr(out), dt,
                                        _ptr(workspace), _nbytes(workspace), _stream(stream)),
           "lmo_decode_attention_q4")
    return out


def lmo_decode_step_q4(cache: KVCache, k_new: torch.Tensor, v_new: torch.Tensor, q: torch.Tensor,
                       length: int = 0, seq_lens: torch.Tensor | None = None,
                       softmax_scale: float | None = None, num_splits: int = 0,
                       out: torch.Tensor | None = None, out_dtype: torch.dtype = torch.float32,
                       workspace: torch.Tensor | None = None, flags: int = 0, stream=None,
                       abi=None) -> torch.Tensor:
    """One decode step of one layer: append the new token's K/V ([B][Hkv][d] or
    [B][Hkv][1][d]) at slot L-1, then attention over L (A2+A3+A4 fused).
    flags=LMO_STEP_CACHE_STABLE: see include/lmo.h."""
    B, Hq, d = q.shape
    if softmax_scale is None:
        softmax_scale = 1.0 / math.sqrt(d)
    if out is None:
        out = torch.empty((B, Hq, d), dtype=out_dtype, device=q.device)
    if workspace is None:
        workspace = attention_workspace(cache.batch, cache.kv_heads, Hq, cache.head_dim,
                                        num_splits, q.device)
    _check_step_args(cache, q, out, seq_lens, workspace, k_new, v_new)
    dt = LMO_F16 if out.dtype == torch.float16 else LMO_F32
    c = abi if abi is not None else cache.abi()
    _check(_lib.lmo_decode_step_q4(ctypes.byref(c), _ptr(k_new), _ptr(v_new), _ptr(q), Hq, length,
                                   _ptr(seq_lens), float(softmax_scale), num_splits, _ptr(out), dt,
                                   _ptr(workspace), _nbytes(workspace), int(flags), _stream(stream)),
           "lmo_decode_step_q4")
    return out


def lmo_gen_fill_f16(dst: torch.Tensor, seed: int, stream_id: int, layer: int, b0: int, h0: int,
                     p0: int, group: int = 1, stream=None) -> torch.Tensor:
    """Device twin of inputs.gen_f16: dst [nb][nh][npos][dim] fp16."""
    nb, nh, npos, dim = dst.shape
    _need_cuda(dst)
    _check(_lib.lmo_gen_fill_f16(_ptr(dst), nb, nh, npos, dim, seed, stream_id, layer, b0, h0, p0,
                                 group, _stream(stream)), "lmo_gen_fill_f16")
    return dst


def lmo_probe_read_stream(buf: torch.Tensor, sink: torch.Tensor, stream=None) -> None:
    """Measurement support: one read-only streaming pass over buf (bench roofline)."""
    _need_cuda(buf, sink)
    _check(_lib.lmo_probe_read_stream(_ptr(buf), buf.numel() * buf.element_size() // 16 * 16, _ptr(sink),
                                      _stream(stream)), "lmo_probe_read_stream")


# ------------------------------------------------------- NEXT-4: offloaded KV

class OffloadKV:
    """Host-offloaded q4 KV caches of `layers` layers (pinned host memory, the
    paper's setting) + a device staging ring of `slots` layer caches, driven by
    the library's executor (lmo_offload_*).  Layout of each host layer =
    KVCache.kv ([B][Hkv][cap][row] bytes)."""

    def __init__(self, layers: int, batch: int, kv_heads: int, capacity: int, head_dim: int,
                 slots: int = 2, device="cuda"):
        cap = (capacity + 15) // 16 * 16
        self.layers, self.batch, self.kv_heads, self.capacity, self.head_dim = \
            layers, batch, kv_heads, cap, head_dim
        self.shape = lmo_kv_cache(None, batch, kv_heads, cap, head_dim)
        self.row = row_bytes(head_dim)
        self.layer_bytes = batch * kv_heads * cap * self.row
        self.host = torch.empty(layers * self.layer_bytes, dtype=torch.uint8).pin_memory()
        n = _lib.lmo_offload_ring_bytes(ctypes.byref(self.shape), slots)
        if n == 0:
            raise LmoError(LMO_ERR_SHAPE, "lmo_offload_ring_bytes")
        self.ring = torch.empty(n, dtype=torch.uint8, device=device)
        self._h = ctypes.c_void_p()
        _check(_lib.lmo_offload_create(ctypes.byref(self.shape), layers,
                                       ctypes.c_void_p(self.host.data_ptr()),
                                       ctypes.c_void_p(self.ring.data_ptr()), slots,
                                       ctypes.byref(self._h)), "lmo_offload_create")

    def host_layer(self, l: int) -> torch.Tensor:
        """View of host layer l as [B][Hkv][cap][row] uint8."""
        return self.host[l * self.layer_bytes:(l + 1) * self.layer_bytes].view(
            self.batch, self.kv_heads, self.capacity, self.row)

    def decode_step(self, k_new: torch.Tensor, v_new: torch.Tensor, q: torch.Tensor, length: int,
                    softmax_scale: float | None = None, num_splits: int = 0,
                    out: torch.Tensor | None = None, out_dtype: torch.dtype = torch.float32,
                    workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
        """All layers' decode step at L = length: k_new/v_new [layers][B][Hkv](1)[d],
        q [layers][B][Hq](1)[d] -> out [layers][B][Hq][d]."""
        nl, B = self.layers, self.batch
        Hq = q.shape[2]
        d = self.head_dim
        if softmax_scale is None:
            softmax_scale = 1.0 / math.sqrt(d)
        if out is None:
            out = torch.empty((nl, B, Hq, d), dtype=out_dtype, device=q.device)
        if workspace is None:
            workspace = attention_workspace(B, self.kv_heads, Hq, d, num_splits, q.device)
        _need_cuda(k_new, v_new, q, out, workspace)
        dt = LMO_F16 if out.dtype == torch.float16 else LMO_F32
        _check(_lib.lmo_offload_decode_step(self._h, _ptr(k_new), _ptr(v_new), _ptr(q), Hq, length,
                                            float(softmax_scale), num_splits, _ptr(out), dt,
                                            _ptr(workspace), _nbytes(workspace), _stream(stream)),
               "lmo_offload_decode_step")
        return out

    def close(self):
        if self._h:
            _lib.lmo_offload_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
