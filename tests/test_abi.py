"""CPU checks of the C-ABI library: it builds, loads, exports every symbol that
include/lmo.h declares, and rejects bad arguments before touching CUDA."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "lmo.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lmo_[a-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_wurypgll25_b200 import build
    build.build()
    from paper_conf_ipps_wurypgll25_b200 import lmo
    return lmo


def test_header_declares_boundary():
    fns = declared_functions()
    for f in ("lmo_quantize_groupwise", "lmo_dequantize_groupwise", "lmo_kv_append_quant",
              "lmo_decode_attention_q4", "lmo_decode_attention_workspace_bytes",
              "lmo_status_string"):
        assert f in fns


def test_library_exports_every_declared_symbol(lib):
    so = ctypes.CDLL(lib.LIB_PATH)
    for f in declared_functions():
        assert hasattr(so, f), f
    assert set(lib.EXPORTS) == set(declared_functions())


def test_status_strings_and_version(lib):
    assert lib._lib.lmo_status_string(0) == b"LMO_OK"
    assert b"ALIGN" in lib._lib.lmo_status_string(4)
    assert lib._lib.lmo_version() >> 16 == 1


def test_argument_validation_without_gpu(lib):
    L = lib._lib
    P = ctypes.c_void_p
    # bits != 4 / group != 64 -> UNSUPPORTED, before any pointer check
    assert L.lmo_quantize_groupwise(P(16), 1, 64, 1, 3, 64, P(16), P(16), None) == 3
    assert L.lmo_quantize_groupwise(P(16), 1, 64, 1, 4, 32, P(16), P(16), None) == 3
    assert L.lmo_quantize_groupwise(P(16), -1, 64, 1, 4, 64, P(16), P(16), None) == 2
    assert L.lmo_quantize_groupwise(None, 1, 64, 1, 4, 64, P(16), P(16), None) == 1
    assert L.lmo_quantize_groupwise(P(18), 1, 64, 1, 4, 64, P(16), P(16), None) == 4
    assert L.lmo_quantize_groupwise(None, 0, 64, 1, 4, 64, None, None, None) == 0   # empty no-op
    assert L.lmo_dequantize_groupwise(P(16), P(16), 1, 64, 1, 4, 64, None, None) == 1
    c = lib.lmo_kv_cache(16, 2, 2, 32, 128)
    assert L.lmo_kv_append_quant(ctypes.byref(c), P(16), P(16), 1, 32, None, None) == 2  # pos overflow
    c.head_dim = 96
    assert L.lmo_kv_append_quant(ctypes.byref(c), P(16), P(16), 1, 0, None, None) == 3
    c.head_dim = 128
    c.capacity = 30
    assert L.lmo_kv_append_quant(ctypes.byref(c), P(16), P(16), 1, 0, None, None) == 2
    c.capacity = 32
    c.kv = 50
    assert L.lmo_kv_append_quant(ctypes.byref(c), P(16), P(16), 1, 0, None, None) == 4
    c.kv = 48
    assert L.lmo_kv_row_bytes(128) == 144 and L.lmo_kv_row_bytes(64) == 72
    assert L.lmo_kv_row_bytes(96) == 0
    # attention: group ratio > 8 unsupported, len > capacity
    assert L.lmo_decode_attention_q4(ctypes.byref(c), P(16), 18, 4, None, 1.0, 0, P(16), 1,
                                     P(16), 1 << 30, None) == 3
    assert L.lmo_decode_attention_q4(ctypes.byref(c), P(16), 4, 33, None, 1.0, 0, P(16), 1,
                                     P(16), 1 << 30, None) == 2
    assert L.lmo_decode_attention_q4(ctypes.byref(c), P(16), 3, 8, None, 1.0, 0, P(16), 1,
                                     P(16), 1 << 30, None) == 2   # 3 % 2 != 0
    assert L.lmo_gen_fill_f16(None, 1, 1, 1, 1, 0, 1, 0, 0, 0, 0, 1, None) == 1


def test_binding_has_no_cpu_fallback():
    """The product package never imports, links or loads the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_wurypgll25_b200")
    bad = re.compile(r"^\s*(import\s+oracle|from\s+oracle|from\s+\.\.\s*oracle)|liblmo_oracle|lmo_oracle\.c",
                     re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not bad.search(txt), f


def test_offload_validation_without_gpu(lib):
    import ctypes
    L = lib._lib
    good = lib.lmo_kv_cache(None, 2, 2, 32, 128)
    bad = lib.lmo_kv_cache(None, 2, 2, 32, 96)
    assert L.lmo_offload_ring_bytes(ctypes.byref(good), 2) == 2 * 2 * 2 * 32 * 144
    assert L.lmo_offload_ring_bytes(ctypes.byref(bad), 2) == 0
    assert L.lmo_offload_ring_bytes(ctypes.byref(good), 0) == 0
    h = ctypes.c_void_p()
    P = ctypes.c_void_p
    assert L.lmo_offload_create(ctypes.byref(good), 0, P(4096), P(4096), 2, ctypes.byref(h)) == lib.LMO_ERR_SHAPE
    assert L.lmo_offload_create(ctypes.byref(good), 2, None, P(4096), 2, ctypes.byref(h)) == lib.LMO_ERR_NULL
    assert L.lmo_offload_create(ctypes.byref(good), 2, P(4100), P(4096), 2, ctypes.byref(h)) == lib.LMO_ERR_ALIGN
    assert L.lmo_offload_decode_step(None, P(16), P(16), P(16), 2, 5, 1.0, 0, P(16), 1, P(16), 1 << 20, None) \
        == lib.LMO_ERR_NULL
    assert L.lmo_offload_destroy(None) == lib.LMO_ERR_NULL
