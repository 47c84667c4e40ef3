"""Byte accounting (bench GB/s numerator) pinned to the sizes PAPER.md prints."""
import json
import os

from paper_conf_ipps_wurypgll25_b200 import configs as C

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_sizes.json")))
GIB = 2 ** 30
OPT30B = dict(layers=48, hidden=7168, vocab=50272, s=64, n=128, bls=640)


def test_kv_cache_157gb():
    got = C.kv_cache_bytes_fp16(OPT30B["layers"], OPT30B["hidden"],
                                OPT30B["s"] + OPT30B["n"] - 1, OPT30B["bls"]) / GIB
    assert abs(got - GOLD["kv_cache_gb"]["value"]) < 0.5        # 156.68 GiB
    # capacity s+n (instead of s+n-1) would print 157.5 -> pins the n-1 reading
    alt = C.kv_cache_bytes_fp16(48, 7168, 64 + 128, 640) / GIB
    assert abs(alt - 157) >= 0.5


def test_weights_55gb():
    got = C.weight_bytes_fp16(OPT30B["layers"], OPT30B["hidden"], OPT30B["vocab"]) / GIB
    assert abs(got - GOLD["weights_gb"]["value"]) < 1.0          # 55.8 GiB


def test_new_kv_per_token_0_8gb():
    got = C.new_kv_bytes_fp16_per_token(OPT30B["layers"], OPT30B["hidden"], OPT30B["bls"]) / GIB
    assert abs(got - GOLD["new_kv_gb_per_token"]["value"]) < 0.05  # 0.82 GiB


def test_q4_row_bytes_and_configs():
    assert C.q4_row_bytes(128) == 72 and C.q4_row_bytes(64) == 36
    w = C.CONFIGS["c2"]
    assert w.steps == 31 and w.max_len == 543 and w.capacity == 544
    assert w.len_at_step(1) == 513 and w.len_at_step(w.steps) == 543
    assert C.CONFIGS["c5"].group_ratio == 8
    # c2 KV bytes at mean L=528: 32*32*528*144 B = 77.9 MB
    assert abs(C.attention_kv_bytes(w, 528) / 1e6 - 77.86) < 0.01
    for w in C.CONFIGS.values():
        assert w.q_heads % w.kv_heads == 0 and w.head_dim % 64 == 0
