"""NEXT-4: host-offloaded q4 KV executor (lmo_offload_*) vs the
device-resident path and the oracle.  The executor only moves bytes (strided
H2D of the old-token rows, D2H of the new row) around the same fused step, so
its outputs must be bit-identical to the resident path's, and its host caches
byte-identical to the resident caches."""
import math

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_wurypgll25_b200 import inputs as I

pytestmark = pytest.mark.gpu
TOL = 2e-3


@pytest.fixture(scope="module")
def lmo():
    from paper_conf_ipps_wurypgll25_b200 import lmo as m
    return m


@pytest.mark.parametrize("slots", [1, 2, 3])
@pytest.mark.parametrize("G,d,nl", [(1, 128, 3), (4, 128, 4), (2, 64, 2)])
def test_offload_matches_resident(lmo, slots, G, d, nl):
    B, Hkv, s0, steps = 3, 4, 45, 4
    Hq = Hkv * G
    seed = 977 + slots + G
    cap = s0 + steps
    res = [lmo.KVCache.empty(B, Hkv, cap, d, zero=True) for _ in range(nl)]
    off = lmo.OffloadKV(nl, B, Hkv, cap, d, slots=slots)
    off.host.fill_(0x5A)                          # untouched rows must not matter
    kall = torch.empty((nl, B, Hkv, cap, d), dtype=torch.float16, device="cuda")
    vall = torch.empty_like(kall)
    for l in range(nl):
        lmo.lmo_gen_fill_f16(kall[l], seed, I.STREAM_K, l, 0, 0, 0)
        lmo.lmo_gen_fill_f16(vall[l], seed, I.STREAM_V, l, 0, 0, 0)
        lmo.lmo_kv_append_quant(res[l], kall[l, :, :, :s0].contiguous(), vall[l, :, :, :s0].contiguous(), 0)
        s2 = s0 + (s0 & 1)                        # whole token pairs (V codes span both rows)
        off.host_layer(l)[:, :, :s2].copy_(res[l].kv[:, :, :s2].cpu())
    torch.cuda.synchronize()
    ws = lmo.attention_workspace(B, Hkv, Hq, d)
    for t in range(1, steps + 1):
        L = s0 + t
        kn = kall[:, :, :, L - 1].contiguous()
        vn = vall[:, :, :, L - 1].contiguous()
        q = torch.empty((nl, B, Hq, 1, d), dtype=torch.float16, device="cuda")
        for l in range(nl):
            lmo.lmo_gen_fill_f16(q[l], seed, I.STREAM_Q, l, 0, 0, t, group=G)
        q = q.view(nl, B, Hq, d)
        want = torch.stack([lmo.lmo_decode_step_q4(res[l], kn[l], vn[l], q[l], L, workspace=ws)
                            for l in range(nl)])
        got = off.decode_step(kn, vn, q, L)
        torch.cuda.synchronize()
        assert torch.equal(got, want), f"step {t}"
    L = s0 + steps
    for l in range(nl):   # every field of tokens [0, L), V codes de-interleaved from the row pairs
        hv = lmo.KVCache(off.host_layer(l), B, Hkv, off.capacity, d).to_host_fields()
        rv = res[l].to_host_fields()
        for key in rv:
            assert np.array_equal(hv[key][:, :, :L], rv[key][:, :, :L]), (l, key)
    # and the last step of layer 0 against the oracle (host cache bytes -> oracle fields)
    host = oracle.new_cache(B, Hkv, res[0].capacity, d)
    oracle.kv_append_quant(host, kall[0, :, :, :L].cpu().numpy(), vall[0, :, :, :L].cpu().numpy(), 0)
    ref = oracle.decode_attention_q4(host, q[0].cpu().numpy(), L, 1 / math.sqrt(d), nthreads=8)
    o = got[0].cpu().numpy().astype(np.float64)
    err = np.max(np.abs(o - ref), axis=-1) / np.max(np.abs(ref), axis=-1)
    assert err.max() <= TOL
    off.close()


def test_offload_argument_errors(lmo):
    off = lmo.OffloadKV(2, 2, 2, 32, 128, slots=2)
    q = torch.zeros((2, 2, 2, 128), dtype=torch.float16, device="cuda")
    kn = torch.zeros((2, 2, 2, 128), dtype=torch.float16, device="cuda")
    with pytest.raises(lmo.LmoError):
        off.decode_step(kn, kn, q, 0)             # len < 1
    with pytest.raises(lmo.LmoError):
        off.decode_step(kn, kn, q, 33)            # len > capacity
    with pytest.raises(lmo.LmoError):
        off.decode_step(kn, kn, q, 5, workspace=torch.zeros(16, dtype=torch.uint8, device="cuda"))
    off.close()
