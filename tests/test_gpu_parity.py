"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by
element on the same seeded inputs.

Bars: codes / mins / scales / dequantized fp16 bit-exact;
attention normwise per (b, h) row max|o_gpu - o_ref| / max|o_ref| <= 2e-3
(BASELINE.json north star), fp32 accumulation vs the fp64 oracle.
"""
import math
import zlib

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_wurypgll25_b200 import inputs as I
from paper_conf_ipps_wurypgll25_b200.configs import CONFIGS

pytestmark = pytest.mark.gpu
TOL = 2e-3


@pytest.fixture(scope="module")
def lmo():
    from paper_conf_ipps_wurypgll25_b200 import lmo as m
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def meta_u16(m):
    """int32 meta tensor -> uint16 pairs {min, scale} (little-endian)."""
    return m.cpu().numpy().view(np.uint16).reshape(*m.shape, 2)


def normwise_err(got, ref):
    got = np.asarray(got, np.float64)
    den = np.maximum(np.max(np.abs(ref), axis=-1), 1e-30)
    return np.max(np.abs(got - ref), axis=-1) / den


def check_attention(got, ref, what="", tol=TOL):
    """Assert the normwise bar (reading 17) and log the margins: the max normwise
    error and the max elementwise relative error with a 1e-6 floor."""
    got = np.asarray(got, np.float64)
    err = normwise_err(got, ref)
    rel = np.abs(got - ref) / np.maximum(np.abs(ref), 1e-6)
    print(f"[parity] {what}: normwise max {err.max():.3e} (bar {tol:.0e}, margin x{tol / max(err.max(), 1e-30):.1f}),"
          f" elementwise rel max {rel.max():.3e}")
    assert err.max() <= tol, (what, err.max(), np.unravel_index(err.argmax(), err.shape))
    return err.max()


# ----------------------------------------------------------------- K6 ------

def test_generator_matches_host(lmo):
    for stream, group in ((I.STREAM_K, 1), (I.STREAM_V, 1), (I.STREAM_Q, 8)):
        d = torch.empty((3, 5, 37, 128), dtype=torch.float16, device="cuda")
        lmo.lmo_gen_fill_f16(d, seed=I.seed_for_config(4), stream_id=stream, layer=7, b0=11, h0=2,
                             p0=1000, group=group)
        h = I.gen_f16(I.seed_for_config(4), stream, 7, 11, 3, 2, 5, 1000, 37, 128, group=group)
        assert np.array_equal(d.cpu().numpy().view(np.uint16), h.view(np.uint16))


# ------------------------------------------------------------ K1 / K5 ------

def adversarial_tensor(rng, rows):
    g = [rng.standard_normal(64) * 10.0 ** rng.uniform(-3, 3) for _ in range(max(rows, 6))]
    g[0] = np.full(64, 3.25)                        # constant
    g[1] = np.full(64, -0.0)                        # signed zero
    g[2] = -3.0 + rng.integers(0, 16, 64) * 0.25    # on-grid
    g[3] = rng.uniform(-65504, 65504, 64)           # extremes
    g[3][:2] = [-65504, 65504]
    g[4] = rng.integers(-3, 4, 64) * 2.0 ** -24     # subnormal
    x = np.zeros(64); x[0], x[1] = 0, 15; x[2:9] = [0.5, 1.5, 2.5, 3.5, 4.5, 13.5, 14.5]
    g[5] = x                                        # ties
    order = rng.permutation(len(g))[:rows]
    return np.concatenate([g[i] for i in order]).astype(np.float16)


@pytest.mark.parametrize("outer,n,inner", [(1, 64, 1), (37, 128, 1), (300, 64 * 5, 1),
                                           (3, 100, 1), (4, 128, 7), (2, 65, 3), (1, 7, 1)])
def test_quantize_bit_exact(lmo, outer, n, inner):
    rng = np.random.default_rng(outer * 1000 + n + inner)
    if inner == 1 and n % 64 == 0:
        x = adversarial_tensor(rng, outer * n // 64).reshape(outer, n, inner)
    else:
        x = (rng.standard_normal((outer, n, inner)) * 3).astype(np.float16)
    c_ref, m_ref = oracle.quantize_groupwise(x, outer, n, inner)
    c, m = lmo.lmo_quantize_groupwise(dev(x), outer, n, inner)
    torch.cuda.synchronize()
    assert np.array_equal(c.cpu().numpy(), c_ref)
    assert np.array_equal(meta_u16(m), m_ref)


def scale_sweep_tensor():
    """Every positive finite fp16 value v as a group range (min 0, max v), plus as
    many groups with a random negative min (range = RN32(v - mn)): exercises the
    kernels' RU16(range/15) derivation at every fp16 step and the code rounding
    at every scale (the paper's scale = (max - min)/(2^b - 1), R2)."""
    rng = np.random.default_rng(7)
    v = np.arange(1, 0x7C00, dtype=np.uint16).view(np.float16).astype(np.float64)
    frac = np.linspace(0.0, 1.0, 64)
    g1 = v[:, None] * frac[None, :]
    mn = -rng.uniform(0, 1, v.size) * v
    g2 = mn[:, None] + (v - mn)[:, None] * rng.permutation(frac)[None, :]
    g2[:, 0], g2[:, 1] = mn, v
    x = np.concatenate([g1, g2]).astype(np.float16)
    x[: v.size, 63] = v.astype(np.float16)                  # exact max
    return x.reshape(-1)


def test_quantize_scale_sweep_bit_exact(lmo):
    x = scale_sweep_tensor()
    rows = x.size // 64
    c_ref, m_ref = oracle.quantize_groupwise(x.reshape(rows, 64, 1), rows, 64, 1)
    c, m = lmo.lmo_quantize_groupwise(dev(x.reshape(rows, 64, 1)), rows, 64, 1)
    torch.cuda.synchronize()
    assert np.array_equal(meta_u16(m), m_ref)
    assert np.array_equal(c.cpu().numpy(), c_ref)
    # the strided (inner > 1) kernel on the same groups, transposed
    xt = np.ascontiguousarray(x.reshape(rows, 64).T).reshape(1, 64, rows)
    c_ref, m_ref = oracle.quantize_groupwise(xt, 1, 64, rows)
    c, m = lmo.lmo_quantize_groupwise(dev(xt), 1, 64, rows)
    torch.cuda.synchronize()
    assert np.array_equal(meta_u16(m), m_ref)
    assert np.array_equal(c.cpu().numpy(), c_ref)


@pytest.mark.parametrize("outer,n,inner", [(64, 128, 1), (3, 100, 1), (4, 128, 7), (513, 64 * 3, 1)])
def test_dequantize_bit_exact(lmo, outer, n, inner):
    rng = np.random.default_rng(n + inner)
    x = (rng.standard_normal((outer, n, inner)) * 10.0 ** rng.uniform(-2, 2)).astype(np.float16)
    c_ref, m_ref = oracle.quantize_groupwise(x, outer, n, inner)
    y_ref = oracle.dequantize_groupwise(c_ref, m_ref, outer, n, inner)
    m_i32 = np.ascontiguousarray(m_ref).view(np.int32).reshape(m_ref.shape[:-1])
    y = lmo.lmo_dequantize_groupwise(dev(c_ref), dev(m_i32), outer, n, inner)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().view(np.uint16), y_ref.view(np.uint16))


def test_weight_dequant_round_trip_shape(lmo):
    """c3 weight leg at a reduced hidden size: quantize (inner-dim groups) then
    dequantize equals the oracle's dequant of the oracle's codes."""
    rng = np.random.default_rng(3)
    h1 = 512
    w = (rng.standard_normal((4 * h1, h1)) * 0.02).astype(np.float16)
    c, m = lmo.lmo_quantize_groupwise(dev(w), 4 * h1, h1, 1)
    y = lmo.lmo_dequantize_groupwise(c, m, 4 * h1, h1, 1)
    c_ref, m_ref = oracle.quantize_groupwise(w, 4 * h1, h1, 1)
    y_ref = oracle.dequantize_groupwise(c_ref, m_ref, 4 * h1, h1, 1)
    assert np.array_equal(y.cpu().numpy().view(np.uint16), y_ref.view(np.uint16))


# ---------------------------------------------------------------- K2 -------

def cache_to_host(cache):
    return cache.to_host_fields()


@pytest.mark.parametrize("d", [64, 128])
def test_append_bit_exact_with_canaries(lmo, d):
    rng = np.random.default_rng(d)
    B, H, cap, n_new = 3, 4, 48, 5
    cache = lmo.KVCache.empty(B, H, cap, d)
    cache.kv.fill_(0xA5)
    host = oracle.new_cache(B, H, cap, d, fill=0xA5)
    k = (rng.standard_normal((B, H, n_new, d)) * 2).astype(np.float16)
    v = rng.standard_normal((B, H, n_new, d)).astype(np.float16)
    lmo.lmo_kv_append_quant(cache, dev(k), dev(v), pos0=17)
    oracle.kv_append_quant(host, k, v, 17)
    # per-sequence positions
    pos = np.array([0, 40, 9], np.int32)
    k2 = (rng.standard_normal((B, H, 3, d))).astype(np.float16)
    lmo.lmo_kv_append_quant(cache, dev(k2), dev(k2), pos_dev=dev(pos))
    oracle.kv_append_quant(host, k2, k2, pos)
    torch.cuda.synchronize()
    got = cache_to_host(cache)
    for key in host:
        assert np.array_equal(got[key], host[key]), key


@pytest.mark.parametrize("d", [64, 128])
def test_append_scale_sweep_bit_exact(lmo, d):
    """The append kernel's quantizer over the every-fp16-range sweep (K and V)."""
    x = scale_sweep_tensor()
    n = x.size // d
    k = x[: n * d].reshape(1, 1, n, d)
    v = np.ascontiguousarray(k[:, :, ::-1])
    cache = lmo.KVCache.empty(1, 1, n, d)
    lmo.lmo_kv_append_quant(cache, dev(k), dev(v), pos0=0)
    host = oracle.new_cache(1, 1, cache.capacity, d)
    oracle.kv_append_quant(host, k, v, 0)
    torch.cuda.synchronize()
    got = cache_to_host(cache)
    for key in host:
        assert np.array_equal(got[key][:, :, :n], host[key][:, :, :n]), key


# ---------------------------------------------------------------- K3 -------

def build_layer(lmo, B, Hkv, cap, d, L, seed, layer=0, lens=None):
    """Fill a q4 cache on the device from the seeded generator (prefill via
    append) and the same cache on the host via the oracle."""
    kf = torch.empty((B, Hkv, L, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, layer, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, layer, 0, 0, 0)
    cache = lmo.KVCache.empty(B, Hkv, cap, d)
    lmo.lmo_kv_append_quant(cache, kf, vf, pos0=0)
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    kh = I.gen_f16(seed, I.STREAM_K, layer, 0, B, 0, Hkv, 0, L, d)
    vh = I.gen_f16(seed, I.STREAM_V, layer, 0, B, 0, Hkv, 0, L, d)
    oracle.kv_append_quant(host, kh, vh, 0)
    return cache, host


CASES = [  # (B, Hkv, G, d, L, num_splits)
    (2, 3, 1, 64, 1, 0), (2, 3, 1, 128, 2, 0), (1, 2, 2, 128, 15, 0), (3, 2, 1, 128, 16, 0),
    (2, 4, 1, 128, 17, 0), (4, 12, 1, 64, 71, 0), (2, 2, 4, 128, 63, 0), (2, 2, 8, 128, 65, 1),
    (3, 5, 1, 128, 100, 3), (2, 2, 8, 64, 1000, 0), (1, 3, 1, 128, 1000, 7), (2, 1, 8, 128, 4090, 0),
    (5, 7, 3, 128, 333, 0), (1, 1, 1, 128, 1, 4), (64, 8, 1, 128, 40, 0), (3, 4, 2, 128, 517, 2),
    (2, 3, 8, 128, 250, 4), (3, 2, 1, 64, 47, 2),
    (3, 5, 1, 128, 100, -1), (2, 2, 8, 128, 65, -1), (64, 8, 1, 128, 40, -1), (2, 3, 2, 64, 333, -1),
    (3, 5, 1, 128, 100, -2), (2, 2, 8, 128, 65, -2), (64, 8, 1, 128, 40, -2), (2, 3, 2, 64, 333, -2),
    (1, 1, 1, 128, 1000, -2), (40, 9, 1, 128, 77, -2), (5, 3, 8, 128, 1, -2), (300, 4, 1, 64, 20, -2),
    # GQA, 592 < pairs <= 1184: the deep-ring 2-CTA/SM instance
    (80, 8, 8, 128, 200, 0), (130, 9, 2, 128, 77, 0), (148, 8, 4, 128, 33, 0),
    # MHA, 592 < pairs <= 1184: the default instance on a 2-CTA/SM grid
    (64, 10, 1, 128, 90, 0), (100, 11, 1, 128, 47, 0),
]


@pytest.mark.parametrize("B,Hkv,G,d,L,ns", CASES)
@pytest.mark.parametrize("out_dtype", [torch.float32, torch.float16])
def test_attention_parity(lmo, B, Hkv, G, d, L, ns, out_dtype):
    seed = 1000 + B * 7 + L
    cap = L + (L % 3)
    cache, host = build_layer(lmo, B, Hkv, cap, d, L, seed)
    Hq = Hkv * G
    q = torch.empty((B, Hq, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hq, d)
    sigma = 1 / math.sqrt(d)
    out = lmo.lmo_decode_attention_q4(cache, q, L, softmax_scale=sigma, num_splits=ns,
                                      out_dtype=out_dtype)
    torch.cuda.synchronize()
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), L, sigma, nthreads=8)
    check_attention(out.float().cpu().numpy(), ref, f"B{B} Hkv{Hkv} G{G} d{d} L{L} ns{ns} {out_dtype}")


def test_attention_per_sequence_lengths_and_reuse(lmo):
    B, Hkv, G, d, cap = 6, 3, 2, 128, 272
    cache, host = build_layer(lmo, B, Hkv, cap, d, cap, 77)
    lens = np.array([1, 0, 272, 17, 128, 250], np.int32)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, 77, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    ws = lmo.attention_workspace(B, Hkv, Hkv * G, d, 0)
    ref_lens = np.maximum(lens, 1)
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), ref_lens, nthreads=8)
    for _ in range(3):   # workspace counters must be reset by each call
        out = lmo.lmo_decode_attention_q4(cache, q, 0, seq_lens=dev(lens), workspace=ws)
        torch.cuda.synchronize()
        o = out.cpu().numpy()
        assert np.all(o[1] == 0)                     # empty sequence -> zero row
        keep = lens > 0
        check_attention(o[keep], ref[keep], "per-sequence lengths, reuse")
    assert int(ws[: 4 * B * Hkv].view(torch.int32).abs().sum()) == 0


@pytest.mark.parametrize("team", [1, 2, 4])
def test_attention_empty_sequence_every_team_size(lmo, team):
    """A per-sequence length of 0 leaves a zero output row for every team size
    (team 1 is the default schedule of the BASELINE configs)."""
    B, Hkv, G, d, cap = 5, 4, 1, 128, 96
    cache, host = build_layer(lmo, B, Hkv, cap, d, cap, 91)
    lens = np.array([40, 0, 96, 1, 0], np.int32)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, 91, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    ws = lmo.attention_workspace(B, Hkv, Hkv * G, d, team)
    out = lmo.lmo_decode_attention_q4(cache, q, 0, seq_lens=dev(lens), workspace=ws, num_splits=team)
    o = out.cpu().numpy()
    assert np.all(o[lens == 0] == 0)
    keep = lens > 0
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), np.maximum(lens, 1), nthreads=4)
    check_attention(o[keep], ref[keep], f"empty sequences, team {team}")


def test_attention_split_modes_agree(lmo):
    """stream-K (0) and fixed splits (1, 5) give the same result within rounding;
    a fixed split count is deterministic."""
    B, Hkv, G, d, L = 4, 4, 2, 128, 700
    cache, _ = build_layer(lmo, B, Hkv, L + 4, d, L, 5)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, 5, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    o0 = lmo.lmo_decode_attention_q4(cache, q, L, num_splits=0)
    o1 = lmo.lmo_decode_attention_q4(cache, q, L, num_splits=1)
    o5 = lmo.lmo_decode_attention_q4(cache, q, L, num_splits=5)
    o5b = lmo.lmo_decode_attention_q4(cache, q, L, num_splits=5)
    torch.cuda.synchronize()
    assert torch.equal(o5, o5b)
    for o in (o0, o5):
        assert (o - o1).abs().max().item() <= 1e-3 * o1.abs().max().item()


# --------------------------------------- full-size sampled (bench launch) --

def sample_pairs(B, Hkv, n=4):
    rng = np.random.default_rng(B * 1000 + Hkv)
    return [(0, 0), (B - 1, Hkv - 1)] + [(int(rng.integers(B)), int(rng.integers(Hkv))) for _ in range(n)]


def oracle_pair(seed, layer, b, kvh, L, d, cap):
    """The oracle's q4 cache of one (sequence, kv head) pair of a full-size layer,
    generated at the pair's GLOBAL coordinates (no value depends on the batch size)."""
    one = oracle.new_cache(1, 1, cap, d)
    kh = I.gen_f16(seed, I.STREAM_K, layer, b, 1, kvh, 1, 0, L, d)
    vh = I.gen_f16(seed, I.STREAM_V, layer, b, 1, kvh, 1, 0, L, d)
    oracle.kv_append_quant(one, kh, vh, 0)
    return one


def check_sampled(got_cache, out, q, w, seed, L, what):
    B, Hkv, d, G = w.batch, w.kv_heads, w.head_dim, w.group_ratio
    for b, kvh in sample_pairs(B, Hkv):
        one = oracle_pair(seed, 0, b, kvh, L, d, w.capacity)
        for k in ("k_codes", "v_codes", "k_meta", "v_meta"):   # append bit-exact at full size
            assert np.array_equal(got_cache[k][b, kvh, :L], one[k][0, 0, :L]), (what, b, kvh, k)
        qh = q[b, kvh * G:(kvh + 1) * G].cpu().numpy()[None]
        ref = oracle.decode_attention_q4(one, qh, L)           # Hq/Hkv = G for a single kv head
        check_attention(out[b, kvh * G:(kvh + 1) * G].cpu().numpy(), ref[0], f"{what} (b={b}, kvh={kvh})")


@pytest.mark.parametrize("key", ["c1", "c2", "c3", "c4", "c5"])
def test_full_size_sampled_rows(lmo, key):
    """One layer at BASELINE.json full size, last decode step (L = s+n-1), the whole
    prompt+generation prefilled through lmo_kv_append_quant, then attention through
    lmo_decode_attention_q4 with the library's default schedule (num_splits=0) and fp32
    out; sampled (b, kv-head) pairs checked one by one against the oracle (c1: all)."""
    w = CONFIGS[key]
    seed = I.seed_for_config(w.index)
    L = w.max_len
    B, Hkv, d, G = w.batch, w.kv_heads, w.head_dim, w.group_ratio
    cache = lmo.KVCache.empty(B, Hkv, w.capacity, d)
    kf = torch.empty((B, Hkv, L, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, 0, 0, 0, 0)
    lmo.lmo_kv_append_quant(cache, kf, vf, pos0=0)
    del kf, vf
    q = torch.empty((B, w.q_heads, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, w.steps - 1, group=G)
    q = q.view(B, w.q_heads, d)
    out = lmo.lmo_decode_attention_q4(cache, q, L)
    torch.cuda.synchronize()
    got = cache_to_host(cache)
    if key == "c1":
        host = oracle.new_cache(B, Hkv, cache.capacity, d)
        oracle.kv_append_quant(host, I.gen_f16(seed, I.STREAM_K, 0, 0, B, 0, Hkv, 0, L, d),
                               I.gen_f16(seed, I.STREAM_V, 0, 0, B, 0, Hkv, 0, L, d), 0)
        for k in host:
            assert np.array_equal(got[k][:, :, :L], host[k][:, :, :L]), k
        ref = oracle.decode_attention_q4(host, q.cpu().numpy(), L, nthreads=8)
        check_attention(out.cpu().numpy(), ref, "c1 full")
        return
    check_sampled(got, out, q, w, seed, L, f"{key} attention L={L}")


@pytest.mark.parametrize("key", ["c2", "c3", "c4", "c5"])
def test_full_size_decode_step_bench_launch(lmo, key):
    """The launch bench.py times, at full size: lmo_decode_step_q4 (fused append of the
    new token at slot L-1 + attention over L) with LMO_STEP_CACHE_STABLE, the default
    schedule, fp32 out and a shared workspace, at the first and the last decode step of
    the workload (L = s+1 and L = s+n-1).  Sampled pairs vs the oracle: the appended
    row bit-exact, attention <= 2e-3."""
    w = CONFIGS[key]
    seed = I.seed_for_config(w.index)
    B, Hkv, d, G, s = w.batch, w.kv_heads, w.head_dim, w.group_ratio, w.prompt
    cache = lmo.KVCache.empty(B, Hkv, w.capacity, d)
    P_ = w.max_len - 1
    kf = torch.empty((B, Hkv, P_ + 1, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, 0, 0, 0, 0)
    ws = lmo.attention_workspace(B, Hkv, w.q_heads, d)
    for t in (1, w.steps):
        L = s + t
        cache.kv.fill_(0x5C)                       # stale bytes beyond the prefilled slots
        lmo.lmo_kv_append_quant(cache, kf[:, :, :L - 1].contiguous(), vf[:, :, :L - 1].contiguous(), pos0=0)
        q = torch.empty((B, w.q_heads, 1, d), dtype=torch.float16, device="cuda")
        lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, t - 1, group=G)
        q = q.view(B, w.q_heads, d)
        out = torch.empty((B, w.q_heads, d), dtype=torch.float32, device="cuda")
        lmo.lmo_decode_step_q4(cache, kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous(), q, L,
                               out=out, workspace=ws, flags=lmo.LMO_STEP_CACHE_STABLE)
        torch.cuda.synchronize()
        check_sampled(cache_to_host(cache), out, q, w, seed, L, f"{key} step t={t} L={L}")


# ------------------------------- attention on adversarial magnitudes --

def custom_layer(lmo, k, v, cap=None):
    """A q4 cache built from explicit fp16 K/V [B][Hkv][L][d] on both sides."""
    B, Hkv, L, d = k.shape
    cache = lmo.KVCache.empty(B, Hkv, cap or L, d)
    lmo.lmo_kv_append_quant(cache, dev(k), dev(v), pos0=0)
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    oracle.kv_append_quant(host, k, v, 0)
    return cache, host


def magnitude_case(name, B, Hkv, G, L, d, rng):
    """K, V, q of one adversarial case (legal inputs: finite fp16, include/lmo.h)."""
    n = lambda *sh: rng.standard_normal(sh)
    k, v, q = n(B, Hkv, L, d), n(B, Hkv, L, d), n(B, Hkv * G, d)
    if name.startswith("v_sigma_"):                      # small-magnitude V: tiny group scales
        v = v * float(name[len("v_sigma_"):])
    elif name == "v_subnormal":                          # V on the fp16 subnormal grid (scale < 2^-14)
        v = rng.integers(-40, 41, v.shape) * 2.0 ** -24
    elif name == "scale_zero_groups":                    # constant (scale-0) K and V groups, some rows all
        for x in (k, v):
            x.reshape(B, Hkv, L, d // 64, 64)[..., :] = np.where(
                rng.random((B, Hkv, L, d // 64, 1)) < 0.5, rng.standard_normal((B, Hkv, L, d // 64, 1)),
                x.reshape(B, Hkv, L, d // 64, 64))
        v[:, :, : L // 3] = 0.75
    elif name == "v_extremes":                           # +-65504 V
        v = rng.uniform(-65504, 65504, v.shape)
        v[..., 0], v[..., 1] = -65504, 65504
    elif name == "k_extremes_q_tiny":                    # +-65504 K met by subnormal-range q
        k = rng.uniform(-65504, 65504, k.shape)
        q = q * 3e-5
    elif name == "q_tiny":                               # |q| < 2^-10 (q/16 would be subnormal)
        q, k = q * 1e-4, k * 100.0
    elif name == "mixed_token_magnitudes":               # per-token V / K magnitudes over 8 / 4 decades
        v = v * 10.0 ** rng.uniform(-6, 2, (B, Hkv, L, 1))
        k = k * 10.0 ** rng.uniform(-3, 1, (B, Hkv, L, 1))
    elif name == "v_growing":                            # V scales grow along the sequence (E lowered late)
        v = v * 10.0 ** np.linspace(-5, 1, L)[None, None, :, None]
    f16 = lambda x: np.clip(x, -65504, 65504).astype(np.float16)
    return f16(k), f16(v), f16(q)


MAG_CASES = ["v_sigma_1e-5", "v_sigma_3e-5", "v_sigma_1e-4", "v_sigma_1e-3", "v_subnormal",
             "scale_zero_groups", "v_extremes", "k_extremes_q_tiny", "q_tiny", "mixed_token_magnitudes",
             "v_growing"]


@pytest.mark.parametrize("G,ns", [(1, 0), (8, 0), (1, 2), (4, -1), (2, -2)])
@pytest.mark.parametrize("name", MAG_CASES)
def test_attention_magnitude_edges(lmo, name, G, ns):
    """Attention over q4 caches of adversarial magnitude (tiny / subnormal / zero group
    scales, +-65504, tiny q), MHA and GQA, default / team / stream-K / SM-team schedules:
    <= 2e-3 normwise vs the oracle (the operand exponents of decode_attn.cu)."""
    rng = np.random.default_rng(zlib.crc32(f"{name}:{G}".encode()))
    B, Hkv, d, L = 2, 2, 128, 300
    k, v, q = magnitude_case(name, B, Hkv, G, L, d, rng)
    cache, host = custom_layer(lmo, k, v)
    out = lmo.lmo_decode_attention_q4(cache, dev(q), L, num_splits=ns)
    torch.cuda.synchronize()
    ref = oracle.decode_attention_q4(host, q, L, nthreads=8)
    check_attention(out.cpu().numpy(), ref, f"{name} G={G} ns={ns}")


@pytest.mark.parametrize("name", ["v_sigma_1e-5", "v_subnormal", "q_tiny", "mixed_token_magnitudes"])
def test_decode_step_magnitude_edges(lmo, name):
    """The fused step (append + attention) on adversarial magnitudes, d = 64 and 128."""
    for d, G in ((128, 1), (64, 8)):
        rng = np.random.default_rng(len(name) + d)
        B, Hkv, L = 3, 2, 97
        k, v, q = magnitude_case(name, B, Hkv, G, L, d, rng)
        cache, _ = custom_layer(lmo, np.ascontiguousarray(k[:, :, :L - 1]), np.ascontiguousarray(v[:, :, :L - 1]),
                                cap=L)
        out = lmo.lmo_decode_step_q4(cache, dev(k[:, :, L - 1]), dev(v[:, :, L - 1]), dev(q), L)
        torch.cuda.synchronize()
        host = oracle.new_cache(B, Hkv, cache.capacity, d)
        oracle.kv_append_quant(host, k, v, 0)
        ref = oracle.decode_attention_q4(host, q, L, nthreads=8)
        check_attention(out.cpu().numpy(), ref, f"step {name} d={d} G={G}")


# ------------------------------------------ fused decode step (A2+A3+A4) ----

@pytest.mark.parametrize("flags", [0, 1])
@pytest.mark.parametrize("B,Hkv,G,d,L,ns", [(4, 6, 1, 128, 300, 0), (2, 2, 8, 128, 129, 0),
                                            (3, 4, 2, 64, 77, 2), (2, 3, 1, 128, 40, 4),
                                            (2, 2, 4, 128, 200, 3), (1, 2, 1, 128, 1, 0),
                                            (3, 5, 1, 128, 33, 0), (2, 2, 8, 128, 16, 0),
                                            (4, 6, 1, 128, 300, -1), (3, 4, 8, 128, 129, -1),
                                            (5, 3, 1, 64, 77, -1), (2, 3, 1, 128, 1, -1),
                                            (7, 5, 2, 128, 47, -1), (4, 6, 1, 128, 300, -2),
                                            (3, 4, 8, 128, 129, -2), (5, 3, 1, 64, 77, -2),
                                            (2, 3, 1, 128, 1, -2), (64, 9, 1, 128, 47, -2),
                                            (80, 8, 8, 128, 129, 0), (100, 7, 2, 128, 300, 0),
                                            (64, 10, 1, 128, 90, 0)])
def test_decode_step_fused_append(lmo, B, Hkv, G, d, L, ns, flags):
    """lmo_decode_step_q4 == append(new token at L-1) then attention over L, for the
    team schedule (one launch) and the stream-K fallback (two launches)."""
    seed = 31 + L
    cap = L + 7
    kf = torch.empty((B, Hkv, L, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, 0, 0, 0, 0)
    cache = lmo.KVCache.empty(B, Hkv, cap, d)
    cache.kv.fill_(0x7B)
    if L > 1:
        lmo.lmo_kv_append_quant(cache, kf[:, :, :L - 1].contiguous(), vf[:, :, :L - 1].contiguous(), 0)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    out = lmo.lmo_decode_step_q4(cache, kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous(),
                                 q, L, num_splits=ns, flags=flags)
    torch.cuda.synchronize()
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    oracle.kv_append_quant(host, kf.cpu().numpy(), vf.cpu().numpy(), 0)
    got = cache_to_host(cache)
    for key in host:
        assert np.array_equal(got[key][:, :, :L], host[key][:, :, :L]), key
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), L, nthreads=8)
    check_attention(out.cpu().numpy(), ref, f"step B{B} Hkv{Hkv} G{G} d{d} L{L} ns{ns} flags{flags}")


@pytest.mark.parametrize("team,G", [(0, 2), (1, 2), (1, 1), (2, 1)])
def test_decode_step_per_sequence_lengths(lmo, team, G):
    B, Hkv, d, cap = 5, 3, 128, 208
    lens = np.array([200, 1, 0, 65, 129], np.int32)
    kf = torch.empty((B, Hkv, cap, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, 9, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, 9, I.STREAM_V, 0, 0, 0, 0)
    cache = lmo.KVCache.empty(B, Hkv, cap, d)
    lmo.lmo_kv_append_quant(cache, kf, vf, 0)               # whole capacity (stale beyond L)
    kn = torch.empty((B, Hkv, 1, d), dtype=torch.float16, device="cuda")
    vn = torch.empty_like(kn)
    lmo.lmo_gen_fill_f16(kn, 10, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vn, 10, I.STREAM_V, 0, 0, 0, 0)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, 9, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    out = lmo.lmo_decode_step_q4(cache, kn, vn, q, 0, seq_lens=dev(lens), num_splits=team)
    torch.cuda.synchronize()
    kh, vh = kf.cpu().numpy().copy(), vf.cpu().numpy().copy()
    for b in range(B):
        if lens[b] > 0:
            kh[b, :, lens[b] - 1] = kn.cpu().numpy()[b, :, 0]
            vh[b, :, lens[b] - 1] = vn.cpu().numpy()[b, :, 0]
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    oracle.kv_append_quant(host, kh, vh, 0)
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), np.maximum(lens, 1), nthreads=8)
    o = out.cpu().numpy()
    keep = lens > 0
    assert np.all(o[~keep] == 0)
    check_attention(o[keep], ref[keep], f"step per-sequence lengths team {team} G{G}")


def test_decode_loop_cache_stable_chain(lmo):
    """Layer-by-layer decode loop (4 layers x 3 steps, back to back on one stream) with
    LMO_STEP_CACHE_STABLE: every output matches the oracle."""
    B, H, d, s0, nl, steps = 3, 4, 128, 90, 4, 3
    cap = s0 + steps
    caches, hosts, outs = [], [], []
    kall = torch.empty((nl, B, H, cap, d), dtype=torch.float16, device="cuda")
    vall = torch.empty_like(kall)
    for l in range(nl):
        lmo.lmo_gen_fill_f16(kall[l], 77, I.STREAM_K, l, 0, 0, 0)
        lmo.lmo_gen_fill_f16(vall[l], 77, I.STREAM_V, l, 0, 0, 0)
        c = lmo.KVCache.empty(B, H, cap, d)
        lmo.lmo_kv_append_quant(c, kall[l, :, :, :s0].contiguous(), vall[l, :, :, :s0].contiguous(), 0)
        caches.append(c)
    q = torch.empty((nl, steps, B, H, 1, d), dtype=torch.float16, device="cuda")
    for l in range(nl):
        for t in range(steps):
            lmo.lmo_gen_fill_f16(q[l, t], 77, I.STREAM_Q, l, 0, 0, t)
    ws = lmo.attention_workspace(B, H, H, d)
    kn = [[kall[l, :, :, s0 + t].contiguous() for t in range(steps)] for l in range(nl)]
    vn = [[vall[l, :, :, s0 + t].contiguous() for t in range(steps)] for l in range(nl)]
    torch.cuda.synchronize()
    res = {}
    for t in range(steps):
        for l in range(nl):
            res[(l, t)] = lmo.lmo_decode_step_q4(caches[l], kn[l][t], vn[l][t], q[l, t].view(B, H, d),
                                                 s0 + t + 1, workspace=ws,
                                                 flags=lmo.LMO_STEP_CACHE_STABLE)
    torch.cuda.synchronize()
    for l in range(nl):
        host = oracle.new_cache(B, H, caches[l].capacity, d)
        oracle.kv_append_quant(host, kall[l].cpu().numpy(), vall[l].cpu().numpy(), 0)
        for t in range(steps):
            ref = oracle.decode_attention_q4(host, q[l, t].view(B, H, d).cpu().numpy(), s0 + t + 1,
                                             nthreads=8)
            check_attention(res[(l, t)].cpu().numpy(), ref, f"cache-stable chain layer {l} step {t}")


# ------------------------------------------------ §8(e): sharding invariance --

@pytest.mark.parametrize("G,d", [(1, 128), (8, 128), (2, 64)])
def test_sharded_step_bit_identical(lmo, G, d):
    """Batch sharding: the fused step on the two halves of a batch --
    each half its own cache, inputs generated at the global coordinates, as two ranks
    hold them -- is bit-identical to one full-batch call when the team size is fixed
    (num_splits=1: one warp per (sequence, kv head) pair, no cross-pair state)."""
    B, Hkv, L, seed = 8, 3, 211, 4242
    Hq = Hkv * G

    def run(b0, nb):
        cache = lmo.KVCache.empty(nb, Hkv, L, d)
        kf = torch.empty((nb, Hkv, L, d), dtype=torch.float16, device="cuda")
        vf = torch.empty_like(kf)
        lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, 0, b0, 0, 0)
        lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, 0, b0, 0, 0)
        lmo.lmo_kv_append_quant(cache, kf[:, :, :L - 1].contiguous(), vf[:, :, :L - 1].contiguous(), pos0=0)
        q = torch.empty((nb, Hq, 1, d), dtype=torch.float16, device="cuda")
        lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, b0, 0, 0, group=G)
        out = lmo.lmo_decode_step_q4(cache, kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous(),
                                     q.view(nb, Hq, d), L, num_splits=1, flags=lmo.LMO_STEP_CACHE_STABLE)
        torch.cuda.synchronize()
        f = cache_to_host(cache)                           # tokens >= L: never written
        return out.cpu(), {k: torch.from_numpy(np.ascontiguousarray(v[:, :, :L])) for k, v in f.items()}

    full, kv_full = run(0, B)
    lo, kv_lo = run(0, B // 2)
    hi, kv_hi = run(B // 2, B // 2)
    assert torch.equal(torch.cat([lo, hi]), full)
    for k in kv_full:
        assert torch.equal(torch.cat([kv_lo[k], kv_hi[k]]), kv_full[k]), k


# ------------------------------------ NEXT-1: FlexGen-exact step (reading 13b) --

@pytest.mark.parametrize("B,Hkv,G,d,L,ns,flags", [
    (4, 6, 1, 128, 300, 0, 0), (2, 2, 8, 128, 129, 0, 0), (3, 4, 2, 64, 77, 2, 0), (2, 3, 1, 128, 40, 4, 0),
    (2, 2, 4, 128, 200, 3, 0), (1, 2, 1, 128, 1, 0, 0), (2, 2, 8, 128, 1, 0, 0), (3, 5, 1, 128, 33, -1, 0),
    (3, 4, 8, 128, 129, -1, 0), (4, 6, 1, 128, 300, -2, 0), (2, 2, 8, 128, 16, 0, 0), (2, 2, 8, 128, 17, 0, 0),
    (4, 6, 1, 128, 300, 0, 1), (2, 2, 8, 128, 129, 0, 1), (64, 9, 1, 128, 47, 0, 1)])
def test_decode_step_flexgen_exact(lmo, B, Hkv, G, d, L, ns, flags):
    """LMO_STEP_FLEXGEN_EXACT: the new token's raw fp16 K/V in its own attention (oracle T6),
    while the cache still receives its quantized row at slot L-1 (bit-exact)."""
    seed = 77 + L + G
    cap = L + 7
    kf = torch.empty((B, Hkv, L, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, seed, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, seed, I.STREAM_V, 0, 0, 0, 0)
    cache = lmo.KVCache.empty(B, Hkv, cap, d)
    cache.kv.fill_(0x3C)
    if L > 1:
        lmo.lmo_kv_append_quant(cache, kf[:, :, :L - 1].contiguous(), vf[:, :, :L - 1].contiguous(), 0)
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, seed, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    kn, vn = kf[:, :, L - 1].contiguous(), vf[:, :, L - 1].contiguous()
    out = lmo.lmo_decode_step_q4(cache, kn, vn, q, L, num_splits=ns,
                                 flags=lmo.LMO_STEP_FLEXGEN_EXACT | (lmo.LMO_STEP_CACHE_STABLE if flags else 0))
    torch.cuda.synchronize()
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    oracle.kv_append_quant(host, kf.cpu().numpy(), vf.cpu().numpy(), 0)
    got = cache_to_host(cache)
    for key in host:
        assert np.array_equal(got[key][:, :, :L], host[key][:, :, :L]), key
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), L, nthreads=8, k_last=kn.cpu().numpy(),
                                     v_last=vn.cpu().numpy())
    o = out.cpu().numpy()
    check_attention(o, ref, f"flexgen B{B} Hkv{Hkv} G{G} d{d} L{L} ns{ns} flags{flags}")
    if L == 1:   # closed form: the raw V row (fp32 of fp16) within rounding of the 1/l normalisation
        want = np.repeat(vn.cpu().numpy().astype(np.float64), G, axis=1)
        assert np.max(np.abs(o - want)) <= 1e-6 * max(1.0, np.abs(want).max())


def test_decode_step_flexgen_exact_per_sequence_lengths(lmo):
    B, Hkv, G, d, cap = 5, 3, 2, 128, 208
    lens = np.array([200, 1, 0, 65, 129], np.int32)
    kf = torch.empty((B, Hkv, cap, d), dtype=torch.float16, device="cuda")
    vf = torch.empty_like(kf)
    lmo.lmo_gen_fill_f16(kf, 19, I.STREAM_K, 0, 0, 0, 0)
    lmo.lmo_gen_fill_f16(vf, 19, I.STREAM_V, 0, 0, 0, 0)
    cache = lmo.KVCache.empty(B, Hkv, cap, d)
    lmo.lmo_kv_append_quant(cache, kf, vf, 0)
    kn = (torch.randn((B, Hkv, d), device="cuda") * 2).half()
    vn = torch.randn((B, Hkv, d), device="cuda").half()
    q = torch.empty((B, Hkv * G, 1, d), dtype=torch.float16, device="cuda")
    lmo.lmo_gen_fill_f16(q, 19, I.STREAM_Q, 0, 0, 0, 0, group=G)
    q = q.view(B, Hkv * G, d)
    out = lmo.lmo_decode_step_q4(cache, kn, vn, q, 0, seq_lens=dev(lens), flags=lmo.LMO_STEP_FLEXGEN_EXACT)
    torch.cuda.synchronize()
    kh, vh = kf.cpu().numpy().copy(), vf.cpu().numpy().copy()
    for b in range(B):
        if lens[b] > 0:
            kh[b, :, lens[b] - 1] = kn.cpu().numpy()[b]
            vh[b, :, lens[b] - 1] = vn.cpu().numpy()[b]
    host = oracle.new_cache(B, Hkv, cache.capacity, d)
    oracle.kv_append_quant(host, kh, vh, 0)
    ref = oracle.decode_attention_q4(host, q.cpu().numpy(), np.maximum(lens, 1), nthreads=8,
                                     k_last=kn.cpu().numpy(), v_last=vn.cpu().numpy())
    o = out.cpu().numpy()
    keep = lens > 0
    assert np.all(o[~keep] == 0)
    check_attention(o[keep], ref[keep], "flexgen per-sequence lengths")
