"""Pins of the CPU oracle against what the paper and the mathematics fix.

None of these re-types the oracle's formulas: each checks a property that a
plausible mistake in lmo_oracle.c (dropped term, wrong sign/index, swapped
nibble, wrong rounding direction, transposed operand) would violate.

Citations: PAPER.md Alg 2, Eq 10, Eq 11,
attention definition.  Readings Q0-Q8/D1/T1-T5: DESIGN.md "Readings".
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle

RNG_SEED = 1234


def F(bits):
    """Exact Fraction value of an fp16 bit pattern, computed independently of
    the oracle via numpy's float16 -> float64 conversion (exact)."""
    return Fraction(float(np.uint16(bits).view(np.float16)))


def fp16_from_fraction_down(x: Fraction) -> float:
    return float(np.float16(float(x)))


def quant_groups(x):
    """Quantize a flat fp16 vector of whole 64-groups; returns (codes[n], mins, scales) with
    codes unpacked by plain indexing (low nibble = even element, reading Q8)."""
    x = np.asarray(x, dtype=np.float16)
    n = x.size
    c, m = oracle.quantize_groupwise(x, 1, n, 1)
    c = c.reshape(-1)
    codes = np.empty(((n + 63) // 64) * 64, dtype=np.int64)
    codes[0::2] = c & 0xF
    codes[1::2] = c >> 4
    m = m.reshape(-1, 2)
    return codes, m[:, 0], m[:, 1]


# ----------------------------------------------------------------- fp16 ----

def test_rn16_matches_numpy_conversion():
    """RN16 helper == numpy's correctly rounded float64->float16 cast (a library
    routine), over random magnitudes incl. subnormals, ties and overflow."""
    rng = np.random.default_rng(RNG_SEED)
    xs = np.concatenate([
        rng.standard_normal(20000) * 10.0 ** rng.uniform(-9, 5, 20000),
        # exact ties between adjacent fp16 values (normal and subnormal)
        (np.arange(1, 4000, dtype=np.float64) + 0.5) * 2.0 ** -24,
        (np.arange(1024, 2048, dtype=np.float64) + 0.5) * 2.0 ** -10,
        np.array([65504.0, 65519.99, 65520.0, 1e9, -0.0, 0.0, 2.0 ** -25, 2.0 ** -25 * 1.0000001]),
    ])
    for v in xs:
        want = np.float64(v).astype(np.float16).view(np.uint16)
        assert oracle.rn16(float(v)) == int(want), v


def test_ru16_is_round_up():
    """RU16(x) is the least fp16 >= x (definition of rounding toward +inf)."""
    rng = np.random.default_rng(RNG_SEED + 1)
    xs = np.concatenate([np.abs(rng.standard_normal(5000)) * 10.0 ** rng.uniform(-9, 4, 5000),
                         np.arange(0, 3000) * 2.0 ** -24])
    for v in xs:
        hb = oracle.ru16(float(v))
        assert F(hb) >= Fraction(float(v))
        if hb > 0:
            assert F(hb - 1) < Fraction(float(v))


# ------------------------------------------------------- quantize (Alg 2) --

def on_grid_group(rng, mn, step):
    k = rng.integers(0, 16, 64)
    k[rng.choice(64, 2, replace=False)] = [0, 15]
    x = (np.float64(mn) + k * np.float64(step)).astype(np.float16)
    assert np.all(x.astype(np.float64) == mn + k * step)  # exact on the grid
    return x, k


@pytest.mark.parametrize("mn,step", [(-3.0, 0.25), (0.0, 1.0), (-1.5, 3 * 2.0 ** -5),
                                     (100.0, 2.0), (-0.75, 5 * 2.0 ** -8)])
def test_on_grid_round_trip_exact(mn, step):
    """Values mn + k*step (k=0..15, both ends present) quantize to code k and
    dequantize (Eq 11) back to x bit-exactly."""
    rng = np.random.default_rng(RNG_SEED + 2)
    x, k = on_grid_group(rng, mn, step)
    codes, mins, scales = quant_groups(x)
    assert np.array_equal(codes, k)
    assert F(mins[0]) == Fraction(mn) and F(scales[0]) == Fraction(step)
    c, m = oracle.quantize_groupwise(x, 1, 64, 1)
    y = oracle.dequantize_groupwise(c, m, 1, 64, 1).reshape(-1)
    assert np.array_equal(y.view(np.uint16), x.view(np.uint16))


@pytest.mark.parametrize("v", [0.0, 1.0, -7.25, 65504.0, -65504.0, 2.0 ** -24])
def test_constant_group(v):
    """max == min: Eq 10 is 0/0; reading 1: scale 0, all codes 0, dequant == x."""
    x = np.full(64, v, dtype=np.float16)
    codes, mins, scales = quant_groups(x)
    assert np.all(codes == 0) and scales[0] == 0
    assert F(mins[0]) == Fraction(float(np.float16(v)))
    c, m = oracle.quantize_groupwise(x, 1, 64, 1)
    y = oracle.dequantize_groupwise(c, m, 1, 64, 1).reshape(-1)
    assert np.array_equal(y, x)


def adversarial_groups(rng):
    g = []
    g.append(rng.standard_normal(64))                                # plain
    g.append(rng.standard_normal(64) * 8)                            # outlier channel scale
    x = rng.standard_normal(64); x[5] = 300.0; g.append(x)           # one outlier
    g.append(rng.uniform(-65504, 65504, 64))                         # full range
    x = rng.uniform(-1, 1, 64); x[0], x[1] = -65504, 65504; g.append(x)  # extremes
    g.append(rng.integers(-3, 4, 64) * 2.0 ** -24)                   # subnormal range
    g.append(1.0 + rng.integers(0, 5, 64) * 2.0 ** -10)              # tiny range at 1.0
    g.append(rng.uniform(1000, 1001, 64))                            # offset group
    x = rng.standard_normal(64); x[::3] = -0.0; g.append(x)           # signed zeros
    return [np.asarray(v, dtype=np.float64).astype(np.float16) for v in g]


def test_reconstruction_error_invariant():
    """|x - (mn + c*scale)| <= scale/2 * (1 + 2^-16), evaluated exactly, for every
    element; scale >= (max-min)/15 (so no in-range value is clipped);
    scale == 0 iff the group is constant; min -> code 0."""
    rng = np.random.default_rng(RNG_SEED + 3)
    groups = adversarial_groups(rng) + [rng.standard_normal(64).astype(np.float16) * 3
                                        for _ in range(200)]
    for x in groups:
        codes, mins, scales = quant_groups(x)
        mn, sc = F(mins[0]), F(scales[0])
        xs = [Fraction(float(v)) for v in x.astype(np.float64)]
        assert mn == min(xs)
        assert sc * 15 >= max(xs) - min(xs) or sc * 15 >= Fraction(
            float(np.float32(float(max(xs) - min(xs)))))
        assert (sc == 0) == (max(xs) == min(xs))
        for xi, ci in zip(xs, codes):
            assert 0 <= ci <= 15
            err = abs(xi - (mn + int(ci) * sc))
            assert err <= sc / 2 * (1 + Fraction(1, 2 ** 16)), (xi, ci, mn, sc)
            if xi == mn:
                assert ci == 0


def test_max_maps_to_15_for_normal_scale_and_monotone():
    rng = np.random.default_rng(RNG_SEED + 4)
    for _ in range(300):
        x = (rng.standard_normal(64) * 10.0 ** rng.uniform(-3, 3)).astype(np.float16)
        codes, mins, scales = quant_groups(x)
        if F(scales[0]) >= Fraction(2.0 ** -14):
            assert codes[int(np.argmax(x))] == 15
        order = np.argsort(x.astype(np.float64), kind="stable")
        assert np.all(np.diff(codes[order]) >= 0)   # monotone in x


def test_ties_round_half_to_even():
    """Reading 2: with a power-of-two step (scale 1, inv 1 exact), half-step
    values land on the even neighbour."""
    x = np.zeros(64)
    x[0], x[1] = 0.0, 15.0
    halves = [0.5, 1.5, 2.5, 3.5, 4.5, 13.5, 14.5]
    x[2:2 + len(halves)] = halves
    codes, mins, scales = quant_groups(x.astype(np.float16))
    assert F(scales[0]) == 1
    assert list(codes[2:2 + len(halves)]) == [0, 2, 2, 4, 4, 14, 14]


def test_q5_reciprocal_then_multiply_golden():
    """Reading Q5 (Eq 10; DESIGN.md "Readings" Q5): t = RN32(RN32(x - mn) *
    RN32(1/scale)), NOT RN32((x - mn) / scale).  Hand-computed group:
      mn = -0.85595703125, mx = 0.93115234375 (both exact fp16), the rest 0;
      range = 1.787109375, range/15 = 0.119140625 exactly (fp16 0x2FA0);
      x = 0.51416015625: d = x - mn = 1.3701171875 = 1403/1024 exactly;
      d / scale = 1403/122 = 11.5 exactly -> half-even rint -> 12 (division);
      RN32(1/scale) = 8.393442... (rounded down), d * inv -> RN32 = 11.499999 -> 11.
    So the oracle must emit code 11 for element 2 (a division mutation gives 12)."""
    x = np.zeros(64)
    x[0], x[1], x[2] = -0.85595703125, 0.93115234375, 0.51416015625
    codes, mins, scales = quant_groups(x.astype(np.float16))
    assert int(scales[0]) == 0x2FA0                  # 0.119140625
    assert int(mins[0]) == 0xBAD9                    # -0.85595703125
    assert int(codes[2]) == 11
    assert int(codes[0]) == 0 and int(codes[1]) == 15


def test_d1_rn32_before_rn16_golden():
    """Reading D1 (Eq 11; DESIGN.md "Readings" D1): y = RN16(RN32(c*scale +
    mn)).  Hand-computed group: 62 elements of 2^-24 (the min), 10.0 and 2.0.
      range = RN32(10 - 2^-24) = 10; scale = RU16(10/15) = 683/1024 (fp16 0x3956);
      x = 2.0: d = RN32(2 - 2^-24) = 2 (tie, even), t = 2 * RN32(1/scale) = 2.9985 -> code 3;
      exact = 3 * 683/1024 + 2^-24 = 2 + 2^-10 + 2^-24;
      RN32(exact) = 2 + 2^-10 (ulp32 at 2 is 2^-22) -> RN16: exact half-ulp tie -> 2.0 = 0x4000;
      without the RN32 step the 2^-24 breaks the tie upward -> 0x4001."""
    x = np.full(64, 2.0 ** -24)
    x[0], x[1] = 10.0, 2.0
    xh = x.astype(np.float16)
    c, m = oracle.quantize_groupwise(xh, 1, 64, 1)
    assert int(m.reshape(-1)[1]) == 0x3956
    codes, _, _ = quant_groups(xh)
    assert int(codes[1]) == 3 and int(codes[0]) == 15
    y = oracle.dequantize_groupwise(c, m, 1, 64, 1).reshape(-1).view(np.uint16)
    assert int(y[1]) == 0x4000
    assert int(y[2]) == 0x0001                       # the min itself: code 0 -> mn exactly


def test_pack_byte_vectors():
    """Reading 9 (low nibble = even element): codes 0..15 -> 0x10 0x32 ... 0xFE."""
    x = (np.arange(64) % 16).astype(np.float16)
    c, m = oracle.quantize_groupwise(x, 1, 64, 1)
    assert list(c.reshape(-1)[:8]) == [0x10, 0x32, 0x54, 0x76, 0x98, 0xBA, 0xDC, 0xFE]
    x = (15 - np.arange(64) % 16).astype(np.float16)
    c, m = oracle.quantize_groupwise(x, 1, 64, 1)
    assert list(c.reshape(-1)[:2]) == [0xEF, 0xCD]


def test_padding_participates_in_minmax():
    """Reading 7: n not a multiple of 64 -> +0 pads enter min/max (Alg 2 l.5-6
    precede l.9-10); padded output shapes use ceil(n/64) groups."""
    x = np.concatenate([np.full(64, 2.0), [1.5]]).astype(np.float16)   # n = 65
    c, m = oracle.quantize_groupwise(x, 1, 65, 1)
    assert c.shape == (1, 64, 1) and m.shape == (1, 2, 1, 2)
    assert F(m[0, 1, 0, 0]) == 0                 # group 2: min is the +0 pad
    sc = F(m[0, 1, 0, 1])
    assert sc * 15 >= Fraction(1.5) and (sc - F(m[0, 1, 0, 1] - 1)) * 15 > 0
    assert c[0, 32, 0] & 0xF == 15              # element 64 (= 1.5) is the max
    assert np.all(c[0, 33:, 0] == 0)            # pads are the min -> code 0
    y = oracle.dequantize_groupwise(c, m, 1, 65, 1)
    assert y.shape == (1, 65, 1)


def test_signed_zero_canonical():
    x = np.full(64, -0.0, dtype=np.float16)
    codes, mins, scales = quant_groups(x)
    assert mins[0] == 0x0000 and scales[0] == 0 and np.all(codes == 0)


def test_strided_quantize_dim_matches_transpose():
    """quantize_dim with inner > 1 equals quantizing the transposed tensor
    with inner == 1 (layout-only change)."""
    rng = np.random.default_rng(RNG_SEED + 5)
    x = (rng.standard_normal((3, 128, 5)) * 2).astype(np.float16)
    c, m = oracle.quantize_groupwise(x, 3, 128, 5)
    xt = np.ascontiguousarray(x.transpose(0, 2, 1))
    ct, mt = oracle.quantize_groupwise(xt, 15, 128, 1)
    assert np.array_equal(c.transpose(0, 2, 1).reshape(15, 64), ct.reshape(15, 64))
    assert np.array_equal(m.transpose(0, 2, 1, 3).reshape(15, 2, 2), mt.reshape(15, 2, 2))


# --------------------------------------------------------- dequantize -------

def test_dequant_within_double_rounding_bound():
    """D1: y = RN16(RN32(c*scale + mn)) lies within 1/2 ulp16 + 1/2 ulp32 of the
    exact real c*scale + mn."""
    rng = np.random.default_rng(RNG_SEED + 6)
    for _ in range(100):
        x = (rng.standard_normal(128) * 10.0 ** rng.uniform(-4, 4)).astype(np.float16)
        c, m = oracle.quantize_groupwise(x, 1, 128, 1)
        y = oracle.dequantize_groupwise(c, m, 1, 128, 1).reshape(-1)
        codes, mins, scales = quant_groups(x)
        for j in range(128):
            exact = F(mins[j // 64]) + int(codes[j]) * F(scales[j // 64])
            yj = Fraction(float(y[j]))
            if exact == 0:
                assert yj == 0
                continue
            e16 = math.frexp(abs(float(exact)))[1] - 1
            ulp16 = Fraction(2) ** max(e16 - 10, -24)
            ulp32 = Fraction(2) ** max(e16 - 23, -149)
            assert abs(yj - exact) <= ulp16 / 2 + ulp32 / 2


# ------------------------------------------------------------ append --------

def test_append_equals_quantize_and_leaves_other_slots():
    """KV append (Eq 7) == Alg 2 on the same rows; canary bytes outside
    [pos, pos+n_new) are untouched."""
    rng = np.random.default_rng(RNG_SEED + 7)
    B, H, cap, d, n_new = 2, 3, 32, 128, 3
    cache = oracle.new_cache(B, H, cap, d, fill=0xA5)
    k = (rng.standard_normal((B, H, n_new, d)) * 2).astype(np.float16)
    v = (rng.standard_normal((B, H, n_new, d))).astype(np.float16)
    pos = np.array([5, 20], dtype=np.int32)
    oracle.kv_append_quant(cache, k, v, pos)
    for b in range(B):
        for name, src in (("k", k), ("v", v)):
            c, m = oracle.quantize_groupwise(src[b], H * n_new, d, 1)
            got_c = cache[name + "_codes"][b, :, pos[b]:pos[b] + n_new]
            got_m = cache[name + "_meta"][b, :, pos[b]:pos[b] + n_new]
            assert np.array_equal(got_c.reshape(-1), c.reshape(-1))
            assert np.array_equal(got_m.reshape(-1), m.reshape(-1))
            mask = np.ones(cap, dtype=bool)
            mask[pos[b]:pos[b] + n_new] = False
            assert np.all(cache[name + "_codes"][b][:, mask] == 0xA5)
            assert np.all(cache[name + "_meta"][b][:, mask] == 0xA5A5)


def test_append_rejects_overflow():
    cache = oracle.new_cache(1, 1, 8, 64)
    k = np.zeros((1, 1, 2, 64), np.float16)
    with pytest.raises(ValueError):
        oracle.kv_append_quant(cache, k, k, [7])


# ---------------------------------------------------------- attention -------

def random_cache(rng, B, Hkv, L, d, cap=None):
    cap = cap or L
    cache = oracle.new_cache(B, Hkv, cap, d)
    k = (rng.standard_normal((B, Hkv, L, d)) * 1.5).astype(np.float16)
    v = rng.standard_normal((B, Hkv, L, d)).astype(np.float16)
    oracle.kv_append_quant(cache, k, v, 0)
    return cache


def exact_rows(cache, name, b, h, L):
    """Exact dequantized rows as Fractions via plain unpacking (independent of
    the oracle's deq_elem)."""
    codes = cache[name + "_codes"][b, h, :L]
    meta = cache[name + "_meta"][b, h, :L]
    d = codes.shape[-1] * 2
    rows = []
    for j in range(L):
        row = []
        for i in range(d):
            byte = int(codes[j, i // 2])
            c = byte & 0xF if i % 2 == 0 else byte >> 4
            row.append(F(meta[j, i // 64, 0]) + c * F(meta[j, i // 64, 1]))
        rows.append(row)
    return rows


def brute_attention(q, krows, vrows, sigma):
    """Independent formula: no max subtraction, math.fsum, exact dequant."""
    qf = [float(v) for v in q]
    z = [sigma * math.fsum(qi * float(kj) for qi, kj in zip(qf, kr)) for kr in krows]
    p = [math.exp(zj) for zj in z]
    s = math.fsum(p)
    d = len(vrows[0])
    return np.array([math.fsum(pj * float(vr[i]) for pj, vr in zip(p, vrows)) / s
                     for i in range(d)])


@pytest.mark.parametrize("L,d,Hq,Hkv", [(1, 64, 2, 2), (5, 64, 4, 2), (8, 64, 3, 1), (7, 128, 2, 1)])
def test_attention_brute_force_tiny(L, d, Hq, Hkv):
    rng = np.random.default_rng(RNG_SEED + 8 + L)
    B = 2
    cache = random_cache(rng, B, Hkv, L, d)
    q = rng.standard_normal((B, Hq, d)).astype(np.float16)
    sigma = 1 / math.sqrt(d)
    out = oracle.decode_attention_q4(cache, q, L, sigma)
    G = Hq // Hkv
    for b in range(B):
        for h in range(Hq):
            kv = h // G                               # T1: contiguous GQA map
            ref = brute_attention(q[b, h], exact_rows(cache, "k", b, kv, L),
                                  exact_rows(cache, "v", b, kv, L), sigma)
            assert np.max(np.abs(out[b, h] - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


# ------------------------------- T6: FlexGen-exact new token (reading 13b) --

def test_flexgen_exact_single_token_is_raw_v():
    """Closed form: with L = 1 the only token has softmax weight 1, so the output is
    the new token's RAW fp16 V row exactly (not its 4-bit reconstruction)."""
    rng = np.random.default_rng(RNG_SEED + 30)
    d, B, Hkv, G = 128, 2, 3, 2
    cache = random_cache(rng, B, Hkv, 4, d)
    k_last = (rng.standard_normal((B, Hkv, d)) * 3).astype(np.float16)
    v_last = (rng.standard_normal((B, Hkv, d)) * 0.7).astype(np.float16)
    q = rng.standard_normal((B, Hkv * G, d)).astype(np.float16)
    o = oracle.decode_attention_q4(cache, q, 1, k_last=k_last, v_last=v_last)
    for b in range(B):
        for h in range(Hkv * G):
            assert np.array_equal(o[b, h], v_last[b, h // G].astype(np.float64))
    # and the quantized path does NOT reproduce it (v_last is off the q4 grid)
    oq = oracle.decode_attention_q4(cache, q, 1)
    assert not np.array_equal(oq, o)


@pytest.mark.parametrize("L,d,Hq,Hkv", [(2, 64, 2, 2), (6, 64, 4, 2), (5, 128, 2, 1)])
def test_flexgen_exact_brute_force_tiny(L, d, Hq, Hkv):
    """Independent brute force: tokens 0..L-2 from the exact dequantized cache, token L-1
    from the raw fp16 K/V (math.fsum, no max subtraction)."""
    rng = np.random.default_rng(RNG_SEED + 31 + L)
    B = 2
    cache = random_cache(rng, B, Hkv, L, d)
    k_last = (rng.standard_normal((B, Hkv, d)) * 1.5).astype(np.float16)
    v_last = rng.standard_normal((B, Hkv, d)).astype(np.float16)
    q = rng.standard_normal((B, Hq, d)).astype(np.float16)
    sigma = 1 / math.sqrt(d)
    out = oracle.decode_attention_q4(cache, q, L, sigma, k_last=k_last, v_last=v_last)
    G = Hq // Hkv
    for b in range(B):
        for h in range(Hq):
            kv = h // G
            kr = exact_rows(cache, "k", b, kv, L - 1) + [[Fraction(float(x)) for x in k_last[b, kv]]]
            vr = exact_rows(cache, "v", b, kv, L - 1) + [[Fraction(float(x)) for x in v_last[b, kv]]]
            ref = brute_attention(q[b, h], kr, vr, sigma)
            assert np.max(np.abs(out[b, h] - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


def test_flexgen_exact_equals_quantized_on_grid():
    """When the new token's K/V lie on their own q4 grid (mn + k*step with a power-of-two
    step, codes 0..15 present), quantization loses nothing, so the FlexGen-exact and the
    quantized readings coincide exactly."""
    rng = np.random.default_rng(RNG_SEED + 32)
    B, Hkv, d, L = 2, 2, 128, 9
    k = (rng.standard_normal((B, Hkv, L, d))).astype(np.float16)
    v = (rng.standard_normal((B, Hkv, L, d))).astype(np.float16)
    for x in (k, v):                                  # last token on-grid, every group
        for b in range(B):
            for h in range(Hkv):
                for gi in range(d // 64):
                    kk = rng.integers(0, 16, 64)
                    kk[:2] = [0, 15]
                    x[b, h, L - 1, gi * 64:(gi + 1) * 64] = (-1.0 + kk * 0.125).astype(np.float16)
    cache = oracle.new_cache(B, Hkv, L, d)
    oracle.kv_append_quant(cache, k, v, 0)
    q = rng.standard_normal((B, Hkv, d)).astype(np.float16)
    a = oracle.decode_attention_q4(cache, q, L)
    f = oracle.decode_attention_q4(cache, q, L, k_last=k[:, :, L - 1], v_last=v[:, :, L - 1])
    assert np.array_equal(a, f)


def test_attention_closed_forms():
    rng = np.random.default_rng(RNG_SEED + 9)
    d, L = 64, 6
    cache = random_cache(rng, 1, 1, L, d)
    vrows = np.array([[float(x) for x in r] for r in exact_rows(cache, "v", 0, 0, L)])
    # L = 1 -> o = v_0
    o = oracle.decode_attention_q4(cache, rng.standard_normal((1, 1, d)).astype(np.float16), 1)
    assert np.allclose(o[0, 0], vrows[0], rtol=0, atol=1e-15)
    # q = 0 -> uniform weights -> mean of the V rows
    o = oracle.decode_attention_q4(cache, np.zeros((1, 1, d), np.float16), L)
    assert np.allclose(o[0, 0], vrows.mean(axis=0), rtol=0, atol=1e-13)
    # one score >= 100 above the rest -> o = that v within e^-100
    c2 = oracle.new_cache(1, 1, L, d)
    k = np.zeros((1, 1, L, d), np.float16)
    k[0, 0, 3, :] = 8.0                     # only token 3 has a non-zero key
    v = rng.standard_normal((1, 1, L, d)).astype(np.float16)
    oracle.kv_append_quant(c2, k, v, 0)
    q = np.full((1, 1, d), 4.0, np.float16)  # z_3 = 4*8*64/8 = 256
    o = oracle.decode_attention_q4(c2, q, L)
    v3 = np.array([float(x) for x in exact_rows(c2, "v", 0, 0, L)[3]])
    assert np.allclose(o[0, 0], v3, rtol=0, atol=1e-40 + 1e-12)
    # all V rows equal -> o = that row
    c3 = oracle.new_cache(1, 1, L, d)
    vrow = rng.standard_normal(d).astype(np.float16)
    vv = np.broadcast_to(vrow, (1, 1, L, d)).copy()
    oracle.kv_append_quant(c3, rng.standard_normal((1, 1, L, d)).astype(np.float16), vv, 0)
    o = oracle.decode_attention_q4(c3, rng.standard_normal((1, 1, d)).astype(np.float16), L)
    r0 = np.array([float(x) for x in exact_rows(c3, "v", 0, 0, 1)[0]])
    assert np.allclose(o[0, 0], r0, rtol=1e-14, atol=1e-14)


def test_attention_permutation_invariant_and_lens():
    rng = np.random.default_rng(RNG_SEED + 10)
    B, Hkv, L, d = 2, 2, 40, 128
    cache = random_cache(rng, B, Hkv, L, d)
    q = rng.standard_normal((B, 4, d)).astype(np.float16)
    o = oracle.decode_attention_q4(cache, q, L)
    perm = rng.permutation(L)
    pc = {k: np.ascontiguousarray(v[:, :, perm]) for k, v in cache.items()}
    op = oracle.decode_attention_q4(pc, q, L)
    assert np.allclose(o, op, rtol=1e-12, atol=1e-12)
    # per-sequence lengths: row b uses only its first lens[b] tokens
    lens = np.array([40, 13], np.int32)
    ol = oracle.decode_attention_q4(cache, q, lens)
    sub = {k: np.ascontiguousarray(v[1:2, :, :13]) for k, v in cache.items()}
    o1 = oracle.decode_attention_q4(sub, q[1:2], 13)
    assert np.allclose(ol[1], o1[0], rtol=0, atol=0)
    assert np.allclose(ol[0], o[0], rtol=0, atol=0)


def test_attention_threads_identical():
    rng = np.random.default_rng(RNG_SEED + 11)
    cache = random_cache(rng, 3, 2, 33, 64)
    q = rng.standard_normal((3, 4, 64)).astype(np.float16)
    a = oracle.decode_attention_q4(cache, q, 33, nthreads=1)
    b = oracle.decode_attention_q4(cache, q, 33, nthreads=5)
    assert np.array_equal(a, b)


# ------------------------------------------------------------ W4A16 (NEXT-3)
def on_grid_matrix(rng, N, K, int_valued=True):
    """W [N][K] whose every 64-group is on its own grid mn + k*step (k = 0..15,
    both ends present), so Alg 2 + Eq 11 reproduce W exactly (pinned above)."""
    W = np.zeros((N, K), np.float64)
    for n in range(N):
        for g in range(K // 64):
            mn = float(rng.integers(-8, 8)) if int_valued else float(rng.integers(-64, 64)) / 8
            step = float(rng.integers(1, 4)) if int_valued else float(rng.integers(1, 9)) / 16
            k = rng.integers(0, 16, 64)
            k[rng.choice(64, 2, replace=False)] = [0, 15]
            W[n, g * 64:(g + 1) * 64] = mn + k * step
    assert np.array_equal(W.astype(np.float16).astype(np.float64), W)
    return W


def test_w4a16_on_grid_integer_exact():
    """y = x W^T (Eq 4's dequan_wgt then matmul) on integer-valued
    x and on-grid integer W: every product and partial sum is an integer far
    below 2^53, so the oracle must reproduce the exact integer matmul of the
    ORIGINAL W -- a wrong code, group min/scale, k index or transpose fails."""
    rng = np.random.default_rng(RNG_SEED + 40)
    N, K, B = 7, 192, 5
    W = on_grid_matrix(rng, N, K)
    x = rng.integers(-20, 21, (B, K)).astype(np.float64)
    c, m = oracle.quantize_groupwise(W.astype(np.float16), N, K, 1)
    y = oracle.w4a16_linear(c, m, N, K, x.astype(np.float16))
    want = np.array([[int(sum(int(x[b, k]) * int(W[n, k]) for k in range(K))) for n in range(N)]
                     for b in range(B)], dtype=np.float64)
    assert np.array_equal(y, want)


def test_w4a16_unit_vectors_pick_dequantized_weights():
    """x = e_k picks column k: y[k][n] = W~[n][k].  On-grid W (non-integer
    steps) must come back exactly; off-grid W within the Eq 10/11 bound
    |W - W~| <= scale/2 (+ the fp16 rounding of D1)."""
    rng = np.random.default_rng(RNG_SEED + 41)
    N, K = 6, 128
    W = on_grid_matrix(rng, N, K, int_valued=False)
    c, m = oracle.quantize_groupwise(W.astype(np.float16), N, K, 1)
    y = oracle.w4a16_linear(c, m, N, K, np.eye(K, dtype=np.float16))
    assert np.array_equal(y, W.T)
    Wr = (rng.standard_normal((N, K)) * 0.05).astype(np.float16)
    c, m = oracle.quantize_groupwise(Wr, N, K, 1)
    y = oracle.w4a16_linear(c, m, N, K, np.eye(K, dtype=np.float16))
    scale = np.array([[F(m[n, k // 64, 0, 1]) for k in range(K)] for n in range(N)], dtype=np.float64)
    err = np.abs(y.T - Wr.astype(np.float64))
    assert np.all(err <= scale / 2 * (1 + 2.0 ** -10) + 2.0 ** -24)


def test_w4a16_constant_rows_and_padding():
    """A constant row (scale 0, codes 0: reading 1) gives y = c * sum_k x.
    K not a multiple of 64 is zero-padded at the end (Q0, pads take part in
    min/max: reading 7): the result equals the explicitly padded problem."""
    rng = np.random.default_rng(RNG_SEED + 42)
    N, K, B = 3, 128, 4
    W = np.zeros((N, K), np.float16)
    W[0, :] = 1.5
    W[1, :] = -0.25
    W[2, :] = 3.0
    x = rng.integers(-9, 10, (B, K)).astype(np.float16)
    c, m = oracle.quantize_groupwise(W, N, K, 1)
    y = oracle.w4a16_linear(c, m, N, K, x)
    sx = x.astype(np.float64).sum(axis=1)
    assert np.array_equal(y, np.outer(sx, [1.5, -0.25, 3.0]))
    K2 = 100
    W2 = (rng.standard_normal((N, K2)) * 0.1).astype(np.float16)
    x2 = rng.standard_normal((B, K2)).astype(np.float16)
    c2, m2 = oracle.quantize_groupwise(W2, N, K2, 1)
    Wp = np.zeros((N, 128), np.float16)
    Wp[:, :K2] = W2
    xp = np.zeros((B, 128), np.float16)
    xp[:, :K2] = x2
    cp, mp = oracle.quantize_groupwise(Wp, N, 128, 1)
    assert np.array_equal(c2, cp) and np.array_equal(m2, mp)
    assert np.array_equal(oracle.w4a16_linear(c2, m2, N, K2, x2), oracle.w4a16_linear(cp, mp, N, 128, xp))
