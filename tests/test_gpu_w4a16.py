"""GPU parity for NEXT-3, the W4A16 linear layer (tcgen05 GEMM with the
dequantization fused in), through the C ABI, against the CPU oracle
(oracle.w4a16_linear: fp64 matmul on the Eq 11 / D1 dequantized weights).

Tolerance: the kernel dequantizes with one fp16 rounding
RN16(c*scale + min) (HFMA2) where D1 rounds twice, RN16(RN32(.)) -- the two can
differ by one fp16 ulp on double-rounding ties -- and accumulates in fp32 on
the tensor cores.  Elementwise bar: |y - y_ref| <= 2^-10 * sum_k |x_k w_k|
+ 1e-6 (one ulp16 on every weight plus fp32 accumulation, far below the
error of a wrong code, group or index, which is O(scale * |x|) per term).
"""
import numpy as np
import pytest
import torch

import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lmo():
    from paper_conf_ipps_wurypgll25_b200 import lmo as m
    return m


def make_weights(rng, N, K):
    W = rng.standard_normal((N, K)) * 0.05
    W[:, rng.choice(K, max(1, K // 50), replace=False)] *= 8.0      # outlier input features
    W = W.astype(np.float16)
    codes, meta = oracle.quantize_groupwise(W, N, K, 1)
    return codes.reshape(N, K // 2), meta.reshape(N, K // 64, 2)


def check(lmo, N, K, batch, k_split, seed):
    rng = np.random.default_rng(seed)
    codes, meta = make_weights(rng, N, K)
    x = rng.standard_normal((batch, K)).astype(np.float16)
    ref = oracle.w4a16_linear(codes, meta, N, K, x)
    wdq = oracle.dequantize_groupwise(codes, meta, N, K, 1).reshape(N, K).astype(np.float64)
    bound = np.abs(x.astype(np.float64)) @ np.abs(wdq).T * 2.0 ** -10 + 1e-6
    y = lmo.lmo_w4a16_linear(torch.from_numpy(codes).cuda(), torch.from_numpy(meta.view(np.int32)).cuda(),
                             N, K, torch.from_numpy(x).cuda(), k_split=k_split)
    torch.cuda.synchronize()
    got = y.cpu().numpy().astype(np.float64)
    err = np.abs(got - ref)
    assert np.all(err <= bound), (err.max(), (err / bound).max())
    return got, ref


@pytest.mark.parametrize("N,K,batch,k_split", [
    (128, 64, 1, 1),          # one tile, one step
    (256, 320, 5, 1),         # ragged batch (< 16), 5 groups
    (256, 320, 5, 2),         # split-K, uneven
    (384, 640, 64, 0),        # auto split
    (128, 1024, 100, 3),      # BN = 128 instance, ragged batch
    (256, 512, 128, 4),
])
def test_w4a16_vs_oracle(lmo, N, K, batch, k_split):
    check(lmo, N, K, batch, k_split, seed=1000 + N + K + batch + k_split)


def test_w4a16_split_invariant_and_deterministic(lmo):
    """k_split = 1 is deterministic run to run; every split agrees with it
    within fp32 rounding."""
    rng = np.random.default_rng(7)
    N, K, B = 256, 1024, 64
    codes, meta = make_weights(rng, N, K)
    x = torch.from_numpy(rng.standard_normal((B, K)).astype(np.float16)).cuda()
    c, m = torch.from_numpy(codes).cuda(), torch.from_numpy(meta.view(np.int32)).cuda()
    y1 = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1).cpu()
    y1b = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1).cpu()
    assert torch.equal(y1, y1b)
    for s in (2, 4, 16):
        ys = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=s).cpu()
        assert torch.allclose(ys, y1, rtol=1e-5, atol=1e-4)


def test_w4a16_on_grid_exact(lmo):
    """On-grid integer weights and integer activations: every product and
    partial sum is an integer < 2^24, so the tensor-core result is exact."""
    rng = np.random.default_rng(11)
    N, K, B = 128, 256, 16
    W = np.zeros((N, K))
    for n in range(N):
        for g in range(K // 64):
            k = rng.integers(0, 16, 64)
            k[:2] = [0, 15]
            W[n, g * 64:(g + 1) * 64] = float(rng.integers(-4, 4)) + k
    x = rng.integers(-3, 4, (B, K)).astype(np.float16)
    codes, meta = oracle.quantize_groupwise(W.astype(np.float16), N, K, 1)
    y = lmo.lmo_w4a16_linear(torch.from_numpy(codes.reshape(N, K // 2)).cuda(),
                             torch.from_numpy(meta.reshape(N, K // 64, 2).view(np.int32)).cuda(), N, K,
                             torch.from_numpy(x).cuda(), k_split=1)
    assert np.array_equal(y.cpu().numpy().astype(np.float64), x.astype(np.float64) @ W.T)


def test_w4a16_config3_layer_sampled(lmo):
    """OPT-30B (config 3) FFN1 shape at batch 64 -- N = 4*h1 = 28672, K = h1 =
    7168 -- in the launch configuration the bench times (auto split); rows
    sampled against the oracle."""
    rng = np.random.default_rng(3)
    N, K, B = 28672, 7168, 64
    W = (rng.standard_normal((N, K), dtype=np.float32) * 0.02).astype(np.float16)
    Wt = torch.from_numpy(W).cuda()
    codes = torch.empty((N, K // 2), dtype=torch.uint8, device="cuda")
    meta = torch.empty((N, K // 64), dtype=torch.int32, device="cuda")
    lmo.lmo_quantize_groupwise(Wt, N, K, 1, codes=codes, meta=meta)
    x = rng.standard_normal((B, K)).astype(np.float16)
    y = lmo.lmo_w4a16_linear(codes, meta, N, K, torch.from_numpy(x).cuda()).cpu().numpy()
    rows = np.sort(rng.choice(N, 24, replace=False))
    ch = codes[rows].cpu().numpy()
    mh = meta[rows].cpu().numpy().view(np.uint16).reshape(len(rows), K // 64, 2)
    ref = oracle.w4a16_linear(ch, mh, len(rows), K, x)
    wdq = oracle.dequantize_groupwise(ch, mh, len(rows), K, 1).reshape(len(rows), K).astype(np.float64)
    bound = np.abs(x.astype(np.float64)) @ np.abs(wdq).T * 2.0 ** -10 + 1e-6
    assert np.all(np.abs(y[:, rows] - ref) <= bound)


def test_w4a16_argument_errors(lmo):
    c = torch.zeros((128, 32), dtype=torch.uint8, device="cuda")
    m = torch.zeros((128, 1), dtype=torch.int32, device="cuda")
    x = torch.zeros((4, 64), dtype=torch.float16, device="cuda")
    with pytest.raises(lmo.LmoError):
        lmo.lmo_w4a16_linear(c, m, 100, 64, x)                     # N % 128
    with pytest.raises(lmo.LmoError):
        lmo.lmo_w4a16_linear(c, m, 128, 60, x[:, :60].contiguous())  # K % 64
    xb = torch.zeros((129, 64), dtype=torch.float16, device="cuda")
    with pytest.raises(lmo.LmoError):
        lmo.lmo_w4a16_linear(c, m, 128, 64, xb)                    # batch > 128


@pytest.mark.parametrize("N,K,batch,k_split", [(128, 64, 3, 1), (256, 320, 5, 2), (384, 1024, 64, 0),
                                                (256, 512, 100, 3)])
def test_w4a16_packed_layout(lmo, N, K, batch, k_split):
    """lmo_w4a16_pack + lmo_w4a16_linear_packed: the packed blocks hold exactly the
    tile's codes then its meta words, and the packed GEMM is bit-identical to the
    row-major one (same arithmetic, same split) and within the oracle bound."""
    rng = np.random.default_rng(2000 + N + K + batch)
    codes, meta = make_weights(rng, N, K)
    c, m = torch.from_numpy(codes).cuda(), torch.from_numpy(meta.view(np.int32)).cuda()
    packed = lmo.lmo_w4a16_pack(c, m, N, K).cpu().numpy()
    KB = K // 64
    blk = packed.reshape(N // 128, KB, 4608)
    # code words k-interleaved (include/lmo.h): nibble k of a word moves to position
    # 4 * (k % 2) + k // 2
    words = codes.view("<u4")
    inter = np.zeros_like(words)
    for k in range(8):
        inter |= ((words >> np.uint32(4 * k)) & np.uint32(0xF)) << np.uint32(4 * (4 * (k % 2) + k // 2))
    inter = inter.view(np.uint8)
    for t in range(N // 128):
        for g in (0, KB - 1):
            assert np.array_equal(blk[t, g, :4096].reshape(128, 32), inter[t * 128:(t + 1) * 128, g * 32:(g + 1) * 32])
            assert np.array_equal(blk[t, g, 4096:].view(np.uint16).reshape(128, 2), meta[t * 128:(t + 1) * 128, g])
    x = torch.from_numpy(rng.standard_normal((batch, K)).astype(np.float16)).cuda()
    y1 = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1).cpu()
    yp = lmo.lmo_w4a16_linear_packed(torch.from_numpy(packed).cuda(), N, K, x, k_split=1).cpu()
    assert torch.equal(y1, yp)
    ys = lmo.lmo_w4a16_linear_packed(torch.from_numpy(packed).cuda(), N, K, x, k_split=k_split).cpu().numpy()
    ref = oracle.w4a16_linear(codes, meta, N, K, x.cpu().numpy())
    wdq = oracle.dequantize_groupwise(codes, meta, N, K, 1).reshape(N, K).astype(np.float64)
    bound = np.abs(x.cpu().numpy().astype(np.float64)) @ np.abs(wdq).T * 2.0 ** -10 + 1e-6
    assert np.all(np.abs(ys - ref) <= bound)


def test_w4a16_row_major_ring_repeatable(lmo):
    """The row-major path's code ring (2-D TMA refills after generic-proxy reads, DESIGN.md
    K7 root cause): at the OPT-30B FFN1 shape, 8 back-to-back runs are bit-identical to
    each other and to the packed path (same arithmetic, 1-D bulk copies)."""
    g = torch.Generator(device="cuda")
    g.manual_seed(3)
    N, K, B = 28672, 7168, 64
    W = (torch.randn(N, K, generator=g, device="cuda") * 0.02).half()
    c, m = lmo.lmo_quantize_groupwise(W, N, K, 1)
    x = torch.randn(B, K, generator=g, device="cuda").half()
    c, m = c.view(N, K // 2), m.view(N, K // 64)
    ref = lmo.lmo_w4a16_linear_packed(lmo.lmo_w4a16_pack(c, m, N, K), N, K, x, k_split=1)
    for _ in range(8):
        y = lmo.lmo_w4a16_linear(c, m, N, K, x, k_split=1)
        assert torch.equal(y, ref)


@pytest.mark.parametrize("packed", [False, True])
def test_w4a16_weight_magnitude_edges(lmo, packed):
    """Groups of every magnitude class the format allows: scale < 2^-10 (a scale/16
    operand would be an fp16 subnormal -- the odd-nibble path must see the full
    scale), all-subnormal weights, constant groups (scale 0) and weights near the
    fp16 range, in both the row-major and the packed (two-groups-per-step) GEMM.
    Bound per weight: one fp16 ulp of the weight, at least one subnormal ulp 2^-24."""
    rng = np.random.default_rng(31)
    N, K, B = 640, 512, 48
    W = rng.standard_normal((N, K))
    W[0:128] *= 1e-4                      # scale ~ 5e-5 < 2^-10
    W[128:256] *= 3e-6                    # every weight subnormal in fp16
    W[256:384] = np.repeat(rng.uniform(-2, 2, (128, K // 64)), 64, axis=1)     # scale 0 groups
    W[384:512] *= 2000.0                  # |w| up to ~1e4
    W[512:640] *= np.where(rng.random((128, K)) < 0.5, 1e-4, 0.05)              # mixed groups
    W = W.astype(np.float16)
    codes, meta = oracle.quantize_groupwise(W, N, K, 1)
    codes, meta = codes.reshape(N, K // 2), meta.reshape(N, K // 64, 2)
    x = rng.standard_normal((B, K)).astype(np.float16)
    ref = oracle.w4a16_linear(codes, meta, N, K, x)
    wdq = oracle.dequantize_groupwise(codes, meta, N, K, 1).reshape(N, K).astype(np.float64)
    ax = np.abs(x.astype(np.float64))
    bound = ax @ (np.abs(wdq).T * 2.0 ** -10 + 2.0 ** -24) + 1e-6
    c, m = torch.from_numpy(codes).cuda(), torch.from_numpy(meta.view(np.int32)).cuda()
    xt = torch.from_numpy(x).cuda()
    if packed:
        y = lmo.lmo_w4a16_linear_packed(lmo.lmo_w4a16_pack(c, m, N, K), N, K, xt, k_split=1)
    else:
        y = lmo.lmo_w4a16_linear(c, m, N, K, xt, k_split=1)
    err = np.abs(y.cpu().numpy().astype(np.float64) - ref)
    r = err / bound
    for lo in range(0, N, 128):
        print(f"rows {lo}-{lo + 127}: max err/bound {r[:, lo:lo + 128].max():.3f}")
    assert np.all(err <= bound), (r.max(), np.unravel_index(r.argmax(), r.shape))


@pytest.mark.parametrize("N,K,batch", [(640, 12800, 8), (640, 12800, 100), (384, 7168, 64), (2560, 1024, 37)])
def test_w4a16_packed_stream_k(lmo, N, K, batch):
    """The automatic split of the packed GEMM uses stream-K when the tiles do not fill the
    resident slots evenly: the tile-steps of all tiles cut into equal ranges, a range may
    end inside one tile and continue in the next (two TMEM accumulators, atomic adds).
    N=640, K=12800: 500 tile-steps over the slots -- most ranges cross a tile boundary.
    Checked against the oracle bound and against the unsplit run (fp32 rounding)."""
    rng = np.random.default_rng(3000 + N + K + batch)
    codes, meta = make_weights(rng, N, K)
    c, m = torch.from_numpy(codes).cuda(), torch.from_numpy(meta.view(np.int32)).cuda()
    packed = lmo.lmo_w4a16_pack(c, m, N, K)
    x = torch.from_numpy(rng.standard_normal((batch, K)).astype(np.float16)).cuda()
    ya = lmo.lmo_w4a16_linear_packed(packed, N, K, x, k_split=0).cpu()
    y1 = lmo.lmo_w4a16_linear_packed(packed, N, K, x, k_split=1).cpu()
    ref = oracle.w4a16_linear(codes, meta, N, K, x.cpu().numpy())
    wdq = oracle.dequantize_groupwise(codes, meta, N, K, 1).reshape(N, K).astype(np.float64)
    absdot = np.abs(x.cpu().numpy().astype(np.float64)) @ np.abs(wdq).T
    assert np.all(np.abs(ya.numpy().astype(np.float64) - ref) <= absdot * 2.0 ** -10 + 1e-6)
    # vs the unsplit run: only the fp32 summation order differs (tensor-core accumulation
    # of the whole K vs atomic adds of range partials): |dy| <= K * 2^-24 * sum|x w|
    assert np.all(np.abs(ya.numpy().astype(np.float64) - y1.numpy()) <= K * 2.0 ** -24 * absdot + 1e-6)


@pytest.mark.parametrize("N,K,B", [(21504, 7168, 64),     # c3 QKV: stream-K, BN = 64
                                   (27648, 9216, 64),     # c4 QKV: stream-K
                                   (24576, 8192, 128),    # c5 QKV: BN = 128, 2 CTAs/SM, split-K
                                   (8192, 32768, 128)])   # c5 FFN2: long K, split-K
def test_w4a16_packed_bench_shapes_sampled(lmo, N, K, B):
    """The packed GEMM at the bench's full shapes in its launch configuration (auto split:
    stream-K or split-K with the overlapped zeroing), sampled output features -- the first
    and last rows of tiles (where stream-K ranges hand a tile over) and random rows --
    against the oracle bound."""
    rng = np.random.default_rng(N + K + B)
    W = (rng.standard_normal((N, K), dtype=np.float32) * 0.02).astype(np.float16)
    Wt = torch.from_numpy(W).cuda()
    codes = torch.empty((N, K // 2), dtype=torch.uint8, device="cuda")
    meta = torch.empty((N, K // 64), dtype=torch.int32, device="cuda")
    lmo.lmo_quantize_groupwise(Wt, N, K, 1, codes=codes, meta=meta)
    del Wt
    packed = lmo.lmo_w4a16_pack(codes, meta, N, K)
    x = rng.standard_normal((B, K)).astype(np.float16)
    y = lmo.lmo_w4a16_linear_packed(packed, N, K, torch.from_numpy(x).cuda()).cpu().numpy()
    rows = np.unique(np.concatenate([[0, 127, 128, N - 128, N - 1], rng.choice(N, 19, replace=False)]))
    ch = codes[rows].cpu().numpy()
    mh = meta[rows].cpu().numpy().view(np.uint16).reshape(len(rows), K // 64, 2)
    ref = oracle.w4a16_linear(ch, mh, len(rows), K, x)
    wdq = oracle.dequantize_groupwise(ch, mh, len(rows), K, 1).reshape(len(rows), K).astype(np.float64)
    bound = np.abs(x.astype(np.float64)) @ np.abs(wdq).T * 2.0 ** -10 + 1e-6
    assert np.all(np.abs(y[:, rows] - ref) <= bound)
