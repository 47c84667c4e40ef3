// common.cuh -- sm_100a device helpers shared by the liblmo kernels.
// (Product code.  Shares nothing with oracle/.)
#pragma once

#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "lmo.h"

namespace lmo {

constexpr int kGroup = 64;   // quantization group (elements)
constexpr int kQMax = 15;    // 2^b - 1, b = 4

// ------------------------------------------------------------ launch stats
void note_launch();                         // lmo_abi.cu
int device_sm_count();                      // cached per device
bool pdl_enabled();                         // programmatic dependent launch on/off

// ------------------------------------------------------- quantization math
// One rounding chain, identical in every kernel that quantizes (K1, K2):
//   range = RN32(mx - mn); scale = RU16(RU32(range / 15)) == RU16(range/15);
//   inv = scale == 0 ? 0 : RN32(1/scale);
//   code = min(15, rint_even(RN32(RN32(x - mn) * inv))).
// Unsigned 32-bit division by a runtime-invariant divisor d >= 1 (Granlund-Montgomery
// round-up multiplier): q = (mulhi(m, n) + n) >> l, exact for every n < 2^32.
struct FastDiv {
    uint32_t d, m, l;
    __host__ __device__ FastDiv() : d(1), m(0), l(0) {}
    __host__ explicit FastDiv(uint32_t div) : d(div) {
        l = 0;
        while ((1ull << l) < div) ++l;
        m = (uint32_t)((((1ull << l) - div) << 32) / div + 1);
    }
    __device__ __forceinline__ uint32_t div(uint32_t n) const {
        return (uint32_t)(((uint64_t)__umulhi(m, n) + n) >> l);
    }
};

struct GroupParams {
    float mn;       // canonical (+0 for a zero min)
    float inv;
    __half mn_h;
    __half scale_h;
};

__device__ __forceinline__ GroupParams group_params(float mn, float mx) {
    GroupParams p;
    p.mn = __fadd_rn(mn, 0.0f);                         // -0 -> +0
    const float range = __fsub_rn(__fadd_rn(mx, 0.0f), p.mn);
    // scale = RU16(RU32(range/15)) = RU16(range/15) (two upward roundings compose):
    // the least fp16 h with 15*h >= range.  Start from RU16 of an approximate
    // quotient (off by at most one fp16 step) and correct with exact tests --
    // 15*h has <= 15 significant bits, so the fp32 product and compare are exact.
    unsigned short hb = __half_as_ushort(__float2half_ru(__fmul_rn(range, 1.0f / 15.0f)));
    const float hf = __half2float(__ushort_as_half(hb));
    const float hp = __half2float(__ushort_as_half((unsigned short)(hb - 1)));
    if (__fmul_rn(hf, 15.0f) < range) hb += 1;
    else if (hb != 0 && __fmul_rn(hp, 15.0f) >= range) hb -= 1;
    p.scale_h = __ushort_as_half(hb);
    const float s = __half2float(p.scale_h);
    p.inv = (s == 0.0f) ? 0.0f : __frcp_rn(s);
    p.mn_h = __float2half_rn(p.mn);                     // exact: mn is an fp16 value
    return p;
}

__device__ __forceinline__ uint32_t quant_code(float x, const GroupParams &p) {
    float d = __fsub_rn(x, p.mn);
    float t = __fmul_rn(d, p.inv);
    // rint half-even for 0 <= t < 2^22: add 1.5*2^23, read the low mantissa bits
    float r = __fadd_rn(t, 12582912.0f);
    uint32_t c = __float_as_uint(r) - 0x4B400000u;
    return c > 15u ? 15u : c;
}

__device__ __forceinline__ uint32_t meta_word(const GroupParams &p) {
    return (uint32_t)__half_as_ushort(p.mn_h) | ((uint32_t)__half_as_ushort(p.scale_h) << 16);
}

// min / max of 8 fp16 values held as 4 half2 (exact: packed fp16 min/max), as floats
__device__ __forceinline__ void minmax8(const uint4 xv, float &mn, float &mx) {
    const __half2 *h = reinterpret_cast<const __half2 *>(&xv);
    __half2 lo = __hmin2(__hmin2(h[0], h[1]), __hmin2(h[2], h[3]));
    __half2 hi = __hmax2(__hmax2(h[0], h[1]), __hmax2(h[2], h[3]));
    mn = fminf(__low2float(lo), __high2float(lo));
    mx = fmaxf(__low2float(hi), __high2float(hi));
}

// 8 codes of one uint4 (8 fp16) packed into a 32-bit word, low nibble first.
// rint: t + 1.5*2^23 leaves the bit pattern 0x4B400000 + c.  Instead of masking
// each code, accumulate bits_k << 4k over k and subtract the constant
// sum(0x4B400000 << 4k) mod 2^32 once (one LEA/IMAD per element).
// The clamp min(15, .) is provably inactive here: x - mn <= range (RN32 is
// monotone), scale >= range/15 and inv = RN32(1/scale), so t <= 15(1+2^-24)^2
// < 15.5 and rint(t) <= 15 -- bit-identical to quant_code() / the oracle.
__device__ __forceinline__ uint32_t codes8(const uint4 xv, const GroupParams &p) {
    const __half2 *h = reinterpret_cast<const __half2 *>(&xv);
    constexpr uint32_t kMagicSum = 0x4B400000u * 0x11111111u;   // sum_k 0x4B400000 << 4k
    uint32_t acc = 0u - kMagicSum;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const float2 f = __half22float2(h[k]);
        const float t0 = __fmul_rn(__fsub_rn(f.x, p.mn), p.inv);
        const float t1 = __fmul_rn(__fsub_rn(f.y, p.mn), p.inv);
        acc += __float_as_uint(__fadd_rn(t0, 12582912.0f)) << (8 * k);
        acc += __float_as_uint(__fadd_rn(t1, 12582912.0f)) << (8 * k + 4);
    }
    return acc;
}

// Quantize one 64-group held by 8 consecutive lanes (lane8 = lane & 7), each
// holding 8 consecutive fp16 elements (16 B).  Returns this lane's 4 code
// bytes (elements 8*lane8 .. 8*lane8+7) and, via `meta`, the group meta word.
__device__ __forceinline__ uint32_t quantize_group_lane8(const uint4 xv, uint32_t &meta) {
    float mn, mx;
    minmax8(xv, mn, mx);
#pragma unroll
    for (int off = 1; off < 8; off <<= 1) {
        mn = fminf(mn, __shfl_xor_sync(0xffffffffu, mn, off));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    }
    const GroupParams p = group_params(mn, mx);
    meta = meta_word(p);
    return codes8(xv, p);
}

// Same, 4 lanes per group (lane4 = lane & 3), each holding 16 consecutive
// elements as two uint4; returns the lane's 8 code bytes.
__device__ __forceinline__ uint2 quantize_group_lane4(const uint4 xa, const uint4 xb, uint32_t &meta) {
    float mn, mx, mn2, mx2;
    minmax8(xa, mn, mx);
    minmax8(xb, mn2, mx2);
    mn = fminf(mn, mn2);
    mx = fmaxf(mx, mx2);
#pragma unroll
    for (int off = 1; off < 4; off <<= 1) {
        mn = fminf(mn, __shfl_xor_sync(0xffffffffu, mn, off));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    }
    const GroupParams p = group_params(mn, mx);
    meta = meta_word(p);
    return make_uint2(codes8(xa, p), codes8(xb, p));
}

// ------------------------------------------------- KV cache row layout (lmo.h)
// Token slot rows of `row` bytes: K codes (d/2) | K meta (d/64 words) | V area (d/2) |
// V meta.  The V codes of a token PAIR (2p, 2p+1) are interleaved in 16-bit chunks of
// 4 dims -- [A c | B c] per 32-bit word -- and the pair's 2 * d/2 bytes fill the V areas
// of rows 2p (chunks 0 .. d/8-1) and 2p+1 (the rest): one 32-bit word is the MMA
// operand "(token A, token B) x 4 dims" without any byte shuffling.
// Store chunk c (codes of dims 4c .. 4c+3 of token `tok`) given the base of row tok & ~1.
__device__ __forceinline__ void store_v_chunk(uint8_t *pair_row0, int d, int c, int tok, uint32_t v16) {
    const int rb = d / 2, row = 2 * (rb + (d / 64) * 4), cpr = rb / 4;   // chunks per row
    uint8_t *p = pair_row0 + (c / cpr) * row + rb + (d / 64) * 4 + 4 * (c % cpr) + 2 * (tok & 1);
    *reinterpret_cast<uint16_t *>(p) = (uint16_t)v16;
}

// ------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t addr = smem_u32(bar);
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "LAB_WAIT:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@P1 bra DONE;\n"
        "bra LAB_WAIT;\n"
        "DONE:\n"
        "}\n" ::"r"(addr),
        "r"(parity)
        : "memory");
}

// 1-D bulk async copy global -> shared (TMA engine, SASS UBLKCP), completion
// counted on an mbarrier.  size and both addresses must be 16-B aligned.
__device__ __forceinline__ void bulk_g2s(void *smem_dst, const void *gmem_src, uint32_t bytes,
                                         uint64_t *bar, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint "
        "[%0], [%1], %2, [%3], %4;\n" ::"r"(smem_u32(smem_dst)),
        "l"(gmem_src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}

// L2 prefetch of a global span (bulk, no completion tracking).  16-B aligned/sized.
__device__ __forceinline__ void bulk_prefetch_l2(const void *gmem_src, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;\n" ::"l"(gmem_src), "r"(bytes) : "memory");
}

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(pol));
    return pol;
}

// D(16x8, f32) += A(16x16, f16, row) * B(16x8, f16, col)   [HMMA]
__device__ __forceinline__ void mma_16816(float (&c)[4], uint32_t a0, uint32_t a1, uint32_t a2,
                                          uint32_t a3, uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, "
        "{%8,%9}, {%0,%1,%2,%3};\n"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

__device__ __forceinline__ uint32_t lop3_and_or(uint32_t x, uint32_t mask, uint32_t orv) {
    uint32_t r;
    asm("lop3.b32 %0, %1, %2, %3, 0xEA;\n" : "=r"(r) : "r"(x), "r"(mask), "r"(orv));  // (x&m)|o
    return r;
}

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;\n" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

__device__ __forceinline__ uint32_t hsub2_u32(uint32_t a, uint32_t b) {
    __half2 r = __hsub2(*reinterpret_cast<__half2 *>(&a), *reinterpret_cast<__half2 *>(&b));
    return *reinterpret_cast<uint32_t *>(&r);
}

__device__ __forceinline__ uint32_t pack_half2(float lo, float hi) {
    __half2 h = __floats2half2_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&h);
}

}  // namespace lmo
