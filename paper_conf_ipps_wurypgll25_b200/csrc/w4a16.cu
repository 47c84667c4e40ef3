// w4a16.cu -- NEXT-3: a linear layer over group-wise q4 weights with the
// dequantization fused into a tcgen05 (UMMA) GEMM.  sm_100a.
//
// Paper: the weights are quantized once and, every decode step, loaded and
// dequantized before the layer's matmuls ("load_weight + dequan_wgt", Eq 4
// P:228-233; Eq 11).  Here the dequantization never
// reaches HBM: the q4 codes (0.5625 B/weight) stream from HBM, are expanded to
// fp16 in shared memory by the producer warps, and the 5th-generation tensor
// cores multiply them with the activations, accumulating in TMEM.
//
//   y[b][n] = sum_k x[b][k] * W~[n][k],   W~[n][k] = RN16(c * scale + min)
//
// W [N][K] is quantized along K (lmo_quantize_groupwise with outer = N,
// n = K, inner = 1): codes [N][K/2] (low nibble = even k), meta [N][K/64]
// {min, scale} fp16 pairs.  K % 64 == 0, N % 128 == 0.
//
// CTA tile: 128 output features (UMMA M) x BN batch columns (UMMA N), K in
// 64-element steps (one quantization group):
//   (warp ids below for LMO_W4_PARTS = 2; the default, 1 thread per weight row, uses
//   dequant warps 0-3, MMA warp 4, TMA warps 5 and 6 -- measured best)
//   warp 9 (one lane)        TMA: the tile's q4 codes of step j (128 rows x 32 B,
//                            2-D tensor map) into a kCodes-deep staging ring
//   warp 10 (one lane)       TMA: the activations of step j (BN x 64 fp16, 2-D
//                            tensor map, SWIZZLE_128B, rows >= batch zero-filled)
//                            straight into the B operand stage
//   warps 0-7 (256 threads)  dequant: thread (row r, half h) expands its 32
//                            weights to fp16 and stores them with tcgen05.st
//                            into the A operand stage in TENSOR MEMORY (lane =
//                            row, 2 fp16 per column) -- the dequantized weights
//                            never touch shared memory; then the epilogue
//                            (warps 0-3: tcgen05.ld of the accumulator)
//   warp 8                   TMEM allocation; one lane issues tcgen05.mma
//                            (A from TMEM, B from smem; 4 x K=16 per step).
// Split-K (grid.y) accumulates fp32 partial tiles with red.global.add.
#include <cuda.h>

#include <algorithm>
#include <atomic>

#include "common.cuh"

namespace lmo {

namespace w4 {
constexpr int kM = 128;          // output features per CTA (UMMA M)
constexpr int kK = 64;           // K per stage (one group, one swizzle atom of fp16)
#ifndef LMO_W4_STAGES
#define LMO_W4_STAGES 4
#endif
#ifndef LMO_W4_CODES
#define LMO_W4_CODES 12
#endif
constexpr int kStages = LMO_W4_STAGES;   // A (TMEM) / B (smem) operand stages
constexpr int kCodes = LMO_W4_CODES;     // q4 code staging depth (steps in flight from HBM)
#ifndef LMO_W4_XSTAGES
#define LMO_W4_XSTAGES 4
#endif
constexpr int kX = LMO_W4_XSTAGES;       // B (activation) stages in smem: prefetched further ahead than A
#ifndef LMO_W4_CPS
#define LMO_W4_CPS 1   // (packed path: 1, 2, 4 measured equal within 2%)
#endif
constexpr int kCPS = LMO_W4_CPS;         // steps per codes TMA (box 32*kCPS B x 128 rows: full lines)
constexpr int kCodeSlots = kCodes / kCPS;
#ifndef LMO_W4_WARP_ARRIVE
#define LMO_W4_WARP_ARRIVE 0   // 1: one mbarrier arrival per producer warp (measured equal)
#endif
#ifndef LMO_W4_STREAMK
#define LMO_W4_STREAMK 1   // auto split of the two-group kernel: stream-K when tiles do not fill the slots evenly
#endif
#ifndef LMO_W4_SK_FILL
#define LMO_W4_SK_FILL 0.8   // stream-K when the split-K grid fills less than this share of the slots
#endif
#ifndef LMO_W4_NODEQ
#define LMO_W4_NODEQ 0
#endif
#ifndef LMO_W4_PARTS
#define LMO_W4_PARTS 1
#endif
constexpr int kParts = LMO_W4_PARTS;     // dequant threads per weight row (each: 64/kParts weights per step)
// MT: 128-row tiles per CTA (1 or 2).  With MT = 2 one CTA covers 256 output features:
// two accumulators and two A stages per step in TMEM share ONE activation stage, so the
// per-step synchronisation and the activation traffic are amortised over twice the weights.
template <int MT>
struct Roles {
    static constexpr int PROD = 128 * kParts * MT;     // dequant threads
    static constexpr int WMMA = PROD / 32;             // warp ids: MMA issuer, codes TMA, activation TMA
    static constexpr int WTC = WMMA + 1, WTX = WMMA + 2;
    static constexpr int THREADS = PROD + 96;
};
constexpr int kProd = Roles<1>::PROD;   // (MT = 1 names kept for the single-tile code paths)

template <int BN, int MT = 1>
struct Smem {
    static constexpr int B = BN * 128;                 // BN x 64 fp16, SWIZZLE_128B
    static constexpr int CODES = kM * 32 * MT;         // 4 KB per tile per step
    static constexpr int OFF_CODES = kX * B;
    static constexpr int PBLK = kM * 32 + kM * 4;      // packed layout: one tile-step = codes | meta (4608 B)
    static constexpr int PSTEP = PBLK * MT;
    static constexpr int CSLOT = PSTEP * kCPS;         // one codes transfer: kCPS steps
    static constexpr int OFF_BARS = OFF_CODES + kCodeSlots * CSLOT;   // (meta: registers / the packed block)
#ifndef LMO_W4_SMEM_PAD
#define LMO_W4_SMEM_PAD 0   // (experiments: extra dynamic smem bytes to limit co-resident CTAs)
#endif
    static constexpr int BYTES = OFF_BARS + 512 + 1024 /* barriers + TMEM slot; align */ + LMO_W4_SMEM_PAD;
};
static_assert((2 * kCodes + 2 * kX + 2 * kStages + 1) * 8 + 4 <= 512, "barrier area");
template <int BN, int MT = 1>
struct Tmem {
    static constexpr int ACC = BN * MT;                // accumulator columns (fp32), tile mt at mt * BN
    static constexpr int A0 = BN * MT;                 // A stages: 32 columns per tile (64 fp16 per lane)
    static constexpr int USED = BN * MT + kStages * 32 * MT;
#ifndef LMO_W4_TMEM_COLS
#define LMO_W4_TMEM_COLS 0   // (experiments: force the TMEM allocation size)
#endif
    static constexpr int COLS = LMO_W4_TMEM_COLS ? LMO_W4_TMEM_COLS
                              : USED <= 32 ? 32 : USED <= 64 ? 64 : USED <= 128 ? 128 : USED <= 256 ? 256 : 512;
    static_assert(USED <= 512, "TMEM");
};

__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(uint32_t dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}

// UMMA shared-memory descriptor: K-major, SWIZZLE_128B, 8-row groups 1024 B apart.
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4)      // start address
         | ((uint64_t)1 << 16)                       // LBO (unused for swizzled K-major)
         | ((uint64_t)(1024 >> 4) << 32)             // SBO: 8 rows x 128 B
         | ((uint64_t)1 << 46)                       // descriptor version (sm_100)
         | ((uint64_t)2 << 61);                      // SWIZZLE_128B
}

// Instruction descriptor: D f32, A/B f16, both K-major, M = 128, N = BN.
template <int BN>
__host__ __device__ constexpr uint32_t umma_idesc() {
    return (1u << 4) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(kM >> 4) << 24);
}

// 8 codes (one word, low nibble first) -> 8 fp16 weights RN16(c * scale + min), in k order.
// (1024 + c) is exact in fp16 (OR into the exponent of 1024); the high nibble of each
// byte is read in place as 1024 + 16c.  Normal groups (scale >= 2^-10): 16c is scaled by
// scale/16, exact there (HADD2 + HFMA2, the HADD2 off the FMA pipe).  TINY groups
// (scale < 2^-10, where scale/16 would lose bits as an fp16 subnormal): 1024 + 16c is
// brought back to c exactly by one HFMA2 (t/16 - 64) and meets the full scale.
// Both give RN16(c * scale + min) with one rounding.
// PK (the packed streaming layout): the word's nibbles are stored k-interleaved
// (positions 0-3 = k 0, 2, 4, 6; positions 4-7 = k 1, 3, 5, 7 -- lmo_w4a16_pack), so the
// four masks already yield k-ordered pairs and no byte permutes are needed.
template <bool TINY, bool PK = false>
__device__ __forceinline__ uint4 deq8(uint32_t w, __half2 sc, __half2 sc16, __half2 mn) {
    const __half2 k1024 = __half2half2(__ushort_as_half(0x6400));
    const uint32_t s8 = w >> 8;
    const uint32_t t0 = lop3_and_or(w, 0x000F000Fu, 0x64006400u);    // (c0, c4) + 1024
    const uint32_t t1 = lop3_and_or(w, 0x00F000F0u, 0x64006400u);    // 16 (c1, c5) + 1024
    const uint32_t t2 = lop3_and_or(s8, 0x000F000Fu, 0x64006400u);   // (c2, c6) + 1024
    const uint32_t t3 = lop3_and_or(s8, 0x00F000F0u, 0x64006400u);   // 16 (c3, c7) + 1024
    auto lo = [&](uint32_t t) { return __hsub2(*reinterpret_cast<const __half2 *>(&t), k1024); };
    auto hi = [&](uint32_t t) {
        return TINY ? __hfma2(*reinterpret_cast<const __half2 *>(&t), __half2half2(__ushort_as_half(0x2C00)),
                              __half2half2(__ushort_as_half(0xD400)))     // t/16 - 64 = c
                    : lo(t);                                            // 16c
    };
    auto f = [&](__half2 c, __half2 s) {
        const __half2 r = __hfma2(c, s, mn);
        return *reinterpret_cast<const uint32_t *>(&r);
    };
    const __half2 shi = TINY ? sc : sc16;
    const uint32_t p0 = f(lo(t0), sc), p1 = f(hi(t1), shi), p2 = f(lo(t2), sc), p3 = f(hi(t3), shi);
    if (PK) return make_uint4(p0, p1, p2, p3);
    return make_uint4(prmt(p0, p1, 0x5410u), prmt(p2, p3, 0x5410u), prmt(p0, p1, 0x7632u),
                      prmt(p2, p3, 0x7632u));
}

// scale < 2^-10 (fp16 0x1400): scale/16 is not exact in fp16
__device__ __forceinline__ bool tiny_scale(uint32_t mw) { return (mw >> 16) < 0x1400u; }


__device__ __forceinline__ void tma_2d(uint32_t dst, const void *tmap, int c0, int c1, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(dst),
        "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

// PACKED: W in the streaming layout of lmo_w4a16_pack -- per (128-row tile, group) one
// contiguous 4608-B block [128 rows x 32 B codes | 128 x 4 B meta], fetched with one 1-D
// bulk copy (full DRAM pages) instead of a 2-D TMA of 128 scattered 32-B row pieces.
template <int BN, bool PACKED, int MT>
__global__ void __launch_bounds__(Roles<MT>::THREADS, 1)
w4a16_kernel(const __grid_constant__ CUtensorMap tm_codes, const __grid_constant__ CUtensorMap tm_x,
             const uint32_t *__restrict__ meta, const uint8_t *__restrict__ packed, float *__restrict__ y, int N,
             int K, int batch, int ksplit) {
    using S = Smem<BN, MT>;
    using TM = Tmem<BN, MT>;
    constexpr int kProd = Roles<MT>::PROD, kWMMA = Roles<MT>::WMMA, kWTC = Roles<MT>::WTC, kWTX = Roles<MT>::WTX;
    static_assert(MT == 1 || (kParts == 1 && kCPS == 1), "two tiles per CTA: one dequant thread per row, kCPS 1");
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const uint32_t sbase = smem_u32(smem);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + S::OFF_BARS);
    uint64_t *c_full = bars, *c_empty = bars + kCodes;                    // codes ring
    uint64_t *x_full = bars + 2 * kCodes, *x_empty = x_full + kX;        // B stages (smem)
    uint64_t *a_full = x_empty + kX, *ab_empty = a_full + kStages;        // A stages (TMEM)
    uint64_t *done = ab_empty + kStages;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(done + 1);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int n0 = blockIdx.x * kM * MT;
    const int KB = K / kK;
    const int kb0 = (int)((long long)blockIdx.y * KB / ksplit), kb1 = (int)((long long)(blockIdx.y + 1) * KB / ksplit);
    const int nsteps = kb1 - kb0;

    if (tid == 0) {
        for (int s = 0; s < kCodes; ++s) {
            mbar_init(&c_full[s], 1);
            mbar_init(&c_empty[s], LMO_W4_WARP_ARRIVE ? kProd / 32 : kProd);
        }
        for (int s = 0; s < kX; ++s) {
            mbar_init(&x_full[s], 1);
            mbar_init(&x_empty[s], 1);
        }
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&a_full[s], LMO_W4_WARP_ARRIVE ? kProd / 32 : kProd);
            mbar_init(&ab_empty[s], 1);
        }
        mbar_init(done, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == kWMMA) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                     "n"(TM::COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    const uint32_t tmem = *tmem_slot;

    if (warp == kWTC) {
        // ------------------------------------------------------ TMA: q4 codes
        if (lane == 0) {
            for (int q = 0; q * kCPS < nsteps; ++q) {
                const int cs = q % kCodeSlots;
                if (q >= kCodeSlots) mbar_wait(&c_empty[cs], ((q / kCodeSlots) - 1) & 1);
                if constexpr (PACKED) {
                    const int ns = min(kCPS, nsteps - q * kCPS);
                    mbar_arrive_expect_tx(&c_full[cs], ns * S::PSTEP);
#pragma unroll
                    for (int mt = 0; mt < MT; ++mt) {
                        const uint8_t *src = packed + ((int64_t)(blockIdx.x * MT + mt) * KB + kb0 + q * kCPS) * S::PBLK;
                        bulk_g2s(smem + S::OFF_CODES + cs * S::CSLOT + mt * S::PBLK * kCPS, src, ns * S::PBLK,
                                 &c_full[cs], policy_evict_first());
                    }
                } else {
                    mbar_arrive_expect_tx(&c_full[cs], S::CODES * kCPS);
                    tma_2d(sbase + S::OFF_CODES + cs * S::CSLOT, &tm_codes, (kb0 + q * kCPS) * 32, n0, &c_full[cs]);
                }
            }
        }
    } else if (warp == kWTX) {
        // ------------------------------------------------------ TMA: activations
        if (lane == 0) {
            for (int j = 0; j < nsteps; ++j) {
                const int xs = j % kX;
                if (j >= kX) mbar_wait(&x_empty[xs], ((j / kX) - 1) & 1);
                mbar_arrive_expect_tx(&x_full[xs], S::B);
                tma_2d(sbase + xs * S::B, &tm_x, (kb0 + j) * kK, 0, &x_full[xs]);
            }
        }
    } else if (warp < kWMMA) {
        // ------------------------------------------------------ dequant -> TMEM
        constexpr int WPT = kK / kParts;                        // weights per thread per step
        // thread -> (tile mt, row r = TMEM lane, part h); MT = 2 implies kParts = 1 (h = 0)
        const int r = tid & (kM - 1), mt = MT == 1 ? 0 : tid >> 7, h = MT == 1 ? tid >> 7 : 0;
        const int tr = mt * kM + r;                              // row within the CTA's rows
        const uint32_t *mrow = meta + (int64_t)(n0 + tr) * (K / kK);
        // row-major path: the group meta word of step j is a plain read-only global load issued
        // two steps ahead into registers (L2-resident: 1/16 of the code bytes).
        uint32_t m_next = 0, m_next2 = 0;
        auto meta_load = [&](int j) -> uint32_t {
            return (!PACKED && j < nsteps) ? __ldg(mrow + kb0 + j) : 0u;
        };
        if (!PACKED) {
            m_next = meta_load(0);
            m_next2 = meta_load(1);
        }
        const uint32_t lane_base = tmem + ((uint32_t)((warp & 3) * 32) << 16) + TM::A0 + mt * 32 + h * (WPT / 2);
        // software pipeline: the dequant of step j overlaps the TMEM store of step j-1
        // (tcgen05.wait::st of j-1 only after step j's arithmetic); two register buffers
        auto produce = [&](int j, uint4 (&v)[WPT / 8]) {
            const int q = j / kCPS, cs = q % kCodeSlots, sub = j - q * kCPS;
            if (sub == 0) mbar_wait(&c_full[cs], (q / kCodeSlots) & 1);
            uint32_t cw[WPT / 8], mw;
            const uint32_t caddr = PACKED ? sbase + S::OFF_CODES + cs * S::CSLOT + (mt * kCPS + sub) * S::PBLK + r * 32 + h * (WPT / 2)
                                          : sbase + S::OFF_CODES + cs * S::CSLOT + tr * (32 * kCPS) + sub * 32 + h * (WPT / 2);
            if constexpr (WPT == 64) {
                asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
                             : "=r"(cw[0]), "=r"(cw[1]), "=r"(cw[2]), "=r"(cw[3]) : "r"(caddr));
                asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
                             : "=r"(cw[4]), "=r"(cw[5]), "=r"(cw[6]), "=r"(cw[7]) : "r"(caddr + 16));
            } else if constexpr (WPT == 32)
                asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
                             : "=r"(cw[0]), "=r"(cw[1]), "=r"(cw[2]), "=r"(cw[3]) : "r"(caddr));
            else
                asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];\n" : "=r"(cw[0]), "=r"(cw[1]) : "r"(caddr));
            if constexpr (PACKED) {
                asm volatile("ld.shared.u32 %0, [%1];\n"
                             : "=r"(mw) : "r"(sbase + S::OFF_CODES + cs * S::CSLOT + (mt * kCPS + sub) * S::PBLK + kM * 32 + r * 4));
            } else {
                mw = m_next;
                m_next = m_next2;
                m_next2 = meta_load(j + 2);
            }
            const bool last_sub = sub == kCPS - 1 || j == nsteps - 1;
            // WAR across proxies: the codes (and meta) were read with generic-proxy loads;
            // the slot is refilled by an async-proxy TMA write once every consumer has
            // arrived.  The mbarrier release/acquire pair does not order a generic read
            // before an async-proxy write, and the hardware does issue the arrive while
            // the shared loads are still in flight: without this fence, rings of 4 or 8
            // stages corrupted rows nondeterministically (scripts/w4_check.py; DESIGN.md
            // K7 "root cause").
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            if (!LMO_W4_WARP_ARRIVE && last_sub) mbar_arrive(&c_empty[cs]);
            const __half2 mn2 = __half2half2(__ushort_as_half((unsigned short)(mw & 0xFFFFu)));
            const __half2 sc2 = __half2half2(__ushort_as_half((unsigned short)(mw >> 16)));
            const __half2 sc16 = __hmul2(sc2, __half2half2(__ushort_as_half(0x2C00)));   // * 1/16
#if LMO_W4_NODEQ   // (experiment: pipeline / MMA bound without the dequant arithmetic)
#pragma unroll
            for (int i = 0; i < WPT / 8; ++i) v[i] = make_uint4(cw[i], cw[i] ^ mw, cw[i], cw[i]);
#else
            if (tiny_scale(mw)) {
#pragma unroll
                for (int i = 0; i < WPT / 8; ++i) v[i] = deq8<true, PACKED>(cw[i], sc2, sc16, mn2);
            } else {
#pragma unroll
                for (int i = 0; i < WPT / 8; ++i) v[i] = deq8<false, PACKED>(cw[i], sc2, sc16, mn2);
            }
#endif
            if (LMO_W4_WARP_ARRIVE && last_sub) {   // codes consumed (results in registers): one arrive per warp
                __syncwarp();
                if (lane == 0) mbar_arrive(&c_empty[cs]);
            }
        };
        auto store = [&](int j, const uint4 (&v)[WPT / 8]) {
            const int st = j % kStages;
            if (j >= kStages) mbar_wait(&ab_empty[st], ((j / kStages) - 1) & 1);
            // order the TMEM store after the MMA that last read this A stage (WAR across the
            // mbarrier): without it a store can overtake the wait under load
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            if constexpr (WPT == 64)
                asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                             "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};\n" ::"r"(lane_base + st * 32 * MT),
                             "r"(v[0].x), "r"(v[0].y), "r"(v[0].z), "r"(v[0].w), "r"(v[1].x), "r"(v[1].y), "r"(v[1].z),
                             "r"(v[1].w), "r"(v[2 % (WPT / 8)].x), "r"(v[2 % (WPT / 8)].y), "r"(v[2 % (WPT / 8)].z),
                             "r"(v[2 % (WPT / 8)].w), "r"(v[3 % (WPT / 8)].x), "r"(v[3 % (WPT / 8)].y),
                             "r"(v[3 % (WPT / 8)].z), "r"(v[3 % (WPT / 8)].w), "r"(v[4 % (WPT / 8)].x),
                             "r"(v[4 % (WPT / 8)].y), "r"(v[4 % (WPT / 8)].z), "r"(v[4 % (WPT / 8)].w),
                             "r"(v[5 % (WPT / 8)].x), "r"(v[5 % (WPT / 8)].y), "r"(v[5 % (WPT / 8)].z),
                             "r"(v[5 % (WPT / 8)].w), "r"(v[6 % (WPT / 8)].x), "r"(v[6 % (WPT / 8)].y),
                             "r"(v[6 % (WPT / 8)].z), "r"(v[6 % (WPT / 8)].w), "r"(v[7 % (WPT / 8)].x),
                             "r"(v[7 % (WPT / 8)].y), "r"(v[7 % (WPT / 8)].z), "r"(v[7 % (WPT / 8)].w)
                             : "memory");
            else if constexpr (WPT == 32)
                asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};\n" ::"r"(
                                 lane_base + st * 32 * MT),
                             "r"(v[0].x), "r"(v[0].y), "r"(v[0].z), "r"(v[0].w), "r"(v[1].x), "r"(v[1].y), "r"(v[1].z),
                             "r"(v[1].w), "r"(v[WPT / 8 - 2].x), "r"(v[WPT / 8 - 2].y), "r"(v[WPT / 8 - 2].z),
                             "r"(v[WPT / 8 - 2].w), "r"(v[WPT / 8 - 1].x), "r"(v[WPT / 8 - 1].y), "r"(v[WPT / 8 - 1].z),
                             "r"(v[WPT / 8 - 1].w)
                             : "memory");
            else
                asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};\n" ::"r"(lane_base + st * 32 * MT),
                             "r"(v[0].x), "r"(v[0].y), "r"(v[0].z), "r"(v[0].w), "r"(v[WPT / 8 - 1].x),
                             "r"(v[WPT / 8 - 1].y), "r"(v[WPT / 8 - 1].z), "r"(v[WPT / 8 - 1].w)
                             : "memory");
        };
        auto publish = [&](int j) {
            asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
            asm volatile("tcgen05.fence::before_thread_sync;\n");
            if (LMO_W4_WARP_ARRIVE) {
                __syncwarp();
                if (lane == 0) mbar_arrive(&a_full[j % kStages]);
            } else {
                mbar_arrive(&a_full[j % kStages]);
            }
        };
        uint4 va[WPT / 8], vb[WPT / 8];
        if (nsteps > 0) {
            produce(0, va);
            store(0, va);
        }
        for (int j = 1; j < nsteps; j += 2) {
            produce(j, vb);
            publish(j - 1);
            store(j, vb);
            if (j + 1 < nsteps) {
                produce(j + 1, va);
                publish(j);
                store(j + 1, va);
            }
        }
        if (nsteps > 0) publish(nsteps - 1);
        cp_wait<0>();
    } else {
        // ------------------------------------------------------ MMA issuer (warp 8)
        constexpr uint32_t idesc = umma_idesc<BN>();
        for (int j = 0; j < nsteps; ++j) {
            const int st = j % kStages, xs = j % kX;
            mbar_wait(&x_full[xs], (j / kX) & 1);
            mbar_wait(&a_full[st], (j / kStages) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
            if (lane == 0) {
                const uint32_t b0 = sbase + xs * S::B;
#pragma unroll
                for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                for (int k = 0; k < kK / 16; ++k) {
                    const uint32_t ta = tmem + TM::A0 + (st * MT + mt) * 32 + k * 8;
                    const uint64_t db = umma_desc(b0 + k * 32);
                    const uint32_t acc = (j > 0 || k > 0) ? 1u : 0u;
                    asm volatile(
                        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem + mt * BN),
                        "r"(ta), "l"(db), "r"(idesc), "r"(acc));
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(&ab_empty[st]))
                             : "memory");
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(&x_empty[xs]))
                             : "memory");
            }
            __syncwarp();
        }
        if (lane == 0)
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                             smem_u32(done))
                         : "memory");
        __syncwarp();
    }

    // ---------------------------------------------------------------- epilogue
    // (split-K: the zeroed y comes from the preceding programmatic-primary zero kernel)
    if (ksplit > 1) asm volatile("griddepcontrol.wait;\n" ::: "memory");
    if (warp < 4 * MT) {
        const int emt = warp >> 2;                               // tile of this epilogue warp
        const int row = emt * kM + (warp & 3) * 32 + lane;       // TMEM lane = output feature
        if (nsteps > 0) {
            mbar_wait(done, 0);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
        }
#pragma unroll
        for (int c0 = 0; c0 < BN; c0 += 32) {
            uint32_t v[32];
            const uint32_t taddr = tmem + ((uint32_t)((warp & 3) * 32) << 16) + emt * BN + c0;
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
                : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                  "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                  "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                  "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                  "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                : "r"(taddr));
            asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
            if (nsteps == 0) continue;
#pragma unroll
            for (int i = 0; i < 32; ++i) {
                const int b = c0 + i;
                if (b < batch) {
                    float *dst = y + (int64_t)b * N + n0 + row;
                    const float val = __uint_as_float(v[i]);
#ifdef LMO_W4_NOATOMIC   // (timing experiment: split-K partials stored, not reduced -- wrong results)
                    *dst = val;
#else
                    if (ksplit > 1) atomicAdd(dst, val);
                    else *dst = val;
#endif
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    if (warp == kWMMA) {
        asm volatile("tcgen05.fence::after_thread_sync;\n");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "n"(TM::COLS));
    }
}

// ---------------------------------------------------------------------------
// Packed layout, TWO quantization groups (K = 128) per pipeline step: every
// per-step synchronisation (code-slot wait, empty arrive + proxy fence, TMEM
// store wait / fence / full arrive, the MMA issuer's waits and commits) is paid
// once per 128 weights per thread instead of once per 64 -- the synchronisation,
// not HBM or the tensor pipe, bounded the one-group kernel (K7).
// One 1-D bulk copy brings the two consecutive 4608-B packed blocks of a step;
// the activations arrive as two SW128 atoms; A = 2 x 32 TMEM columns per stage.
#ifdef LMO_W4_EXP_TL   // (experiment: per-step clock timeline of CTA (0, 0) of the two-group kernel)
__device__ unsigned int g_w4_tl[16][512];
#define W4TL(slot, j) do { if (blockIdx.x == 0 && blockIdx.y == 0 && (j) < 512) g_w4_tl[slot][j] = (unsigned)clock(); } while (0)
#else
#define W4TL(slot, j) do { } while (0)
#endif
namespace g2 {
#ifndef LMO_W4_G2_C
#define LMO_W4_G2_C 6
#endif
#ifndef LMO_W4_G2_XS
#define LMO_W4_G2_XS 3
#endif
constexpr int kC = LMO_W4_G2_C;       // code slots (2 groups each)
constexpr int kXS = LMO_W4_G2_XS;     // activation stages
#ifndef LMO_W4_G2_AS
#define LMO_W4_G2_AS 2
#endif
constexpr int kAS = LMO_W4_G2_AS;      // A stages in TMEM (64 columns each)
// Per-instance pipeline shape.  BN = 128 (batch 65-128): 2 activation stages and 3 code slots
// (93 KB of shared memory) and no stream-K accumulator (256 TMEM columns), so TWO CTAs fit
// per SM -- measured c5 layer 255 -> 208 us; with the 3-stage / 6-slot shape and a second
// accumulator (512 columns) only one fits.  BN = 64: the 3 / 6 shape with stream-K.
template <int BN>
struct Cfg {
    static constexpr int XS = BN == 128 ? 2 : kXS;     // activation stages
    static constexpr int C = BN == 128 ? 3 : kC;       // code slots
    static constexpr bool SK = BN != 128 && LMO_W4_STREAMK;   // stream-K (second accumulator)
};
template <int BN>
struct Smem {
    static constexpr int XS = Cfg<BN>::XS, C = Cfg<BN>::C;
    static constexpr int B = 2 * BN * 128;             // two SW128 atoms: BN x 128 fp16
    static constexpr int PBLK = kM * 32 + kM * 4;      // one packed tile-group block
    static constexpr int CSLOT = 2 * PBLK;
    static constexpr int OFF_CODES = XS * B;
    static constexpr int OFF_BARS = OFF_CODES + C * CSLOT;
    static constexpr int BYTES = OFF_BARS + 512 + 1024;
};
template <int BN>
struct Tmem {
    static constexpr int A0 = BN;
    static constexpr int ACC1 = BN + kAS * 64;          // stream-K: second tile's accumulator
    static constexpr int USED = ACC1 + (Cfg<BN>::SK ? BN : 0);
    static constexpr int COLS = USED <= 128 ? 128 : USED <= 256 ? 256 : 512;
};
static_assert((2 * kC + 2 * kXS + 2 * kAS + 1) * 8 + 4 <= 512, "barrier area");
}  // namespace g2

// y = 0 for the split / stream-K GEMMs' atomic epilogues; triggers its programmatic dependent
// (the GEMM) at once so the GEMM's main loop overlaps it
__global__ void w4_zero_kernel(float4 *__restrict__ p, int64_t n4) {
    asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory");
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
}

// DW = dequant warps: 4 (thread = weight row, both groups) or 8 (warp w: rows 32 (w % 4) ..,
// group w / 4 -- two warps per SMSP, half the dependent chain per thread; one mbarrier
// arrival per warp).
template <int BN, int DW>
__global__ void __launch_bounds__(DW * 32 + 96, 1)
w4a16_g2_kernel(const __grid_constant__ CUtensorMap tm_x, const uint8_t *__restrict__ packed,
                float *__restrict__ y, int N, int K, int batch, int ksplit, int sk) {
    using S = g2::Smem<BN>;
    using TM = g2::Tmem<BN>;
    constexpr int kWMMA = DW, kWTC = DW + 1, kWTX = DW + 2;
    constexpr int kArrive = DW == 8 ? DW : 128;          // arrivals per step on c_empty / a_full
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const uint32_t sbase = smem_u32(smem);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + S::OFF_BARS);
    uint64_t *c_full = bars, *c_empty = bars + S::C;
    uint64_t *x_full = bars + 2 * S::C, *x_empty = x_full + S::XS;
    uint64_t *a_full = x_empty + S::XS, *ab_empty = a_full + g2::kAS;
    uint64_t *done = ab_empty + g2::kAS;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(done + 1);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int KB = K / kK, KS = KB / 2;                 // groups, steps
    // Work of this CTA: steps [0, nsteps) = k-steps g0 .. of tile tile0, then (stream-K) from
    // step jsw on k-steps 0 .. of tile tile0 + 1.  Split-K (sk = 0): tile blockIdx.x, the
    // blockIdx.y-th of ksplit k ranges.  Stream-K (sk = 1, gridDim.y = 1, gridDim.x >= tiles):
    // the tile-steps of all tiles, linearised tile-major, cut into gridDim.x equal ranges --
    // equal work per resident slot, each range within at most two tiles.
    int tile0, g0, nsteps, jsw;
    if (sk) {
        const long long T = (long long)(N / kM) * KS;
        const long long a0 = (long long)blockIdx.x * T / gridDim.x, a1 = (long long)(blockIdx.x + 1) * T / gridDim.x;
        tile0 = (int)(a0 / KS);
        g0 = (int)(a0 - (long long)tile0 * KS);
        nsteps = (int)(a1 - a0);
        jsw = min(nsteps, KS - g0);
    } else {
        const int s0 = (int)((long long)blockIdx.y * KS / ksplit), s1 = (int)((long long)(blockIdx.y + 1) * KS / ksplit);
        tile0 = blockIdx.x;
        g0 = s0;
        nsteps = s1 - s0;
        jsw = nsteps;
    }
    auto tile_of = [&](int j) { return j < jsw ? tile0 : tile0 + 1; };
    auto kstep_of = [&](int j) { return j < jsw ? g0 + j : j - jsw; };

    if (tid == 0) {
        for (int s = 0; s < S::C; ++s) {
            mbar_init(&c_full[s], 1);
            mbar_init(&c_empty[s], kArrive);
        }
        for (int s = 0; s < S::XS; ++s) {
            mbar_init(&x_full[s], 1);
            mbar_init(&x_empty[s], 1);
        }
        for (int s = 0; s < g2::kAS; ++s) {
            mbar_init(&a_full[s], kArrive);
            mbar_init(&ab_empty[s], 1);
        }
        mbar_init(done, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == kWMMA) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                     "n"(TM::COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    const uint32_t tmem = *tmem_slot;

    if (warp == kWTC) {
        if (lane == 0) {   // codes: one bulk copy of a step's two consecutive packed blocks
            for (int q = 0; q < nsteps; ++q) {
                const int cs = q % S::C;
                if (q >= S::C) mbar_wait(&c_empty[cs], ((q / S::C) - 1) & 1);
                W4TL(0, q);
                mbar_arrive_expect_tx(&c_full[cs], S::CSLOT);
                const uint8_t *src = packed + ((int64_t)tile_of(q) * KB + 2 * kstep_of(q)) * S::PBLK;
                bulk_g2s(smem + S::OFF_CODES + cs * S::CSLOT, src, S::CSLOT, &c_full[cs], policy_evict_first());
            }
        }
    } else if (warp == kWTX) {
        if (lane == 0) {   // activations: two 64-wide SW128 boxes per step
            for (int j = 0; j < nsteps; ++j) {
                const int xs = j % S::XS;
                if (j >= S::XS) mbar_wait(&x_empty[xs], ((j / S::XS) - 1) & 1);
                W4TL(1, j);
#ifdef LMO_W4_EXP_NOX   // (timing experiment: activations loaded only for the first kXS steps -- wrong results)
                if (j >= S::XS) { mbar_arrive(&x_full[xs]); continue; }
#endif
                mbar_arrive_expect_tx(&x_full[xs], S::B);
                const int kg = 2 * kstep_of(j);
                tma_2d(sbase + xs * S::B, &tm_x, kg * kK, 0, &x_full[xs]);
                tma_2d(sbase + xs * S::B + BN * 128, &tm_x, (kg + 1) * kK, 0, &x_full[xs]);
            }
        }
    } else if (warp < kWMMA) {
        // dequant -> TMEM: thread = weight row r = TMEM lane (DW = 8: group gi = warp / 4 only)
        const int r = tid & (kM - 1);
        const uint32_t lane_base = tmem + ((uint32_t)((warp & 3) * 32) << 16) + TM::A0;
        constexpr int G0 = 0, G1 = DW == 8 ? 1 : 2;           // groups of this thread: [g_lo, g_lo + G1)
        const int g_lo = DW == 8 ? (warp >> 2) : 0;
        for (int j = 0; j < nsteps; ++j) {
            const int cs = j % S::C, st = j % g2::kAS;
            if (tid == 0) W4TL(2, j);
            mbar_wait(&c_full[cs], (j / S::C) & 1);
            if (tid == 0) W4TL(3, j);
            if (j >= g2::kAS) mbar_wait(&ab_empty[st], ((j / g2::kAS) - 1) & 1);
            if (tid == 0) W4TL(4, j);
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
#pragma unroll
            for (int gg = G0; gg < G1; ++gg) {
                const int gi = g_lo + gg;
                const uint32_t blk = sbase + S::OFF_CODES + cs * S::CSLOT + gi * S::PBLK;
                uint32_t cw[8], mw;
                asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
                             : "=r"(cw[0]), "=r"(cw[1]), "=r"(cw[2]), "=r"(cw[3]) : "r"(blk + r * 32));
                asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
                             : "=r"(cw[4]), "=r"(cw[5]), "=r"(cw[6]), "=r"(cw[7]) : "r"(blk + r * 32 + 16));
                asm volatile("ld.shared.u32 %0, [%1];\n" : "=r"(mw) : "r"(blk + kM * 32 + r * 4));
#ifdef LMO_W4_EXP_TL
                if (tid == 0 && blockIdx.x == 0 && blockIdx.y == 0 && j < 512) g_w4_tl[8 + 3 * gg][j] = (unsigned)clock() + (mw & cw[7] & 0);
#endif
                const __half2 mn2 = __half2half2(__ushort_as_half((unsigned short)(mw & 0xFFFFu)));
                const __half2 sc2 = __half2half2(__ushort_as_half((unsigned short)(mw >> 16)));
                const __half2 sc16 = __hmul2(sc2, __half2half2(__ushort_as_half(0x2C00)));   // * 1/16
                uint4 v[8];
#if LMO_W4_NODEQ   // (experiment: the pipeline without the dequant arithmetic)
                if (true) {
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[i] = make_uint4(cw[i], cw[i] ^ mw, cw[i], cw[i]);
                } else
#endif
                if (tiny_scale(mw)) {
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[i] = deq8<true, true>(cw[i], sc2, sc16, mn2);
                } else {
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[i] = deq8<false, true>(cw[i], sc2, sc16, mn2);
                }
                asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                             "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};\n" ::"r"(
                                 lane_base + st * 64 + gi * 32),
                             "r"(v[0].x), "r"(v[0].y), "r"(v[0].z), "r"(v[0].w), "r"(v[1].x), "r"(v[1].y), "r"(v[1].z),
                             "r"(v[1].w), "r"(v[2].x), "r"(v[2].y), "r"(v[2].z), "r"(v[2].w), "r"(v[3].x), "r"(v[3].y),
                             "r"(v[3].z), "r"(v[3].w), "r"(v[4].x), "r"(v[4].y), "r"(v[4].z), "r"(v[4].w), "r"(v[5].x),
                             "r"(v[5].y), "r"(v[5].z), "r"(v[5].w), "r"(v[6].x), "r"(v[6].y), "r"(v[6].z), "r"(v[6].w),
                             "r"(v[7].x), "r"(v[7].y), "r"(v[7].z), "r"(v[7].w)
                             : "memory");
#ifdef LMO_W4_EXP_TL
                if (tid == 0 && blockIdx.x == 0 && blockIdx.y == 0 && j < 512) g_w4_tl[9 + 3 * gg][j] = (unsigned)clock() + (v[7].w & v[0].x & 0);
#endif
            }
            // the slot's generic-proxy reads before its async-proxy refill (see w4a16_kernel)
#ifndef LMO_W4_EXP_NOFENCE
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
#endif
            if (DW == 8) {
                __syncwarp();
                if (lane == 0) mbar_arrive(&c_empty[cs]);
            } else {
                mbar_arrive(&c_empty[cs]);
            }
            if (tid == 0) W4TL(14, j);
#ifndef LMO_W4_EXP_NOWAITST
            asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
#endif
            if (tid == 0) W4TL(15, j);
            asm volatile("tcgen05.fence::before_thread_sync;\n");
            if (DW == 8) {
                __syncwarp();
                if (lane == 0) mbar_arrive(&a_full[st]);
            } else {
                mbar_arrive(&a_full[st]);
            }
            if (tid == 0) W4TL(5, j);
        }
    } else {
        // MMA issuer: 2 groups x 4 x (K = 16) per step
        constexpr uint32_t idesc = umma_idesc<BN>();
        for (int j = 0; j < nsteps; ++j) {
            const int st = j % g2::kAS, xs = j % S::XS;
            mbar_wait(&x_full[xs], (j / S::XS) & 1);
            if (lane == 0) W4TL(6, j);
            mbar_wait(&a_full[st], (j / g2::kAS) & 1);
            if (lane == 0) W4TL(7, j);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
            if (lane == 0) {
                const uint32_t b0 = sbase + xs * S::B;
                const uint32_t dacc = tmem + (j < jsw ? 0u : (uint32_t)TM::ACC1);   // this step's tile accumulator
                const bool first = j == 0 || j == jsw;
#ifdef LMO_W4_EXP_MMA1   // (timing experiment: one MMA per step -- wrong results)
                for (int gi = 0; gi < 1; ++gi)
                    for (int k = 0; k < 1; ++k) {
#else
#pragma unroll
                for (int gi = 0; gi < 2; ++gi)
#pragma unroll
                    for (int k = 0; k < kK / 16; ++k) {
#endif
                        const uint32_t ta = tmem + TM::A0 + st * 64 + gi * 32 + k * 8;
                        const uint64_t db = umma_desc(b0 + gi * BN * 128 + k * 32);
                        const uint32_t acc = (!first || gi > 0 || k > 0) ? 1u : 0u;
                        asm volatile(
                            "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                            "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(dacc),
                            "r"(ta), "l"(db), "r"(idesc), "r"(acc));
                    }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(&ab_empty[st]))
                             : "memory");
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(&x_empty[xs]))
                             : "memory");
            }
            __syncwarp();
        }
        if (lane == 0)
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                             smem_u32(done))
                         : "memory");
        __syncwarp();
    }

    // epilogue: warps 0-3 read the accumulator(s) (TMEM lane = output feature); stream-K
    // ranges and split-K partials are added atomically (y zeroed on the stream first)
    if (warp < 4) {
        const int row = (warp & 3) * 32 + lane;
        if (nsteps > 0) {
            mbar_wait(done, 0);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
        }
        // the zeroed y: written by the preceding (programmatic-primary) zero kernel
        if (ksplit > 1 || sk) asm volatile("griddepcontrol.wait;\n" ::: "memory");
        for (int seg = 0; seg < 2; ++seg) {
            if (seg == 0 ? jsw == 0 : nsteps <= jsw) continue;
            const int n0 = (tile0 + seg) * kM;
            const uint32_t aoff = seg == 0 ? 0u : (uint32_t)TM::ACC1;
#pragma unroll
            for (int c0 = 0; c0 < BN; c0 += 32) {
                uint32_t v[32];
                const uint32_t taddr = tmem + ((uint32_t)((warp & 3) * 32) << 16) + aoff + c0;
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                    "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                      "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                      "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                      "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                      "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                    : "r"(taddr));
                asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                    const int b = c0 + i;
                    if (b < batch) {
                        float *dst = y + (int64_t)b * N + n0 + row;
                        const float val = __uint_as_float(v[i]);
                        if (ksplit > 1 || sk) atomicAdd(dst, val);
                        else *dst = val;
                    }
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    if (warp == kWMMA) {
        asm volatile("tcgen05.fence::after_thread_sync;\n");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "n"(TM::COLS));
    }
}

}  // namespace w4

#ifndef LMO_W4_G2
#define LMO_W4_G2 1   // packed weights, K % 128 == 0: two quantization groups per pipeline step
#endif
#ifndef LMO_W4_G2_DW
#define LMO_W4_G2_DW 4   // dequant warps of the two-group kernel (4 or 8: measured equal within noise)
#endif
#ifndef LMO_W4_MT
#define LMO_W4_MT 1   // 2: two 128-row tiles per CTA when N % 256 == 0 (measured slower: 213 vs 190 us)
#endif
static int w4a16_mt(int N) { return (LMO_W4_MT == 2 && N % (2 * w4::kM) == 0) ? 2 : 1; }

#ifdef LMO_W4_EXP_TL
extern "C" int lmo_exp_w4_timeline(unsigned int *host) {
    return (int)cudaMemcpyFromSymbol(host, w4::g_w4_tl, sizeof(w4::g_w4_tl));
}
#endif

// Resident CTAs per SM of a W4A16 instance: shared memory (with the per-block
// reservation), tensor memory columns (512 per SM) and threads.  (The runtime's
// occupancy query reported 1 for the two-group instance where ncu and the split-K
// timings show 2: 7168 x 28672 ran at 67 instead of 41 us with the auto split.)
static int w4a16_resident_ctas(int smem_bytes, int tmem_cols, int threads) {
    int dev = 0, smem_sm = 0, reserved = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev);
    int occ = smem_sm / (smem_bytes + reserved);
    occ = std::min(occ, 512 / tmem_cols);
    occ = std::min(occ, 2048 / threads);
    return std::max(occ, 1);
}

int w4a16_auto_split(int N, int K, int ctas_per_sm) {
    // the most K splits that still fit ONE wave of resident CTAs (ctas_per_sm: the occupancy
    // of the instance being launched); measured on the OPT-30B layer GEMMs: more CTAs than
    // one wave (or a half-empty last wave) costs more than the split-K atomics save
    const int MT = w4a16_mt(N);
    const int tiles = N / (w4::kM * MT), KB = K / w4::kK;
    const int slots = device_sm_count() * (ctas_per_sm > 0 ? ctas_per_sm : 1);
    int s = slots / tiles;
    if (s > 8) s = 8;
    if (s > KB / 4) s = KB / 4;
    return s < 1 ? 1 : s;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_tiled() {
    static EncodeTiledFn fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(p);
    }
    return fn;
}

// One code word (k 0..7 at nibble positions 0..7) -> the packed layout's k-interleaved
// word: positions 0-3 hold k 0, 2, 4, 6 and positions 4-7 hold k 1, 3, 5, 7.
__device__ __forceinline__ uint32_t interleave_nibbles(uint32_t w) {
    uint32_t o = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) o |= ((w >> (4 * k)) & 0xFu) << (4 * ((k & 1) * 4 + (k >> 1)));
    return o;
}

// Pack W (codes [N][K/2], meta [N][K/64]) into the streaming layout: block (tile, g) of
// 4608 B = [128 rows x 32 B codes (k-interleaved words) | 128 x 4 B meta] at
// ((tile * K/64) + g) * 4608.
__global__ void w4a16_pack_kernel(const uint8_t *__restrict__ codes, const uint32_t *__restrict__ meta,
                                  uint8_t *__restrict__ packed, int N, int K) {
    const int KB = K / w4::kK;
    const int64_t nchunks = (int64_t)(N / w4::kM) * KB * (w4::kM * 2 + w4::kM / 4);   // 16-B chunks
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < nchunks; c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t blk = c / (w4::kM * 2 + w4::kM / 4);
        const int w = (int)(c - blk * (w4::kM * 2 + w4::kM / 4));
        const int tile = (int)(blk / KB), g = (int)(blk - (int64_t)tile * KB);
        uint4 v;
        if (w < w4::kM * 2) {              // codes: row w/2, half w%2
            const int r = w >> 1, hh = w & 1;
            v = *reinterpret_cast<const uint4 *>(codes + (int64_t)(tile * w4::kM + r) * (K / 2) + g * 32 + hh * 16);
            v = make_uint4(interleave_nibbles(v.x), interleave_nibbles(v.y), interleave_nibbles(v.z),
                           interleave_nibbles(v.w));
        } else {                           // meta: rows 4(w-256) .. +3
            const int r0 = (w - w4::kM * 2) * 4;
            const uint32_t *mp = meta + (int64_t)(tile * w4::kM + r0) * KB + g;
            v = make_uint4(mp[0], mp[KB], mp[2 * KB], mp[3 * KB]);
        }
        *reinterpret_cast<uint4 *>(packed + blk * 4608 + (int64_t)w * 16) = v;
    }
}

cudaError_t launch_w4a16_pack(const uint8_t *codes, const void *meta, uint8_t *packed, int N, int K, cudaStream_t st) {
    const int64_t nchunks = (int64_t)(N / w4::kM) * (K / w4::kK) * (w4::kM * 2 + w4::kM / 4);
    const int grid = (int)std::min<int64_t>((nchunks + 255) / 256, (int64_t)device_sm_count() * 16);
    w4a16_pack_kernel<<<grid, 256, 0, st>>>(codes, static_cast<const uint32_t *>(meta), packed, N, K);
    const cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) note_launch();
    return e;
}

// codes/meta (row-major, 2-D TMA path) or packed (streaming layout, 1-D bulk path)
cudaError_t launch_w4a16(const uint8_t *codes, const void *meta, const uint8_t *packed, const void *x, float *y,
                         int N, int K, int batch, int ksplit, cudaStream_t st) {
    EncodeTiledFn enc = encode_tiled();
    if (!enc) return cudaErrorNotSupported;
    const int BN = batch <= 64 ? 64 : 128;   // UMMA N = the batch rounded up (an N = 32 instance for
                                             // batch <= 32 measured equal on c2: 76.4 vs 74-76 us/layer)
    CUtensorMap tc, tx;
    {   // x [batch][K] fp16, box 64 x BN rows, SWIZZLE_128B (rows >= batch are zero-filled)
        const cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)batch};
        const cuuint64_t strides[1] = {(cuuint64_t)K * 2};
        const cuuint32_t box[2] = {(cuuint32_t)w4::kK, (cuuint32_t)BN}, es[2] = {1, 1};
        if (enc(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void *>(x), dims, strides, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return cudaErrorInvalidValue;
    }
    if (packed) {
        tc = tx;                                                   // (unused by the packed path)
    } else {   // codes [N][K/2] u8, box 32*kCPS B x 128 rows (out-of-range columns zero-filled)
        const cuuint64_t dims[2] = {(cuuint64_t)K / 2, (cuuint64_t)N};
        const cuuint64_t strides[1] = {(cuuint64_t)K / 2};
        const cuuint32_t box[2] = {32 * w4::kCPS, (cuuint32_t)(w4::kM * w4a16_mt(N))}, es[2] = {1, 1};
        if (enc(&tc, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<uint8_t *>(codes), dims, strides, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return cudaErrorInvalidValue;
    }
    const int MT = w4a16_mt(N);
    const uint32_t *m = static_cast<const uint32_t *>(meta);
    if (packed && LMO_W4_G2 && MT == 1 && K % (2 * w4::kK) == 0) {   // two groups per pipeline step
        cudaError_t pre = cudaSuccess;
        auto go2 = [&](auto kern, int smem_bytes, int tmem_cols, bool sk_ok) {
            // attributes and the resident-CTA count once per (device, instance): the host path of a
            // small GEMM is launch-bound (c2 layer: ~50 us of host enqueue for 4 GEMMs)
            static std::atomic<int> occ_cache[64][2];
            int dev = 0;
            cudaGetDevice(&dev);
            if (dev < 0 || dev >= 64) dev = 0;
            const int bi = BN == 64 ? 0 : 1;
            int occ = occ_cache[dev][bi].load(std::memory_order_acquire);
            if (occ == 0) {
                cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
                cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared);
                occ = w4a16_resident_ctas(smem_bytes, tmem_cols, LMO_W4_G2_DW * 32 + 96);
                occ_cache[dev][bi].store(occ, std::memory_order_release);
            }
            int sk_ctas = 0;
            if (ksplit <= 0) {
                ksplit = w4a16_auto_split(N, K, occ);
                // Stream-K when the tiles do not fill the resident slots evenly (e.g. 168 or 224
                // tiles on 296 slots: 2-tile SMs beside 1-tile SMs): the linearised tile-steps cut
                // into whole waves of equal ranges (K7)
                // (measured: only a poorly filled split pays for stream-K's second epilogue --
                // c3 QKV 168 tiles 44.2 -> 37.6 us, c5 QKV 192 tiles 84.0 -> 70.7, but c3 FFN2
                // 56 tiles x 5 splits 40.9 -> 43.2)
                const int64_t tiles = N / w4::kM, slots = (int64_t)device_sm_count() * occ;
                const int64_t T = tiles * (K / (2 * w4::kK));
                const int64_t used = tiles * ksplit, waves_used = (used + slots - 1) / slots;
                const double fill = (double)used / (double)(slots * waves_used);
                if (sk_ok && fill < LMO_W4_SK_FILL) {
                    const int64_t waves = (tiles + slots - 1) / slots;
                    sk_ctas = (int)std::min<int64_t>(slots * waves, T);
                    ksplit = 1;
                }
            }
            if (ksplit > K / (2 * w4::kK)) ksplit = K / (2 * w4::kK);
            const bool zero = ksplit > 1 || sk_ctas > 0;
            if (zero) {
                // y is zeroed by a PDL-triggering kernel and the GEMM is launched as its programmatic
                // dependent: the GEMM's main loop overlaps the zeroing (x and the codes are ready --
                // their producer finished before the zero kernel started) and only its epilogue
                // atomics wait (griddepcontrol.wait) for the zeros
                const int64_t n4 = (int64_t)batch * N / 4;
                w4::w4_zero_kernel<<<device_sm_count(), 256, 0, st>>>(reinterpret_cast<float4 *>(y), n4);
                pre = cudaGetLastError();
                if (pre != cudaSuccess) return;
                note_launch();
            }
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = sk_ctas > 0 ? dim3(sk_ctas, 1) : dim3(N / w4::kM, ksplit);
            cfg.blockDim = dim3(LMO_W4_G2_DW * 32 + 96);
            cfg.dynamicSmemBytes = smem_bytes;
            cfg.stream = st;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            attr[0].val.programmaticStreamSerializationAllowed = (zero && pdl_enabled()) ? 1 : 0;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            pre = cudaLaunchKernelEx(&cfg, kern, tx, packed, y, (int)N, (int)K, (int)batch, sk_ctas > 0 ? 1 : ksplit,
                                     sk_ctas > 0 ? 1 : 0);
        };
        if (BN == 64)
            go2(w4::w4a16_g2_kernel<64, LMO_W4_G2_DW>, w4::g2::Smem<64>::BYTES, w4::g2::Tmem<64>::COLS, w4::g2::Cfg<64>::SK);
        else
            go2(w4::w4a16_g2_kernel<128, LMO_W4_G2_DW>, w4::g2::Smem<128>::BYTES, w4::g2::Tmem<128>::COLS,
                w4::g2::Cfg<128>::SK);
        if (pre != cudaSuccess) return pre;
        const cudaError_t e = cudaGetLastError();
        if (e == cudaSuccess) note_launch();
        return e;
    }
    cudaError_t pre = cudaSuccess;
    auto go = [&](auto kern, int sm, int threads) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared);
        if (ksplit <= 0) {   // auto: one wave of the resident CTAs of THIS instance
            int occ = 0;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, threads, sm);
            ksplit = w4a16_auto_split(N, K, occ);
        }
        if (ksplit > K / w4::kK) ksplit = K / w4::kK;
        if (ksplit > 1) {   // zeroing overlapped with the GEMM (as in the two-group path)
            w4::w4_zero_kernel<<<device_sm_count(), 256, 0, st>>>(reinterpret_cast<float4 *>(y), (int64_t)batch * N / 4);
            pre = cudaGetLastError();
            if (pre != cudaSuccess) return;
            note_launch();
        }
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(N / (w4::kM * MT), ksplit);
        cfg.blockDim = dim3(threads);
        cfg.dynamicSmemBytes = sm;
        cfg.stream = st;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = (ksplit > 1 && pdl_enabled()) ? 1 : 0;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        pre = cudaLaunchKernelEx(&cfg, kern, tc, tx, m, packed, y, (int)N, (int)K, (int)batch, ksplit);
    };
    constexpr int T1 = w4::Roles<1>::THREADS, T2 = w4::Roles<2>::THREADS;
    if (MT == 2) {
        if (BN == 64) {
            if (packed) go(w4::w4a16_kernel<64, true, 2>, w4::Smem<64, 2>::BYTES, T2);
            else go(w4::w4a16_kernel<64, false, 2>, w4::Smem<64, 2>::BYTES, T2);
        } else {
            if (packed) go(w4::w4a16_kernel<128, true, 2>, w4::Smem<128, 2>::BYTES, T2);
            else go(w4::w4a16_kernel<128, false, 2>, w4::Smem<128, 2>::BYTES, T2);
        }
    } else if (BN == 64) {
        if (packed) go(w4::w4a16_kernel<64, true, 1>, w4::Smem<64>::BYTES, T1);
        else go(w4::w4a16_kernel<64, false, 1>, w4::Smem<64>::BYTES, T1);
    } else {
        if (packed) go(w4::w4a16_kernel<128, true, 1>, w4::Smem<128>::BYTES, T1);
        else go(w4::w4a16_kernel<128, false, 1>, w4::Smem<128>::BYTES, T1);
    }
    if (pre != cudaSuccess) return pre;
    const cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) note_launch();
    return e;
}

}  // namespace lmo
