// decode_attn.cu -- K3+K4: decode-step attention over the q4 KV cache with the
// dequantization fused in, plus the in-kernel split combine.  sm_100a.
//
// Paper: attention score QK^T/sqrt(d_k) then softmax over the KV cache
// that "is only decompressed" each token (Eq 6); the paper's
// fastest setting is exactly GPU attention over a 4-bit KV cache (P:105,
// P:132).  Design:
//
//  * Persistent grid, warp = unit of work.  The 16-token blocks of all
//    (sequence, kv-head) pairs form one global list; it is cut into V equal
//    contiguous ranges, one per resident warp ("stream-K"), so every warp
//    streams the same number of bytes whatever the batch / length mix.
//    A pair cut by a range boundary yields partial results (m, l, acc) that
//    the LAST arriving warp of that pair merges (flash-decoding combine,
//    A4) -- no second launch.  num_splits=k>0 instead cuts each pair into k
//    fixed parts.
//  * Each warp owns a private kStages-deep ring in shared memory filled by
//    1-D TMA bulk copies (cp.async.bulk, SASS UBLKCP) with mbarrier
//    completion: K codes, K meta, V codes, V meta of one 16-token block per
//    stage.  No CTA-wide barrier in the main loop.
//  * Dequantization is folded algebraically:
//      q.k_j = sum_g [ scale_jg * (sum_{i in g} q_i c_ji) + min_jg * Qs_g ]
//      o     = (sum_j p_j min_jg) + sum_j (p_j scale_jg) c_j
//    so the tensor cores only ever see EXACT 4-bit codes (converted to fp16
//    by the LOP3 magic-number trick) against fp16 q (K side) or fp16
//    p*scale (V side), accumulating in fp32 (mma.sync m16n8k16, HMMA).
//  * GQA: the query heads sharing a kv head are the MMA's head dimension, so
//    a KV tile is read once for all of them (8 q heads per kv head cost the
//    same HMMA count as 1).
#include "common.cuh"

namespace lmo {

constexpr int kBlk = 16;      // tokens per warp-block (MMA k extent)
constexpr int kWarps = 4;     // warps per CTA
constexpr int kStages = 4;    // per-warp TMA ring depth
constexpr int kMaxBatchSmem = 1024;  // per-sequence-length mode: prefix array in smem

template <int D>
struct Geo {
    static constexpr int NG = D / 64;              // quantization groups per row
    static constexpr int KC = kBlk * D / 2;        // code bytes per block (K or V)
    static constexpr int KM = kBlk * NG * 4;       // meta bytes per block (K or V)
    static constexpr int STAGE = 2 * (KC + KM);    // bytes per stage
    static constexpr int REC = D + 4;              // partial record floats per head
};

struct AttnArgs {
    const uint8_t *kc, *vc;
    const uint32_t *km, *vm;
    int B, Hkv, cap;
    const __half *q;
    int Hq, G;
    int len;                  // uniform length (lens == nullptr)
    const int32_t *lens;      // per-sequence lengths or nullptr
    float scale_log2;         // softmax_scale * log2(e)
    int num_splits;           // 0 = stream-K
    void *out;
    int out_f16;
    int *counters;            // [B*Hkv]
    float *partials;          // [slots][G][REC]
};

// ---------------------------------------------------------------- work map
struct WorkMap {
    const int *prefix;   // smem, B+1 (per-seq mode) or nullptr (uniform)
    int B, Hkv, nbu;     // nbu: blocks per pair in uniform mode
    int64_t N;           // total blocks
    int64_t V;           // virtual warps
    int W;               // physical warps in grid
    int k;               // num_splits (0 = stream-K)

    __device__ __forceinline__ int64_t seq_start(int b) const {
        return prefix ? (int64_t)prefix[b] : (int64_t)b * Hkv * nbu;
    }
    __device__ __forceinline__ int seq_nb(int b) const {
        return prefix ? (prefix[b + 1] - prefix[b]) / Hkv : nbu;
    }
    // global block x -> (b, kvh, blk, nb)
    __device__ __forceinline__ void decode(int64_t x, int &b, int &kvh, int &blk, int &nb) const {
        if (!prefix) {
            const int64_t pair = x / nbu;
            blk = (int)(x - pair * nbu);
            b = (int)(pair / Hkv);
            kvh = (int)(pair - (int64_t)b * Hkv);
            nb = nbu;
        } else {
            int lo = 0, hi = B;  // largest b with prefix[b] <= x  (prefix[B] = N > x)
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (prefix[mid] <= x) lo = mid; else hi = mid;
            }
            b = lo;
            nb = seq_nb(b);
            const int r = (int)(x - prefix[b]);
            kvh = r / nb;
            blk = r - kvh * nb;
        }
    }
    __device__ __forceinline__ int64_t pair_start(int b, int kvh) const {
        return seq_start(b) + (int64_t)kvh * seq_nb(b);
    }
    // start of virtual warp v's range
    __device__ __forceinline__ int64_t R(int64_t v) const {
        if (k == 0) return v * N / V;
        const int64_t p = v / k;
        if (p >= (int64_t)B * Hkv) return N;
        const int j = (int)(v - p * k);
        const int b = (int)(p / Hkv), kvh = (int)(p - (int64_t)b * Hkv);
        const int nb = seq_nb(b);
        return pair_start(b, kvh) + (int64_t)j * nb / k;
    }
    // virtual warp whose range contains block x
    __device__ __forceinline__ int64_t vwarp_of(int64_t x) const {
        if (k == 0) return ((x + 1) * V + N - 1) / N - 1;
        int b, kvh, blk, nb;
        decode(x, b, kvh, blk, nb);
        int j = (int)(((int64_t)(blk + 1) * k + nb - 1) / nb) - 1;
        if (j > k - 1) j = k - 1;
        return ((int64_t)b * Hkv + kvh) * k + j;
    }
    __device__ __forceinline__ int64_t slot_of(int64_t v, int64_t pstart) const {
        return k == 0 ? 2 * v + (R(v) < pstart ? 1 : 0) : v;
    }
};

struct Cursor {
    int64_t x, xend, v;
    int b, kvh, blk, nb;
    bool done;

    __device__ __forceinline__ void enter(const WorkMap &wm, int64_t v0) {
        v = v0;
        while (v < wm.V) {
            x = wm.R(v);
            xend = wm.R(v + 1);
            if (x < xend) {
                wm.decode(x, b, kvh, blk, nb);
                done = false;
                return;
            }
            v += wm.W;
        }
        done = true;
    }
    __device__ __forceinline__ void advance(const WorkMap &wm) {
        ++x;
        ++blk;
        if (x >= xend) {
            enter(wm, v + wm.W);
        } else if (blk >= nb) {
            wm.decode(x, b, kvh, blk, nb);
        }
    }
};

// ------------------------------------------------------------ fragments
__device__ __forceinline__ int tok_perm(int n) { return n ^ ((n >> 1) & 1); }  // 0,1,3,2,4,5,7,6

// K codes word -> 4 half2 of exact codes: (nib0,nib4) (nib1,nib5) (nib2,nib6) (nib3,nib7)
__device__ __forceinline__ void unpack_k(uint32_t w, uint32_t (&u)[4]) {
    const uint32_t s = w >> 8;
    u[0] = hsub2_u32(lop3_and_or(w, 0x000F000Fu, 0x64006400u), 0x64006400u);
    u[1] = hsub2_u32(lop3_and_or(w, 0x00F000F0u, 0x54005400u), 0x54005400u);
    u[2] = hsub2_u32(lop3_and_or(s, 0x000F000Fu, 0x64006400u), 0x64006400u);
    u[3] = hsub2_u32(lop3_and_or(s, 0x00F000F0u, 0x54005400u), 0x54005400u);
}

// V code words of two tokens (same dims) -> 8 half2 (tokA nib p, tokB nib p), p = 0..7
__device__ __forceinline__ void unpack_v(uint32_t wa, uint32_t wb, uint32_t (&j)[8]) {
    const uint32_t lo = prmt(wa, wb, 0x5410u);
    const uint32_t hi = prmt(wa, wb, 0x7632u);
    const uint32_t lo8 = lo >> 8, hi8 = hi >> 8;
    j[0] = hsub2_u32(lop3_and_or(lo, 0x000F000Fu, 0x64006400u), 0x64006400u);
    j[1] = hsub2_u32(lop3_and_or(lo, 0x00F000F0u, 0x54005400u), 0x54005400u);
    j[2] = hsub2_u32(lop3_and_or(lo8, 0x000F000Fu, 0x64006400u), 0x64006400u);
    j[3] = hsub2_u32(lop3_and_or(lo8, 0x00F000F0u, 0x54005400u), 0x54005400u);
    j[4] = hsub2_u32(lop3_and_or(hi, 0x000F000Fu, 0x64006400u), 0x64006400u);
    j[5] = hsub2_u32(lop3_and_or(hi, 0x00F000F0u, 0x54005400u), 0x54005400u);
    j[6] = hsub2_u32(lop3_and_or(hi8, 0x000F000Fu, 0x64006400u), 0x64006400u);
    j[7] = hsub2_u32(lop3_and_or(hi8, 0x00F000F0u, 0x54005400u), 0x54005400u);
}

__device__ __forceinline__ float2 meta_f2(uint32_t mw) {
    const __half2 h = *reinterpret_cast<const __half2 *>(&mw);
    return __half22float2(h);   // .x = min, .y = scale
}

__device__ __forceinline__ float warp_max4(float v) {  // over the 4 t-lanes of a g
    v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 1));
    return fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 2));
}
__device__ __forceinline__ float warp_sum4(float v) {
    v += __shfl_xor_sync(0xffffffffu, v, 1);
    return v + __shfl_xor_sync(0xffffffffu, v, 2);
}

template <int D>
__device__ __forceinline__ void store_row8(const AttnArgs &a, int64_t row, int dim0, const float *v) {
    // 8 consecutive dims of output row `row` (= b*Hq + h)
    if (a.out_f16) {
        uint4 pk;
        pk.x = pack_half2(v[0], v[1]);
        pk.y = pack_half2(v[2], v[3]);
        pk.z = pack_half2(v[4], v[5]);
        pk.w = pack_half2(v[6], v[7]);
        *reinterpret_cast<uint4 *>(static_cast<__half *>(a.out) + row * D + dim0) = pk;
    } else {
        float *o = static_cast<float *>(a.out) + row * D + dim0;
        reinterpret_cast<float4 *>(o)[0] = make_float4(v[0], v[1], v[2], v[3]);
        reinterpret_cast<float4 *>(o)[1] = make_float4(v[4], v[5], v[6], v[7]);
    }
}

// -------------------------------------------------------------- the kernel
template <int D>
__global__ void __launch_bounds__(kWarps * 32, 4) decode_attn_q4_kernel(const AttnArgs a) {
    using GG = Geo<D>;
    constexpr int NG = GG::NG;
    extern __shared__ __align__(128) uint8_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);                 // [kWarps][kStages]
    uint8_t *ring = smem + 128;                                           // [kWarps][kStages][STAGE]
    int *prefix = reinterpret_cast<int *>(ring + kWarps * kStages * GG::STAGE);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;

    // ---- work map (every CTA computes the same one)
    WorkMap wm;
    wm.B = a.B;
    wm.Hkv = a.Hkv;
    wm.k = a.num_splits;
    wm.W = gridDim.x * kWarps;
    if (a.lens) {
        if (warp == 0) {   // exclusive scan of Hkv*ceil(L_b/16) over b, lane-chunked
            const int per = (a.B + 31) / 32;
            const int b0 = min(a.B, lane * per), b1 = min(a.B, b0 + per);
            int s = 0;
            for (int b = b0; b < b1; ++b) {
                const int L = min(a.lens[b], a.cap);
                s += L > 0 ? a.Hkv * ((L + kBlk - 1) / kBlk) : 0;
            }
            int incl = s;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const int y = __shfl_up_sync(0xffffffffu, incl, off);
                if (lane >= off) incl += y;
            }
            int run = incl - s;
            for (int b = b0; b < b1; ++b) {
                prefix[b] = run;
                const int L = min(a.lens[b], a.cap);
                run += L > 0 ? a.Hkv * ((L + kBlk - 1) / kBlk) : 0;
            }
            if (lane == 31) prefix[a.B] = incl;
        }
        __syncthreads();
        wm.prefix = prefix;
        wm.nbu = 0;
        wm.N = prefix[a.B];
    } else {
        wm.prefix = nullptr;
        wm.nbu = (a.len + kBlk - 1) / kBlk;
        wm.N = (int64_t)a.B * a.Hkv * wm.nbu;
    }
    if (wm.k == 0) wm.V = wm.N < wm.W ? wm.N : wm.W;
    else wm.V = (int64_t)a.B * a.Hkv * wm.k;

    const int gw = blockIdx.x * kWarps + warp;

    // ---- zero rows of empty sequences (per-sequence mode only)
    if (a.lens) {
        for (int b = gw; b < a.B; b += wm.W) {
            if (a.lens[b] > 0) continue;
            for (int i = lane; i < a.Hq * D; i += 32) {
                const int64_t off = (int64_t)b * a.Hq * D + i;
                if (a.out_f16) static_cast<__half *>(a.out)[off] = __float2half_rn(0.f);
                else static_cast<float *>(a.out)[off] = 0.f;
            }
        }
    }

    uint64_t *wbar = bars + warp * kStages;
    uint8_t *wring = ring + warp * kStages * GG::STAGE;
    if (lane == 0) {
        for (int s = 0; s < kStages; ++s) mbar_init(&wbar[s], 1);
        fence_mbar_init();
    }
    __syncwarp();

    __shared__ Cursor pcs[kWarps];   // producer cursors (lane 0 only)
    Cursor cc;
    cc.enter(wm, gw);
    if (cc.done) return;
    Cursor &pc = pcs[warp];
    if (lane == 0) pc = cc;
    const uint64_t pol = policy_evict_first();

    auto issue = [&](const Cursor &c, int slot) {
        const int64_t tok0 = ((int64_t)c.b * a.Hkv + c.kvh) * a.cap + (int64_t)c.blk * kBlk;
        uint8_t *dst = wring + slot * GG::STAGE;
        mbar_arrive_expect_tx(&wbar[slot], GG::STAGE);
        bulk_g2s(dst, a.kc + tok0 * (D / 2), GG::KC, &wbar[slot], pol);
        bulk_g2s(dst + GG::KC, a.km + tok0 * NG, GG::KM, &wbar[slot], pol);
        bulk_g2s(dst + GG::KC + GG::KM, a.vc + tok0 * (D / 2), GG::KC, &wbar[slot], pol);
        bulk_g2s(dst + 2 * GG::KC + GG::KM, a.vm + tok0 * NG, GG::KM, &wbar[slot], pol);
    };

    if (lane == 0) {
        for (int s = 0; s < kStages && !pc.done; ++s) {
            issue(pc, s);
            pc.advance(wm);
        }
    }
    __syncwarp();

    const float NEG_INF = -INFINITY;
    const uint32_t ZERO = 0u;
    uint32_t it = 0;            // blocks consumed by this warp
    int qb = -1, qkvh = -1;     // pair whose q is loaded
    uint32_t qa[NG][4][2];      // q A-fragments
    float qs[NG];               // per-group sums of q (head g)
    const bool head_ok = g < a.G;

    while (!cc.done) {
        // ------------------------------------------------ segment start
        const int b = cc.b, kvh = cc.kvh, blk0 = cc.blk, nb = cc.nb;
        const int64_t vseg = cc.v;
        const int64_t pstart = cc.x - blk0;
        const int64_t seg_n = min((int64_t)(nb - blk0), cc.xend - cc.x);
        const bool full = (blk0 == 0) && (seg_n == nb);
        const int L = a.lens ? min(a.lens[b], a.cap) : a.len;

        if (b != qb || kvh != qkvh) {
            qb = b;
            qkvh = kvh;
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
                uint4 q0 = make_uint4(0, 0, 0, 0), q1 = q0;
                if (head_ok) {
                    const __half *qp = a.q + (((int64_t)b * a.Hq + kvh * a.G + g) * D + grp * 64 + 16 * t);
                    q0 = *reinterpret_cast<const uint4 *>(qp);
                    q1 = *reinterpret_cast<const uint4 *>(qp + 8);
                }
                const __half *h0 = reinterpret_cast<const __half *>(&q0);
                const __half *h1 = reinterpret_cast<const __half *>(&q1);
                __half q16[16];
                float sum = 0.f;
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    q16[i] = h0[i];
                    q16[8 + i] = h1[i];
                    sum += __half2float(h0[i]) + __half2float(h1[i]);
                }
                qs[grp] = warp_sum4(sum);
#pragma unroll
                for (int kbl = 0; kbl < 4; ++kbl) {
#pragma unroll
                    for (int r = 0; r < 2; ++r) {
                        const int idx = 2 * kbl + r;
                        const int i0 = 8 * (idx >> 2) + (idx & 3);
                        __half2 pr = __halves2half2(q16[i0], q16[i0 + 4]);
                        qa[grp][kbl][r] = *reinterpret_cast<uint32_t *>(&pr);
                    }
                }
            }
        }

        float m_run = head_ok ? NEG_INF : 0.f;
        float l_run = 0.f;
        float pm[NG];
        float acc[NG * 4][4];
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) pm[grp] = 0.f;
#pragma unroll
        for (int i = 0; i < NG * 4; ++i) acc[i][0] = acc[i][1] = acc[i][2] = acc[i][3] = 0.f;

        for (int64_t jb = 0; jb < seg_n; ++jb) {
            const int slot = it % kStages;
            mbar_wait(&wbar[slot], (it / kStages) & 1);
            const uint8_t *sKc = wring + slot * GG::STAGE;
            const uint8_t *sKm = sKc + GG::KC;
            const uint8_t *sVc = sKm + GG::KM;
            const uint8_t *sVm = sVc + GG::KC;
            const int tokbase = (blk0 + (int)jb) * kBlk;

            // ---- scores: S[head g, group][token] via HMMA on exact codes
            float sacc[2][4];
#pragma unroll
            for (int nbk = 0; nbk < 2; ++nbk) {
                sacc[nbk][0] = sacc[nbk][1] = sacc[nbk][2] = sacc[nbk][3] = 0.f;
                const int tok = 8 * nbk + tok_perm(g);
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    const uint2 w = *reinterpret_cast<const uint2 *>(sKc + tok * (D / 2) + grp * 32 + 8 * t);
                    uint32_t u[8];
                    unpack_k(w.x, *reinterpret_cast<uint32_t(*)[4]>(&u[0]));
                    unpack_k(w.y, *reinterpret_cast<uint32_t(*)[4]>(&u[4]));
#pragma unroll
                    for (int kbl = 0; kbl < 4; ++kbl) {
                        if (grp == 0)
                            mma_16816(sacc[nbk], qa[0][kbl][0], ZERO, qa[0][kbl][1], ZERO, u[2 * kbl], u[2 * kbl + 1]);
                        else
                            mma_16816(sacc[nbk], ZERO, qa[grp][kbl][0], ZERO, qa[grp][kbl][1], u[2 * kbl], u[2 * kbl + 1]);
                    }
                }
            }

            // ---- K meta of this thread's 4 tokens, scores in log2 domain
            float z[2][2];
            bool ok[2][2];
#pragma unroll
            for (int nbk = 0; nbk < 2; ++nbk) {
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const int tok = 8 * nbk + tok_perm(2 * t + e);
                    ok[nbk][e] = head_ok && (tokbase + tok < L);
                    const uint32_t *mp = reinterpret_cast<const uint32_t *>(sKm) + tok * NG;
                    float sc = 0.f;
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
                        const float2 f = meta_f2(mp[grp]);       // (min, scale)
                        sc = fmaf(sacc[nbk][e + 2 * grp], f.y, sc);
                        sc = fmaf(f.x, qs[grp], sc);
                    }
                    z[nbk][e] = ok[nbk][e] ? sc * a.scale_log2 : NEG_INF;
                }
            }

            // ---- online softmax (per head g; lanes 4g..4g+3 agree)
            float mblk = fmaxf(fmaxf(z[0][0], z[0][1]), fmaxf(z[1][0], z[1][1]));
            mblk = warp_max4(mblk);
            const float m_new = fmaxf(m_run, mblk);
            if (__any_sync(0xffffffffu, m_new > m_run)) {
                const float alpha = (m_new > m_run) ? exp2f(m_run - m_new) : 1.f;
                m_run = m_new;
                l_run *= alpha;
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) pm[grp] *= alpha;
                const float a0 = __shfl_sync(0xffffffffu, alpha, 8 * t);
                const float a1 = __shfl_sync(0xffffffffu, alpha, 8 * t + 4);
#pragma unroll
                for (int i = 0; i < NG * 4; ++i) {
                    acc[i][0] *= a0;
                    acc[i][1] *= a1;
                    acc[i][2] *= a0;
                    acc[i][3] *= a1;
                }
            }
            float p[2][2];
#pragma unroll
            for (int nbk = 0; nbk < 2; ++nbk)
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    p[nbk][e] = ok[nbk][e] ? exp2f(z[nbk][e] - m_run) : 0.f;
                    l_run += p[nbk][e];
                }

            // ---- V: O^T[dim][head] += V^T codes . (p * scale)
            const int tA0 = tok_perm(2 * t), tB0 = tok_perm(2 * t + 1);
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
                float2 vm[2][2];
#pragma unroll
                for (int nbk = 0; nbk < 2; ++nbk)
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int tok = 8 * nbk + tok_perm(2 * t + e);
                        vm[nbk][e] = meta_f2(reinterpret_cast<const uint32_t *>(sVm)[tok * NG + grp]);
                        if (!ok[nbk][e]) vm[nbk][e] = make_float2(0.f, 0.f);   // masked tail: meta may be garbage
                        pm[grp] = fmaf(p[nbk][e], vm[nbk][e].x, pm[grp]);     // V min term sum_j p_j min_jg
                    }
                const uint32_t bp0 = pack_half2(p[0][0] * vm[0][0].y, p[0][1] * vm[0][1].y);
                const uint32_t bp1 = pack_half2(p[1][0] * vm[1][0].y, p[1][1] * vm[1][1].y);
                const uint8_t *vbase = sVc + grp * 32 + 4 * g;
                const uint32_t wa0 = *reinterpret_cast<const uint32_t *>(vbase + tA0 * (D / 2));
                const uint32_t wb0 = *reinterpret_cast<const uint32_t *>(vbase + tB0 * (D / 2));
                const uint32_t wa1 = *reinterpret_cast<const uint32_t *>(vbase + (8 + tA0) * (D / 2));
                const uint32_t wb1 = *reinterpret_cast<const uint32_t *>(vbase + (8 + tB0) * (D / 2));
                uint32_t j0[8], j1[8];
                unpack_v(wa0, wb0, j0);
                unpack_v(wa1, wb1, j1);
#pragma unroll
                for (int mbl = 0; mbl < 4; ++mbl)
                    mma_16816(acc[grp * 4 + mbl], j0[2 * mbl], j0[2 * mbl + 1], j1[2 * mbl], j1[2 * mbl + 1], bp0, bp1);
            }
            __syncwarp();
            if (lane == 0 && !pc.done) {
                issue(pc, slot);
                pc.advance(wm);
            }
            ++it;
            cc.advance(wm);
        }

        // ------------------------------------------------ segment end
        const float l_tot = warp_sum4(l_run);
        float pm_tot[NG];
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) pm_tot[grp] = warp_sum4(pm[grp]);
        const int hA = 2 * t, hB = 2 * t + 1;
        const float lA = __shfl_sync(0xffffffffu, l_tot, 8 * t);
        const float lB = __shfl_sync(0xffffffffu, l_tot, 8 * t + 4);
        const float mA = __shfl_sync(0xffffffffu, m_run, 8 * t);
        const float mB = __shfl_sync(0xffffffffu, m_run, 8 * t + 4);
        float vA[NG][8], vB[NG][8];
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) {
            const float pA = __shfl_sync(0xffffffffu, pm_tot[grp], 8 * t);
            const float pB = __shfl_sync(0xffffffffu, pm_tot[grp], 8 * t + 4);
#pragma unroll
            for (int mbl = 0; mbl < 4; ++mbl) {
                vA[grp][2 * mbl] = acc[grp * 4 + mbl][0] + pA;
                vA[grp][2 * mbl + 1] = acc[grp * 4 + mbl][2] + pA;
                vB[grp][2 * mbl] = acc[grp * 4 + mbl][1] + pB;
                vB[grp][2 * mbl + 1] = acc[grp * 4 + mbl][3] + pB;
            }
        }
        const int64_t rowbase = (int64_t)b * a.Hq + (int64_t)kvh * a.G;
        if (full) {
            const float iA = 1.f / lA, iB = 1.f / lB;
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    vA[grp][i] *= iA;
                    vB[grp][i] *= iB;
                }
                if (hA < a.G) store_row8<D>(a, rowbase + hA, grp * 64 + 8 * g, vA[grp]);
                if (hB < a.G) store_row8<D>(a, rowbase + hB, grp * 64 + 8 * g, vB[grp]);
            }
        } else {
            // partial record for this (virtual warp, pair) slot
            const int64_t slot = wm.slot_of(vseg, pstart);
            float *rec = a.partials + slot * (int64_t)a.G * GG::REC;
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
                if (hA < a.G) {
                    float *r = rec + hA * GG::REC + grp * 64 + 8 * g;
                    __stcg(reinterpret_cast<float4 *>(r), make_float4(vA[grp][0], vA[grp][1], vA[grp][2], vA[grp][3]));
                    __stcg(reinterpret_cast<float4 *>(r) + 1, make_float4(vA[grp][4], vA[grp][5], vA[grp][6], vA[grp][7]));
                }
                if (hB < a.G) {
                    float *r = rec + hB * GG::REC + grp * 64 + 8 * g;
                    __stcg(reinterpret_cast<float4 *>(r), make_float4(vB[grp][0], vB[grp][1], vB[grp][2], vB[grp][3]));
                    __stcg(reinterpret_cast<float4 *>(r) + 1, make_float4(vB[grp][4], vB[grp][5], vB[grp][6], vB[grp][7]));
                }
            }
            if (g == 0) {
                if (hA < a.G) { __stcg(rec + hA * GG::REC + D, mA); __stcg(rec + hA * GG::REC + D + 1, lA); }
                if (hB < a.G) { __stcg(rec + hB * GG::REC + D, mB); __stcg(rec + hB * GG::REC + D + 1, lB); }
            }
            __threadfence();
            __syncwarp();
            // number of segments of this pair
            const int64_t pend = pstart + nb;
            const int64_t v0 = wm.vwarp_of(pstart), v1 = wm.vwarp_of(pend - 1);
            int nseg = 0;
            for (int64_t v = v0; v <= v1; ++v) nseg += (wm.R(v) < wm.R(v + 1)) ? 1 : 0;
            const int pair = b * a.Hkv + kvh;
            int last = 0;
            if (lane == 0) last = (atomicAdd(&a.counters[pair], 1) == nseg - 1);
            last = __shfl_sync(0xffffffffu, last, 0);
            if (last) {
                __threadfence();
                constexpr int DPL = D / 32;      // dims per lane
                for (int h = 0; h < a.G; ++h) {
                    float M = NEG_INF;
                    for (int64_t v = v0; v <= v1; ++v) {
                        if (!(wm.R(v) < wm.R(v + 1))) continue;
                        const float *r = a.partials + wm.slot_of(v, pstart) * (int64_t)a.G * GG::REC + h * GG::REC;
                        M = fmaxf(M, __ldcg(r + D));
                    }
                    float l = 0.f, o[DPL];
#pragma unroll
                    for (int i = 0; i < DPL; ++i) o[i] = 0.f;
                    for (int64_t v = v0; v <= v1; ++v) {
                        if (!(wm.R(v) < wm.R(v + 1))) continue;
                        const float *r = a.partials + wm.slot_of(v, pstart) * (int64_t)a.G * GG::REC + h * GG::REC;
                        const float w = exp2f(__ldcg(r + D) - M);
                        l = fmaf(__ldcg(r + D + 1), w, l);
#pragma unroll
                        for (int i = 0; i < DPL; ++i) o[i] = fmaf(__ldcg(r + lane * DPL + i), w, o[i]);
                    }
                    const float il = 1.f / l;
                    const int64_t row = rowbase + h;
#pragma unroll
                    for (int i = 0; i < DPL; ++i) {
                        const int64_t off = row * D + lane * DPL + i;
                        if (a.out_f16) static_cast<__half *>(a.out)[off] = __float2half_rn(o[i] * il);
                        else static_cast<float *>(a.out)[off] = o[i] * il;
                    }
                }
                if (lane == 0) a.counters[pair] = 0;
            }
        }
    }
}

// ---------------------------------------------------------------- host side
template <int D>
static size_t smem_bytes() {
    return 128 + (size_t)kWarps * kStages * Geo<D>::STAGE + (kMaxBatchSmem + 1) * sizeof(int);
}

template <int D>
static int ctas_per_sm() {
    static int occ[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (occ[dev] == 0) {
        cudaFuncSetAttribute(decode_attn_q4_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem_bytes<D>());
        int n = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, decode_attn_q4_kernel<D>, kWarps * 32,
                                                      smem_bytes<D>());
        occ[dev] = n > 0 ? n : 1;
    }
    return occ[dev];
}

int attn_max_warps(int head_dim) {
    const int occ = head_dim == 64 ? ctas_per_sm<64>() : ctas_per_sm<128>();
    return device_sm_count() * occ * kWarps;
}

size_t attn_workspace_bytes(int B, int Hkv, int Hq, int D, int num_splits) {
    const int G = Hq / Hkv;
    const size_t counters = ((size_t)B * Hkv * sizeof(int) + 255) / 256 * 256;
    const size_t slots = num_splits > 0 ? (size_t)B * Hkv * num_splits : 2 * (size_t)attn_max_warps(D);
    return counters + slots * G * (D + 4) * sizeof(float);
}

cudaError_t launch_decode_attention(const lmo_kv_cache &c, const void *q, int Hq, int len,
                                    const int32_t *lens, float softmax_scale, int num_splits,
                                    void *out, int out_f16, void *ws, cudaStream_t st) {
    AttnArgs a;
    a.kc = c.k_codes;
    a.vc = c.v_codes;
    a.km = reinterpret_cast<const uint32_t *>(c.k_meta);
    a.vm = reinterpret_cast<const uint32_t *>(c.v_meta);
    a.B = c.batch;
    a.Hkv = c.kv_heads;
    a.cap = c.capacity;
    a.q = static_cast<const __half *>(q);
    a.Hq = Hq;
    a.G = Hq / c.kv_heads;
    a.len = len;
    a.lens = lens;
    a.scale_log2 = softmax_scale * 1.4426950408889634f;
    a.num_splits = num_splits;
    a.out = out;
    a.out_f16 = out_f16;
    const size_t counters = ((size_t)c.batch * c.kv_heads * sizeof(int) + 255) / 256 * 256;
    a.counters = static_cast<int *>(ws);
    a.partials = reinterpret_cast<float *>(static_cast<uint8_t *>(ws) + counters);

    const int D = c.head_dim;
    const int max_ctas = attn_max_warps(D) / kWarps;
    int64_t want_warps;
    if (lens) {
        want_warps = (int64_t)max_ctas * kWarps;
    } else {
        const int64_t nbu = (len + kBlk - 1) / kBlk;
        const int64_t N = (int64_t)c.batch * c.kv_heads * nbu;
        want_warps = num_splits > 0 ? (int64_t)c.batch * c.kv_heads * num_splits : N;
    }
    int64_t ctas = (want_warps + kWarps - 1) / kWarps;
    if (ctas > max_ctas) ctas = max_ctas;
    if (ctas < 1) ctas = 1;
    if (D == 64)
        decode_attn_q4_kernel<64><<<(unsigned)ctas, kWarps * 32, smem_bytes<64>(), st>>>(a);
    else
        decode_attn_q4_kernel<128><<<(unsigned)ctas, kWarps * 32, smem_bytes<128>(), st>>>(a);
    note_launch();
    return cudaGetLastError();
}

}  // namespace lmo
