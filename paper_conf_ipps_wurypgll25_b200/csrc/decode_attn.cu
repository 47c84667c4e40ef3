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
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "common.cuh"

namespace lmo {

constexpr int kBlk = 16;      // tokens per MMA sub-block = unit of the work partition
constexpr int kSub = 2;       // sub-blocks per pipeline stage (32 tokens)
constexpr int kStageTok = kBlk * kSub;
#ifndef LMO_ATTN_WARPS
#define LMO_ATTN_WARPS 4
#endif
#ifndef LMO_ATTN_STAGES
#define LMO_ATTN_STAGES 3
#endif
#ifndef LMO_ATTN_PROFILE
#define LMO_ATTN_PROFILE 0
#endif
#ifndef LMO_LAZY_MAX
#define LMO_LAZY_MAX 0   // measured: no gain (c2), 3% loss (c5 GQA)
#endif
#ifndef LMO_Q_PF_L1
#define LMO_Q_PF_L1 0    // next segment's q rows: prefetch into L1 (1) or L2 (0)
#endif
#ifndef LMO_FENCE_CTA
#define LMO_FENCE_CTA 0  // mbarrier init made visible to the async proxy with a CTA-scope fence
#endif
#ifndef LMO_UNIFIED
#define LMO_UNIFIED 1    // MHA: one masked loop body for every stage (0: separate FULL / GEN bodies)
#endif
#ifndef LMO_GQA_VOTE
#define LMO_GQA_VOTE 1   // GQA FULL stages: rescale only when a running max moved (one vote)
#endif
#ifndef LMO_SMALL_CTAS_PER_SM
#define LMO_SMALL_CTAS_PER_SM 2   // small-batch team launches: resident CTAs per SM (0: no cap); measured
#endif                            // better than a 3-per-SM cap for 256-CTA launches
#ifndef LMO_TEAM_RING_ONLY
#define LMO_TEAM_RING_ONLY 1   // the T > 1 instance merges only on chip: launched only when every
#endif                         // team has at most one pair (else the generic instance, L2 merge)
#ifndef LMO_GQA_HOIST
#define LMO_GQA_HOIST 0   // 1: one V-exponent vote per stage before any p (measured 1% slower than per sub-block)
#endif
#ifndef LMO_NO_SCH
#define LMO_NO_SCH 0     // 1: every schedule runs the generic kernel instance (experiments)
#endif
#ifndef LMO_ATTN_MINBLOCKS_GQA
#define LMO_ATTN_MINBLOCKS_GQA 4   // 2: GQA with up to 255 registers -- faster on an 11-layer probe, slower in the 80-layer bench
#endif
#ifndef LMO_ATTN_MINBLOCKS
#define LMO_ATTN_MINBLOCKS 4
#endif
#ifndef LMO_EARLY_STAGES
#define LMO_EARLY_STAGES 2   // CACHE_STABLE: stages per warp streamed before griddepcontrol.wait
#endif
#ifndef LMO_HALF_GRID_MHA
#define LMO_HALF_GRID_MHA 1   // MHA launches with ~1 pair per warp of a 2-CTA/SM grid: 2 CTAs per SM
#endif
#ifndef LMO_DEEP_GQA
#define LMO_DEEP_GQA 1   // GQA launches with ~1 pair per warp of a 2-CTA/SM grid: deep-ring instance
#endif
constexpr int kWarps = LMO_ATTN_WARPS;    // warps per CTA
constexpr int kStages = LMO_ATTN_STAGES;  // per-warp TMA ring depth (stages of 32 tokens)
constexpr int kMaxBatchSmem = 1024;  // per-sequence-length mode: prefix array in smem

template <int D>
struct Geo {
    static constexpr int NG = D / 64;              // quantization groups per row
    static constexpr int RB = D / 2;               // code bytes per K (or V) row
    static constexpr int MB = NG * 4;              // meta bytes per K (or V) row
    static constexpr int ROW = 2 * (RB + MB);       // compressed K+V token row (144 B at D=128)
    static constexpr int OKM = RB;                 // offsets inside a row
    static constexpr int OVC = RB + MB;
    static constexpr int OVM = 2 * RB + MB;
    static constexpr int STAGE = kStageTok * ROW;  // bytes per stage
    static constexpr int REC = D + 4;              // partial record floats per head
};

#if LMO_ATTN_PROFILE
__device__ unsigned long long *g_attn_prof = nullptr;   // [slot][warp][16]: wait, total, stages, sm/warp/segs,
                                                        // globaltimer at entry, loop start, first data, end
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif

// ---------------------------------------------------------------- work map
// Global list of 16-token blocks: sequence-major, then kv head, then block
// (all int32: the ABI bounds keep N < 2^31).
struct WorkMap {
    const int *prefix;   // smem, B+1 (per-sequence lengths) or nullptr (uniform length)
    int B, Hkv, nbu;     // nbu: blocks per pair in uniform mode
    int N;               // total blocks
    int V;               // virtual warps (ranges)
    int W;               // physical warps in the grid
    int k;               // num_splits (0 = stream-K)
    int T;               // team mode: warps per (b, kvh) pair (1, 2, 4); 0 = stream-K / fixed splits
    int n_teams;         // team mode: teams in the grid
    int tsh;             // team mode: log2(T)
    int sm;              // SM-team mode: CTA c owns pairs [c*P/C, (c+1)*P/C), split evenly over its warps
    int P, C, NW;        // SM-team mode: pairs, CTAs, warps per CTA
    int vb, X0, n;       // SM-team mode, this CTA: first virtual warp, first block, blocks
    FastDiv dHkv;        // division by Hkv

    __device__ __forceinline__ int seq_start(int b) const { return prefix ? prefix[b] : b * Hkv * nbu; }
    __device__ __forceinline__ int seq_nb(int b) const {
        return prefix ? (prefix[b + 1] - prefix[b]) / Hkv : nbu;
    }
    // global block x -> (b, kvh, blk, nb)
    __device__ __forceinline__ void decode(int x, int &b, int &kvh, int &blk, int &nb) const {
        if (!prefix) {
            const int pair = x / nbu;
            blk = x - pair * nbu;
            b = pair / Hkv;
            kvh = pair - b * Hkv;
            nb = nbu;
        } else {
            int lo = 0, hi = B;  // largest b with prefix[b] <= x  (prefix[B] = N > x)
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (prefix[mid] <= x) lo = mid; else hi = mid;
            }
            b = lo;
            nb = seq_nb(b);
            const int r = x - prefix[b];
            kvh = r / nb;
            blk = r - kvh * nb;
        }
    }
    // start of virtual warp v's range
    __device__ __forceinline__ int R(int v) const {
        if (sm) return X0 + (v - vb) * n / NW;   // v in [vb, vb + NW] (this CTA's warps)
        if (k == 0) return (int)((long long)v * N / V);
        const int p = v / k;
        if (p >= B * Hkv) return N;
        const int j = v - p * k;
        const int b = p / Hkv, kvh = p - b * Hkv;
        const int nb = seq_nb(b);
        return seq_start(b) + kvh * nb + j * nb / k;
    }
    // virtual warp whose range contains block x
    __device__ __forceinline__ int vwarp_of(int x) const {
        if (k == 0) return (int)(((long long)(x + 1) * V + N - 1) / N) - 1;
        int b, kvh, blk, nb;
        decode(x, b, kvh, blk, nb);
        int j = ((blk + 1) * k + nb - 1) / nb - 1;
        if (j > k - 1) j = k - 1;
        return (b * Hkv + kvh) * k + j;
    }
};

struct AttnArgs {
    const uint8_t *kv;        // [B][Hkv][cap][ROW]
    int B, Hkv, cap;
    const __half *q;
    int Hq, G;
    int len;                  // uniform length (lens == nullptr)
    const int32_t *lens;      // per-sequence lengths or nullptr
    float scale_log2;         // softmax_scale * log2(e)
    int num_splits;           // 0 = stream-K
    int team;                 // > 0: pair-team mode with this many warps per pair
    void *out;
    int out_f16;
    int *counters;            // [B*Hkv]
    float *partials;          // [slots][G][REC]
    const __half *k_new;      // fused append (team mode): [B][Hkv][D] new token K, or nullptr
    const __half *v_new;      //                            new token V
    int early;                // prefetch the old-token cache before griddepcontrol.wait
    int flex;                 // LMO_STEP_FLEXGEN_EXACT: slot L-1 is attended with the raw fp16
    const __half *raw_k;      //   k_new / v_new [B][Hkv][D] instead of its quantized form
    const __half *raw_v;
    int prof_slot;            // (LMO_ATTN_PROFILE builds) record slot of this launch
    WorkMap wm;               // host-computed work map (uniform length; completed on device
                              // from the length prefix in per-sequence mode)
};

// Iterates the segments (maximal runs of blocks of one (b, kv head) pair) of
// the virtual warps v = gw, gw + W, ...  Within a range the two PARTIAL
// segments (first and last) come first and the full pairs in the middle come
// last, so the cross-warp merges happen early and every warp ends on
// independent work.
struct SegIter {
    int v, x0, x1, a, c, phase, mpos;
    int sx, sn, b, kvh, blk, nb;    // current segment
    bool done;

    __device__ __noinline__ void set_seg(const WorkMap &wm, int x, int n) {
        sx = x;
        sn = n;
        wm.decode(x, b, kvh, blk, nb);
    }
    // team mode: v = pair index, x0 = rank of this warp in its team (inline: cheap)
    template <int SCH>
    __device__ __forceinline__ void team_seg(const WorkMap &wm) {
        if (v >= wm.B * wm.Hkv) {
            done = true;
            return;
        }
        b = (int)wm.dHkv.div((uint32_t)v);
        kvh = v - b * wm.Hkv;
        nb = wm.seq_nb(b);
        const int T = SCH == 1 ? 1 : wm.T;
        const int lo = SCH == 1 ? 0 : x0 * nb / T, hi = SCH == 1 ? nb : (x0 + 1) * nb / T;
        blk = lo;
        sn = hi - lo;
        sx = wm.seq_start(b) + kvh * nb + lo;
        done = false;
    }
    // SM teams: the warp's range [x0, x1) walked pair by pair from cursor a (inline: cheap)
    __device__ __forceinline__ void sm_seg(const WorkMap &wm) {
        if (a >= x1) {
            done = true;
            return;
        }
        const int p = a / wm.nbu;
        b = (int)wm.dHkv.div((uint32_t)p);
        kvh = p - b * wm.Hkv;
        nb = wm.nbu;
        blk = a - p * wm.nbu;
        sx = a;
        sn = min(x1, (p + 1) * wm.nbu) - a;
        a += sn;
        done = false;
    }
    template <int SCH>
    __device__ __forceinline__ void begin_v(const WorkMap &wm) {
        if (SCH != 0 || wm.T) {
            team_seg<SCH>(wm);
        } else if (wm.sm) {
            x0 = wm.R(v);
            x1 = wm.R(v + 1);
            a = x0;
            sm_seg(wm);
        } else {
            begin_v_sk(wm);
        }
    }
    __device__ __noinline__ void begin_v_sk(const WorkMap &wm) {
        while (v < wm.V) {
            x0 = wm.R(v);
            x1 = wm.R(v + 1);
            if (x0 < x1) {
                wm.decode(x0, b, kvh, blk, nb);
                a = min(x1, x0 - blk + nb);
                if (a < x1) {
                    int b1, kvh1, blk1, nb1;
                    wm.decode(x1 - 1, b1, kvh1, blk1, nb1);
                    c = x1 - 1 - blk1;
                } else {
                    c = x1;
                }
                sx = x0;
                sn = a - x0;
                phase = 0;
                done = false;
                return;
            }
            v += wm.W;
        }
        done = true;
    }
    // out of line: runs only at segment transitions, keeps the hot loop small (I-cache)
    template <int SCH>
    __device__ __forceinline__ void next(const WorkMap &wm) {
        if (SCH != 0 || wm.T) {
            v += wm.n_teams;
            team_seg<SCH>(wm);
        } else if (wm.sm) {
            sm_seg(wm);
        } else {
            next_sk(wm);
        }
    }
    __device__ __noinline__ void next_sk(const WorkMap &wm) {
        if (phase == 0 && a < x1) {
            phase = 1;
            set_seg(wm, c, x1 - c);
        } else if (phase == 1 && a < c) {
            phase = 2;
            mpos = a;
            set_seg(wm, mpos, 0);
            sn = nb;
        } else if (phase == 2 && mpos + nb < c) {
            mpos += nb;
            set_seg(wm, mpos, 0);
            sn = nb;
        } else {
            v += wm.W;
            begin_v_sk(wm);
        }
    }
};

// ------------------------------------------------------------ fragments
// Token order inside a 16-token block: MMA row r <-> token tperm(r).  With the
// pair-interleaved V codes (round 2) the natural order is bank-conflict free.
__device__ __forceinline__ int tperm(int r) { return r; }

// Exact 4-bit codes as fp16 SUBNORMALS (no bias, no fp16 add):
//   (x & 0x000F000F) reads the nibbles at bits 0-3 / 16-19 as c * 2^-24,
//   (x & 0x00F000F0) reads the nibbles at bits 4-7 / 20-23 as 16*c * 2^-24 = c * 2^-20.
// K side, one word (8 dims) ->
//   u[0] = (nib0, nib4) * 2^-24, u[1] = (nib1, nib5) * 2^-20,
//   u[2] = (nib2, nib6) * 2^-24, u[3] = (nib3, nib7) * 2^-20.
// The 2^-20 slots meet q/16 in the MMA (see the q fragments), so every
// product is q_i c_i 2^-24.
// x >> 8 (an IMAD.HI on the FMA pipe instead of the SHF was measured 13% slower: DESIGN.md §6)
__device__ __forceinline__ uint32_t shr8(uint32_t x) { return x >> 8; }

__device__ __forceinline__ void unpack_k(uint32_t w, uint32_t *u) {
    const uint32_t s = shr8(w);
    u[0] = w & 0x000F000Fu;
    u[1] = w & 0x00F000F0u;
    u[2] = s & 0x000F000Fu;
    u[3] = s & 0x00F000F0u;
}

// V side: the cache stores the V codes of a token pair (2p, 2p+1) interleaved in 16-bit
// chunks of 4 dims (include/lmo.h): lo = [A dims 8g..8g+3 | B same dims], hi = dims
// 8g+4..8g+7 -> 8 half2 (A nib p, B nib p); even p in the 2^-24 form, odd p in 2^-20.
__device__ __forceinline__ void unpack_v(uint32_t lo, uint32_t hi, uint32_t *j) {
    const uint32_t lo8 = shr8(lo), hi8 = shr8(hi);
    j[0] = lo & 0x000F000Fu;
    j[1] = lo & 0x00F000F0u;
    j[2] = lo8 & 0x000F000Fu;
    j[3] = lo8 & 0x00F000F0u;
    j[4] = hi & 0x000F000Fu;
    j[5] = hi & 0x00F000F0u;
    j[6] = hi8 & 0x000F000Fu;
    j[7] = hi8 & 0x00F000F0u;
}

__device__ __forceinline__ float2 meta_f2(uint32_t mw) {
    const __half2 h = *reinterpret_cast<const __half2 *>(&mw);
    return __half22float2(h);   // .x = min, .y = scale
}

// explicit shared-window loads (32-bit addresses; volatile: data arrives via TMA)
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];\n" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds64(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];\n" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
// two V code words (d = 128: 8-byte aligned; d = 64: the V area starts at byte 36 of a
// 72-byte row, 4-byte alignment only)
template <int NG>
__device__ __forceinline__ uint2 load_v2(uint32_t a) {
    if constexpr (NG == 2) return lds64(a);
    else return make_uint2(lds32(a), lds32(a + 4));
}
// the NG meta words of one row (NG = 1: 4-byte aligned only)
template <int NG>
__device__ __forceinline__ uint2 load_meta(uint32_t a) {
    if constexpr (NG == 2) return lds64(a);
    else return make_uint2(lds32(a), 0u);
}

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;\n" : "=f"(y) : "f"(x));
    return y;
}

// floor(log2(h)) of a positive finite fp16 bit pattern (subnormals included)
__device__ __forceinline__ int floor_log2_h(uint32_t h) {
    const int e = (int)(h >> 10);
    return e ? e - 15 : (31 - __clz((int)h)) - 24;
}
// 2^e as an fp32 (e in [-126, 127])
__device__ __forceinline__ float exp2i(int e) { return __uint_as_float((uint32_t)(e + 127) << 23); }

__device__ __forceinline__ uint32_t movmatrix_t(uint32_t x) {
    uint32_t y;
    asm("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;\n" : "=r"(y) : "r"(x));
    return y;
}

__device__ __forceinline__ float max_over_g(float v) {   // lanes with equal t (xor 4, 8, 16)
    v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 4));
    v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 8));
    return fmaxf(v, __shfl_xor_sync(0xffffffffu, v, 16));
}
__device__ __forceinline__ float sum_over_g(float v) {
    v += __shfl_xor_sync(0xffffffffu, v, 4);
    v += __shfl_xor_sync(0xffffffffu, v, 8);
    return v + __shfl_xor_sync(0xffffffffu, v, 16);
}
__device__ __forceinline__ float sum_over_t(float v) {
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
// Per 16-token sub-block and lane (g = lane/4, t = lane%4):
//  K-MMA   S^T[token][head] (16x8) = Kc[token][dims] (A, codes as fp16 subnormals)
//                                   x q^T[dims][head] (B, fp16), one accumulator per group
//  scores  z = sigma*log2e * sum_g ( 2^20 scale_tg S_g + min_tg Qs_g )    (folded dequant)
//  softmax running max / sum per head (heads 2t, 2t+1 live in this lane)
//  P^T     (p * scaleV) packed fp16, transposed in registers with movmatrix
//  V-MMA   O^T[dim][head] (16x8 per 16 dims) += Vc^T[dims][token] (A) x P^T[token][head] (B)
//  min     Pm[head][g] += sum_token p * minV
// Stages (kSub sub-blocks) are software-pipelined: the K part of stage i+1 is
// issued before the softmax/V part of stage i.  All control state (work map,
// iterators, segment descriptors) lives in shared memory so that the
// registers hold only the math state.

struct SegDesc {      // the segment the consumer is processing
    int b, kvh, blk0, nb, sn, v, x0, L;
};

struct WarpCtl {
    SegIter pc;       // producer iterator (lane 0)
    SegIter cc;       // consumer iterator (lane 0)
    SegDesc seg;      // current consumer segment (all lanes read)
    const uint8_t *psrc;   // producer: source of the next stage
    int ptok, pend, pLb;   // producer: next stage's first token, segment end token (< L), L of the pair
    int pdone;             // producer: no more stages
    int qb, qkvh;     // pair whose q fragments are loaded
    int pissued;      // stages issued by the pre-wait prologue
};

// Producer segment setup (out of line): skip empty segments, then the byte cursor
// of the new segment's tokens < L.
template <int D, int SCH>
__device__ __noinline__ void prod_seg(WarpCtl &ctl, const WorkMap &wm, const uint8_t *kv,
                                     const int32_t *lens, int cap, int len) {
    SegIter &pc = ctl.pc;
    while (!pc.done && pc.sn == 0) pc.template next<SCH>(wm);
    if (pc.done) {
        ctl.pdone = 1;
        return;
    }
    const int Lb = lens ? min(lens[pc.b], cap) : len;
    const int t0 = pc.blk * kBlk;
    ctl.pdone = 0;
    ctl.pLb = Lb;
    ctl.ptok = t0;
    ctl.pend = min((pc.blk + pc.sn) * kBlk, Lb);
    ctl.psrc = kv + (((int64_t)pc.b * wm.Hkv + pc.kvh) * cap + t0) * Geo<D>::ROW;
}

template <int D>
struct KState {       // per-stage scores handed from the K part to the V part
    float z[kSub][2][2];
};

// smem layout: mbarriers [NW][kStages] (128-B aligned block), rings [NW][kStages][STAGE], prefix
template <int NW, int ST = kStages>
__host__ __device__ constexpr int bars_bytes() { return (NW * ST * 8 + 127) / 128 * 128; }
// Deep-ring instance (ST = kDeepStages, 2 CTAs per SM): GQA launches with about one pair per
// warp at 2 CTAs/SM keep twice the bytes in flight per busy warp (c5: 41.1 -> 39.0 us)
#ifndef LMO_DEEP_STAGES
#define LMO_DEEP_STAGES 5
#endif
constexpr int kDeepStages = LMO_DEEP_STAGES;

// SCH: 0 = any schedule (runtime work map mode); 1 = pair teams with T = 1 (one warp
// per pair, the default); 2 = pair teams with T > 1.  The specialised instances drop
// the other modes' code (smaller kernel: fewer cold instruction-cache misses).
template <int D, bool MHA, int NW, int SCH = 0, int ST = kStages>
__global__ void __launch_bounds__(NW * 32, NW == kWarps ? (ST != kStages ? 2 : MHA ? LMO_ATTN_MINBLOCKS : LMO_ATTN_MINBLOCKS_GQA) : 1)
decode_attn_q4_kernel(const AttnArgs a) {
    using GG = Geo<D>;
    constexpr bool TEAMK = SCH != 0;
    constexpr int NG = GG::NG;
    extern __shared__ __align__(128) uint8_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);                 // [NW][ST]
    uint8_t *ring = smem + bars_bytes<NW, ST>();                              // [NW][ST][STAGE]
    int *prefix = reinterpret_cast<int *>(ring + NW * ST * GG::STAGE);
    __shared__ WorkMap wms;
    __shared__ WarpCtl ctls[NW];

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int g = lane >> 2, t = lane & 3;
    // Programmatic dependent launch: let the next kernel in the stream be scheduled
    // as soon as our CTAs retire (its griddepcontrol.wait still waits for our full
    // completion and memory flush).  Without `early`, wait here for the previous
    // kernel before touching anything; with `early` (caller guarantees the previous
    // kernel does not write this cache's old tokens), first start streaming the
    // old-token cache blocks, then wait.
#if LMO_ATTN_PROFILE
    const unsigned long long prof_g0 = gtimer();
#endif
    asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory");
    const bool early = a.early && !a.lens;
    // per-sequence lengths may be produced by the previous kernel: wait first.  Uniform
    // length: the work map and producer setup read only the launch arguments and run
    // before the wait (they overlap the previous kernel's tail).
    if (a.lens) asm volatile("griddepcontrol.wait;\n" ::: "memory");
#if LMO_ATTN_PROFILE
    const unsigned long long prof_gw = gtimer();   // after the (non-early) wait
#endif

    // ---- work map (identical in every CTA)
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
    }
    if (threadIdx.x == 0) {
        WorkMap wm = a.wm;
        if (SCH == 0 && wm.sm) {
            const int p0 = (int)((long long)blockIdx.x * wm.P / wm.C);
            const int p1 = (int)((long long)(blockIdx.x + 1) * wm.P / wm.C);
            wm.vb = blockIdx.x * wm.NW;
            wm.X0 = p0 * wm.nbu;
            wm.n = (p1 - p0) * wm.nbu;
        }
        if (a.lens) {
            wm.prefix = prefix;
            wm.N = prefix[a.B];
            wm.V = wm.k == 0 ? (wm.N < wm.W ? wm.N : wm.W) : a.B * a.Hkv * wm.k;
        }
        wms = wm;
    }
    __syncthreads();
#if LMO_ATTN_PROFILE
    const unsigned long long prof_gm = gtimer();   // after the work map
#endif

    const int gw = blockIdx.x * NW + warp;

    // ---- zero rows of empty sequences (per-sequence mode only)
    if (a.lens) {
        for (int b = gw; b < a.B; b += wms.W) {
            if (a.lens[b] > 0) continue;
            for (int i = lane; i < a.Hq * D; i += 32) {
                const int64_t off = (int64_t)b * a.Hq * D + i;
                if (a.out_f16) static_cast<__half *>(a.out)[off] = __float2half_rn(0.f);
                else static_cast<float *>(a.out)[off] = 0.f;
            }
        }
    }

    uint64_t *wbar = bars + warp * ST;
    uint8_t *wring = ring + warp * ST * GG::STAGE;
    WarpCtl &ctl = ctls[warp];
    const uint64_t pol = policy_evict_first();

    // Producer (lane 0): one stage = the next (up to) 32 tokens < L_b of the producer's
    // current segment (exact-size tail, 16-B granular).  The per-stage path is a pointer
    // bump; segment transitions (work-map arithmetic) run out of line.
    auto issue = [&](int slot) {
        const int n = min(kStageTok, ctl.pend - ctl.ptok);
        // whole token pairs (a pair's V codes span both rows); cap % 16 == 0 keeps it in bounds
        const uint32_t bytes = ((n + 1) & ~1) * GG::ROW;
        mbar_arrive_expect_tx(&wbar[slot], bytes);
        bulk_g2s(wring + slot * GG::STAGE, ctl.psrc, bytes, &wbar[slot], pol);
        ctl.psrc += kStageTok * GG::ROW;
        ctl.ptok += kStageTok;
        if (ctl.ptok >= ctl.pend) {
            ctl.pc.template next<SCH>(wms);
            prod_seg<D, SCH>(ctl, wms, a.kv, a.lens, a.cap, a.len);
        }
    };

    // producer prologue: barrier init, first segment, up to ST bulk copies.  Before
    // the fused append has run (early mode) a stage that holds the append slot L-1 is
    // not issued yet; the ring is topped up after the append.
    auto holds_append_slot = [&]() {
        return ctl.ptok + min(kStageTok, ctl.pend - ctl.ptok) >= ctl.pLb;
    };
#if LMO_ATTN_PROFILE
    unsigned long long prof_gf = 0, prof_gb = 0;
#endif
    auto prologue_setup = [&]() {
        if (lane == 0) {
            for (int s = 0; s < ST; ++s) mbar_init(&wbar[s], 1);
            if (LMO_FENCE_CTA) asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            else fence_mbar_init();
#if LMO_ATTN_PROFILE
            prof_gf = gtimer();
#endif
            if (TEAMK || wms.T) {
                // team ids interleaved across CTAs (tau = team-in-CTA * grid + CTA): the busy
                // teams spread evenly over the SMs when there are fewer pairs than teams
                ctl.cc.v = (SCH == 1 ? warp : warp / wms.T) * gridDim.x + blockIdx.x;   // team id = first pair
                ctl.cc.x0 = SCH == 1 ? 0 : warp % wms.T;                              // rank in team
            } else {
                ctl.cc.v = gw;
            }
            ctl.cc.template begin_v<SCH>(wms);
            ctl.pc = ctl.cc;
            ctl.qb = -1;
            ctl.qkvh = -1;
            prod_seg<D, SCH>(ctl, wms, a.kv, a.lens, a.cap, a.len);
#if LMO_ATTN_PROFILE
            prof_gb = gtimer();
#endif
        }
        __syncwarp();
    };
    auto prologue = [&](int maxs) {              // issue up to maxs (<= ST) stages
        if (lane == 0) {
            int s = 0;
            for (; s < maxs && !ctl.pdone; ++s) {
                if (a.k_new && holds_append_slot()) break;
                issue(s);
            }
            ctl.pissued = s;
        }
        __syncwarp();
    };
    // q B-fragments of pair (b, kvh): qf[grp] for head g (MHA: q in all 8 columns ->
    // every lane's C holds real scores); qs = per-group sums of q for heads 2t, 2t+1
    uint32_t qf[NG][4][2];
    float qs[NG][2];
    const float zs = a.scale_log2;            // sigma * log2(e)
    float zk = 0.f;                           // K-score scale of the loaded q: zs * 2^24 * 2^-Eq
    auto fetch_q = [&](int b, int kvh, uint4 (&raw)[NG][2]) {
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) {
            raw[grp][0] = raw[grp][1] = make_uint4(0, 0, 0, 0);
            if (MHA || g < a.G) {
                const __half *qp = a.q + (((int64_t)b * a.Hq + kvh * a.G + (MHA ? 0 : g)) * D + grp * 64 + 16 * t);
                raw[grp][0] = *reinterpret_cast<const uint4 *>(qp);
                raw[grp][1] = *reinterpret_cast<const uint4 *>(qp + 8);
            }
        }
    };
    // The MMA operand is q' = q * 2^Eq (one power of two per pair, max|q'| in [2^14, 2^15)),
    // and the 2^-20 code slots meet q'/16: without the rescale a small q (|q| < 2^-10)
    // would become an fp16 subnormal after /16 and lose bits.  2^-Eq is folded into zk.
    auto build_q = [&](const uint4 (&raw)[NG][2]) {
        // max |q| of the pair on packed halves (sign bit cleared: an fp16 bit pattern
        // compares as an unsigned 16-bit integer)
        uint32_t mx2 = 0;
#pragma unroll
        for (int grp = 0; grp < NG; ++grp)
#pragma unroll
            for (int k = 0; k < 2; ++k) {
                const uint32_t w[4] = {raw[grp][k].x, raw[grp][k].y, raw[grp][k].z, raw[grp][k].w};
#pragma unroll
                for (int i = 0; i < 4; ++i) mx2 = __vmaxu2(mx2, w[i] & 0x7FFF7FFFu);
            }
        const uint32_t mx = __reduce_max_sync(0xffffffffu, max(mx2 & 0xFFFFu, mx2 >> 16));
        int eq = 0;
        if (mx) eq = 14 - floor_log2_h(mx);               // in [-1, 38]
        zk = zs * 16777216.0f * exp2i(-eq);
        // q' = q * 2^eq on packed halves: exact for eq >= 0 (scaling up keeps every bit, no
        // overflow by the choice of eq) and one RN for eq = -1 -- the same value as
        // RN16(float(q) * 2^eq).  2^eq > 2^15 is applied in up to three exact steps
        // (warp-uniform branch; q with max|q| < 2^-1 only).
        const int e1 = min(eq, 15);
        const __half2 s1 = __halves2half2(__ushort_as_half((uint16_t)((e1 + 15) << 10)),
                                          __ushort_as_half((uint16_t)((e1 + 15) << 10)));
        const __half2 s16 = __float2half2_rn(0.0625f);
        auto scale = [&](uint32_t x) -> __half2 {
            __half2 h = __hmul2(*reinterpret_cast<const __half2 *>(&x), s1);
            if (eq > 15) {
                const int e2 = min(eq - 15, 15), e3 = eq - 15 - e2;
                h = __hmul2(h, __halves2half2(__ushort_as_half((uint16_t)((e2 + 15) << 10)),
                                              __ushort_as_half((uint16_t)((e2 + 15) << 10))));
                h = __hmul2(h, __halves2half2(__ushort_as_half((uint16_t)((e3 + 15) << 10)),
                                              __ushort_as_half((uint16_t)((e3 + 15) << 10))));
            }
            return h;
        };
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) {
            // B fragment of k-block kbl: r = 0 -> (q[i0], q[i0+4]) meets the 2^-24 code slots,
            // r = 1 -> (q[i0+1], q[i0+5]) / 16 meets the 2^-20 slots (i0 = 8*(kbl>>1) + 2*(kbl&1))
#pragma unroll
            for (int kbl = 0; kbl < 4; ++kbl) {
                const uint4 &rw = raw[grp][kbl >> 1];
                const uint32_t wa = (kbl & 1) ? rw.y : rw.x, wb = (kbl & 1) ? rw.w : rw.z;
                const __half2 p0 = scale(prmt(wa, wb, 0x5410u));
                const __half2 p1 = __hmul2(scale(prmt(wa, wb, 0x7632u)), s16);
                qf[grp][kbl][0] = *reinterpret_cast<const uint32_t *>(&p0);
                qf[grp][kbl][1] = *reinterpret_cast<const uint32_t *>(&p1);
            }
            // Qs of heads 2t, 2t+1 from the MMA itself: A = 1 on the k rows of the 2^-24 slots
            // and 16 on the q'/16 rows, so C[., n] = sum of head n's q' (products exact), and
            // the lane's C columns 2t, 2t+1 are exactly its heads.  Qs = C * 2^-eq.
            float c[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
            for (int kbl = 0; kbl < 4; ++kbl)
                mma_16816(c, 0x3C003C00u, 0x3C003C00u, 0x4C004C00u, 0x4C004C00u, qf[grp][kbl][0], qf[grp][kbl][1]);
            qs[grp][0] = c[0] * exp2i(-eq);
            qs[grp][1] = c[1] * exp2i(-eq);
        }
    };
    auto load_q = [&](int b, int kvh) {
        uint4 raw[NG][2];
        fetch_q(b, kvh, raw);
        build_q(raw);
    };

    // ---- fused append (A2) of each pair's new token at slot L_b - 1, by the warp that
    // owns the pair's last block (team rank T-1) -- before the bulk copies of that block,
    // so its own TMA reads see the quantized token (proxy fence below).
    // appending pairs of this warp: [app_lo, app_hi) step app_step.  Teams: rank T-1 of
    // each team, pairs p_first, p_first + n_teams, ...  Stream-K (uniform length): the
    // pairs whose last block lies in this warp's range [R(gw), R(gw+1)).
    bool app_warp = false;
    int app_lo = 0, app_hi = 0, app_step = 1;
    if (a.k_new) {
        if (TEAMK || wms.T) {
            app_warp = SCH == 1 ? true : (gw % wms.T) == wms.T - 1;
            app_lo = (SCH == 1 ? warp : warp / wms.T) * gridDim.x + blockIdx.x;
            app_hi = a.B * a.Hkv;
            app_step = wms.n_teams;
        } else if (gw < wms.V) {
            app_lo = wms.R(gw) / wms.nbu;
            app_hi = wms.R(gw + 1) / wms.nbu;
            app_warp = app_lo < app_hi;
        }
    }
    const int lane8 = lane & 7, kvsel = lane / (8 * NG), grp8 = (lane >> 3) % NG;
    const bool lane_ok = lane < 16 * NG;
    const int p_first = SCH == 1 ? warp * gridDim.x + blockIdx.x
                                 : (TEAMK || wms.T) ? (warp / wms.T) * gridDim.x + blockIdx.x : 0;
    bool first_ok = (TEAMK || wms.T) && p_first < a.B * a.Hkv;
    int fb = 0, fk = 0;                 // pair of the warp's first segment (q prefetch)
    auto app_src = [&](int p) {
        return (kvsel == 0 ? a.k_new : a.v_new) + (int64_t)p * D + grp8 * 64 + lane8 * 8;
    };
    uint4 xv_first = make_uint4(0, 0, 0, 0), xv_second = make_uint4(0, 0, 0, 0);
    uint4 qraw[NG][2];
    // Team mode knows the warp's first pair: issue its q and new-token loads, then
    // (non-early) the bulk copies, and only then consume the loads -- the small loads
    // are queued ahead of the stage traffic and their latencies overlap.
    auto fetch_first = [&]() {
        if (app_warp && lane_ok && app_lo < app_hi) {
            xv_first = *reinterpret_cast<const uint4 *>(app_src(app_lo));
            if (app_lo + app_step < app_hi)      // the warp's second pair: load now, overlapped
                xv_second = *reinterpret_cast<const uint4 *>(app_src(app_lo + app_step));
        }
        if (TEAMK || wms.T) {
            fb = (int)wms.dHkv.div((uint32_t)p_first);
            fk = p_first - fb * a.Hkv;
        } else {                        // stream-K / SM teams: set by the producer prologue
            first_ok = !ctl.cc.done;
            fb = ctl.cc.b;
            fk = ctl.cc.kvh;
        }
        if (first_ok) fetch_q(fb, fk, qraw);
    };
    auto finish_first = [&]() {
        if (first_ok) {
            __syncwarp();
            if (lane == 0) {
                ctl.qb = fb;
                ctl.qkvh = fk;
            }
            build_q(qraw);
        }
        if (app_warp) {
            for (int p = app_lo; p < app_hi; p += app_step) {
                const int b = (int)wms.dHkv.div((uint32_t)p);
                const int Lb = a.lens ? min(a.lens[b], a.cap) : a.len;
                uint4 xv = p == app_lo ? xv_first : xv_second;
                if (p > app_lo + app_step && lane_ok) xv = *reinterpret_cast<const uint4 *>(app_src(p));
                uint32_t mw;
                const uint32_t w = quantize_group_lane8(xv, mw);
                if (lane_ok && Lb >= 1) {
                    uint8_t *row = const_cast<uint8_t *>(a.kv) + ((int64_t)p * a.cap + Lb - 1) * GG::ROW +
                                   kvsel * (GG::RB + GG::MB);
                    if (kvsel == 0) {
                        reinterpret_cast<uint32_t *>(row + grp8 * 32)[lane8] = w;
                    } else {                      // pair-interleaved V codes: two 16-bit chunks
                        uint8_t *pr = const_cast<uint8_t *>(a.kv) + ((int64_t)p * a.cap + ((Lb - 1) & ~1)) * GG::ROW;
                        const int c = 16 * grp8 + 2 * lane8;
                        store_v_chunk(pr, D, c, Lb - 1, w & 0xFFFFu);
                        store_v_chunk(pr, D, c + 1, Lb - 1, w >> 16);
                    }
                    if (lane8 == 0) reinterpret_cast<uint32_t *>(row + GG::RB)[grp8] = mw;
                }
            }
            asm volatile("fence.proxy.async.global;\n" ::: "memory");
        }
        __syncwarp();
    };

    // Early mode: bulk copies of old-token stages first (they may run before the previous
    // kernel has finished), then the wait, then q / new token.  Otherwise the small loads
    // go first.  Stages holding the append slot are held back until after the append.
    // (Stream-K / SM teams learn their first pair from the producer prologue.)
    prologue_setup();
    if (early) {
        // L2 prefetch, ahead of the stage copies, of what the wait releases: the first pair's
        // q rows and the new-token K/V rows of the warp's first two appending pairs.  A
        // prefetch only warms L2 (the point of coherence; L1 is not filled): the loads after
        // the wait still see the producer's writes.
        if (TEAMK || wms.T) {
            const int p0 = p_first;
            if (p0 < a.B * a.Hkv) {
                const int b0 = (int)wms.dHkv.div((uint32_t)p0), k0 = p0 - b0 * a.Hkv;
                const char *qb = reinterpret_cast<const char *>(a.q + ((int64_t)b0 * a.Hq + (int64_t)k0 * a.G) * D);
                const int qlines = a.G * D * 2 / 128;
                if (lane < qlines) asm volatile("prefetch.global.L2 [%0];" ::"l"(qb + lane * 128));
            }
            if (app_warp && lane < 4 * NG) {
                const int pa = app_lo + (lane >= 2 * NG ? app_step : 0);
                if (pa < app_hi) {
                    const int part = lane % (2 * NG);            // K lines then V lines of one row
                    const __half *src = (part < NG ? a.k_new : a.v_new) + (int64_t)pa * D;
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(reinterpret_cast<const char *>(src) +
                                                                    (part % NG) * 128));
                }
            }
        }
        prologue(min(ST, a.early));   // a.early = stages to stream before the wait
        asm volatile("griddepcontrol.wait;\n" ::: "memory");
        fetch_first();
    } else if (!(TEAMK || wms.T)) {
        if (!a.lens) asm volatile("griddepcontrol.wait;\n" ::: "memory");
        prologue(ST);
        fetch_first();
    } else {
        if (!a.lens) asm volatile("griddepcontrol.wait;\n" ::: "memory");
        fetch_first();
        prologue(ST);
    }
#if LMO_ATTN_PROFILE
    const unsigned long long prof_gp = gtimer();   // after the producer prologue
#endif
    finish_first();

#if LMO_ATTN_PROFILE
    const unsigned long long prof_ga = gtimer();   // after the fused append
#endif
    if (lane == 0)   // top the ring up (stages held back for the append)
        for (int s = ctl.pissued; s < ST && !ctl.pdone; ++s) issue(s);
    __syncwarp();

    // ---- per-lane constant shared-memory offsets inside a stage (sub-block 0)
    const int tk0 = tperm(g), tk1 = 8 + tperm(g);                    // this lane's K/meta tokens
    const uint32_t ring_u32 = smem_u32(wring);
    const uint32_t offK0 = ring_u32 + tk0 * GG::ROW + 8 * t;
    const uint32_t offKm0 = ring_u32 + tk0 * GG::ROW + GG::OKM;
    const uint32_t offVm0 = ring_u32 + tk0 * GG::ROW + GG::OVM;
    // V codes of token pair (2t, 2t+1), dims 8g..8g+7 of group grp: chunk c = (grp*64 + 8g)/4
    // lives in row 2t + c / (RB/4), word c % (RB/4) (d = 128: row 2t + grp, word 2g)
    const uint32_t offV0 = ring_u32 + (2 * t + (NG == 2 ? 0 : (g >> 2))) * GG::ROW + GG::OVC +
                           8 * (NG == 2 ? g : (g & 3));
    constexpr int dK1 = 8 * GG::ROW;   // token row +8
    constexpr int dM1 = 8 * GG::ROW;
    constexpr int dSC = kBlk * GG::ROW; // sub-block stride
    constexpr int dSM = kBlk * GG::ROW;

    const float NEG_INF = -INFINITY;
    int slot = 0;                             // consumer ring position
    uint32_t phase = 0;
#if LMO_ATTN_PROFILE
    long long prof_wait = 0, prof_t0 = clock64(), prof_seg = 0, prof_st = 0;
    long long prof_cs = 0, prof_ce = 0, prof_c0 = 0;   // cycles in segment start / end sections
    const unsigned long long prof_g1 = gtimer();
    unsigned long long prof_g2 = 0, prof_gq = 0;
#endif
    int team_k = 0;                           // pairs finished (team mode: scratch double buffer)

    for (;;) {
        {   // every lane reads the flag before lane 0 advances the iterator (WAR on ctl.cc)
            const bool all_done = ctl.cc.done;
            __syncwarp();
            if (all_done) break;
        }
        // ------------------------------------------------ segment start
#if LMO_ATTN_PROFILE
        prof_c0 = clock64();
#endif
        if (lane == 0) {
            SegIter &cc = ctl.cc;
            SegDesc d;
            d.b = cc.b; d.kvh = cc.kvh; d.blk0 = cc.blk; d.nb = cc.nb; d.sn = cc.sn;
            d.v = cc.v; d.x0 = cc.x0;
            d.L = a.lens ? min(a.lens[cc.b], a.cap) : a.len;
            ctl.seg = d;
            cc.template next<SCH>(wms);
        }
        __syncwarp();
        // L: tokens taken from the q4 cache (FlexGen-exact: all but the new token at L-1,
        // which the pair's last segment adds from its raw fp16 K/V in the epilogue)
        const int seg_n = ctl.seg.sn, blk0 = ctl.seg.blk0, L = ctl.seg.L - a.flex;
        const int Lseg = min(L, (blk0 + seg_n) * kBlk);   // end (exclusive) of this segment's tokens
#if LMO_ATTN_PROFILE
        ++prof_seg;
#endif
        {
            const int b = ctl.seg.b, kvh = ctl.seg.kvh;
            if (b != ctl.qb || kvh != ctl.qkvh) {
                __syncwarp();
                if (lane == 0) {
                    ctl.qb = b;
                    ctl.qkvh = kvh;
                }
                load_q(b, kvh);
            }
        }

#if LMO_ATTN_PROFILE
        if (prof_seg == 1) prof_gq = gtimer();
        prof_cs += clock64() - prof_c0;
#endif
        // prefetch the next segment's q rows into L2 (its first use is latency-critical)
        if (!ctl.cc.done && lane < a.G) {
            const int nb_ = ctl.cc.b, nk_ = ctl.cc.kvh;
            const char *qn = reinterpret_cast<const char *>(a.q + ((int64_t)nb_ * a.Hq + nk_ * a.G + lane) * D);
#pragma unroll
            for (int o = 0; o < D * 2; o += 128)
                if (LMO_Q_PF_L1) asm volatile("prefetch.global.L1 [%0];" ::"l"(qn + o));
                else asm volatile("prefetch.global.L2 [%0];" ::"l"(qn + o));
        }

        float m_run[2] = {NEG_INF, NEG_INF};
        float l_run[2] = {0.f, 0.f};
        float pm[2][NG];
        float acc[NG * 4][4];
#pragma unroll
        for (int grp = 0; grp < NG; ++grp) pm[0][grp] = pm[1][grp] = 0.f;
#pragma unroll
        for (int i = 0; i < NG * 4; ++i) acc[i][0] = acc[i][1] = acc[i][2] = acc[i][3] = 0.f;
        // V operand exponent: the MMA's B operand is w = p' * scaleV with p' = exp2(z - mE),
        // mE = m_run - Ei, so every w < 2^15 and the largest ones are normal fp16 (a small V
        // scale would otherwise make p * scaleV an fp16 subnormal).  l, Pm and acc all carry
        // the same 2^Ei, which cancels in o = (acc + Pm) / l; the partial records store mE.
        // Ei starts at 0 with vthr = the least nonzero scale, so the first nonzero V scale
        // sets it; afterwards it only decreases (a stage whose scale * 2^Ei >= 2^15).
        int Ei = 0;
        uint32_t vthr = 0x10000u;                 // V meta word >= vthr <=> scale >= 2^(15 - Ei)
        // (finite sentinel while no token has been seen: a segment whose tokens are all
        // masked -- FlexGen-exact's last block -- then gets p = exp2(-inf - sentinel) = 0
        // instead of exp2(-inf + inf) = NaN; records store -inf for it, see rec_m)
        float mE[2] = {-1e30f, -1e30f};
        // rare, warp-uniform: lower Ei to fit the largest V scale vx (meta word) of the warp;
        // returns the factor applied to l, Pm and acc (the caller rescales its live p)
        auto v_exp = [&](uint32_t vx) -> float {
            const int fl = floor_log2_h(__reduce_max_sync(0xffffffffu, vx >> 16));
            const int En = 14 - fl;
            const float f = exp2i(En - Ei);
            Ei = En;
            const int k = fl + 1;                 // new threshold 2^k
            vthr = (k >= -14 ? (uint32_t)(k + 15) << 10 : 1u << (k + 24)) << 16;
            l_run[0] *= f;
            l_run[1] *= f;
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
                pm[0][grp] *= f;
                pm[1][grp] *= f;
            }
#pragma unroll
            for (int i = 0; i < NG * 4; ++i) {
                acc[i][0] *= f;
                acc[i][1] *= f;
                acc[i][2] *= f;
                acc[i][3] *= f;
            }
            mE[0] = m_run[0] - (float)Ei;
            mE[1] = m_run[1] - (float)Ei;
            return f;
        };

        // K part of one stage (ring position sl/ph): wait for the data, scores
        auto wait_stage = [&](int sl, uint32_t ph) {
#if LMO_ATTN_PROFILE
            const long long pw0 = clock64();
#endif
            mbar_wait(&wbar[sl], ph);
#if LMO_ATTN_PROFILE
            if (!prof_g2) prof_g2 = gtimer();
            prof_wait += clock64() - pw0;
#endif
        };
        // mode M (decltype(full)::value): 1 = FULL (all kSub sub-blocks present, no ragged
        // tail: branch-free, no masking); 0 = GEN (sub-block count and tail tested);
        // 2 = MASKED (LMO_UNIFIED: every sub-block computed, tokens >= Lseg masked -- one
        // branch-free body for every stage of a segment, half the code)
        auto stage_k = [&](auto full, int sl, int jb, KState<D> &ks) {
            constexpr int M = (int)decltype(full)::value;
            constexpr bool F = M != 0;
            const uint32_t st = sl * GG::STAGE;
            const int nsub = F ? kSub : min(kSub, seg_n - jb);
            if constexpr (MHA) {
                // every lane scores ONE token of the stage: sub-block ls = t>>1, row g (+8 if t odd)
                const int ls = t >> 1, hi = t & 1;
                float S[NG];
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) S[grp] = 0.f;
#pragma unroll
                for (int s = 0; s < kSub; ++s) {
                    if (s < nsub) {
                        const uint32_t ss = st + s * dSC;
#pragma unroll
                        for (int grp = 0; grp < NG; ++grp) {
                            const uint2 w0 = lds64(ss + offK0 + grp * 32);
                            const uint2 w1 = lds64(ss + offK0 + dK1 + grp * 32);
                            uint32_t u0[8], u1[8];
                            unpack_k(w0.x, u0);
                            unpack_k(w0.y, u0 + 4);
                            unpack_k(w1.x, u1);
                            unpack_k(w1.y, u1 + 4);
                            float c[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                            for (int kbl = 0; kbl < 4; ++kbl)
                                mma_16816(c, u0[2 * kbl], u1[2 * kbl], u0[2 * kbl + 1], u1[2 * kbl + 1],
                                          qf[grp][kbl][0], qf[grp][kbl][1]);
                            if (s == ls) S[grp] = hi ? c[2] : c[0];
                        }
                    }
                }
                const int row = hi ? tk1 : tk0;
                const uint2 km = load_meta<NG>(ring_u32 + st + ls * dSM + row * GG::ROW + GG::OKM);
                float z = 0.f;
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    const float2 f = meta_f2(grp == 0 ? km.x : km.y);
                    z = fmaf(S[grp], f.y * zk, fmaf(f.x * zs, qs[grp][0], z));
                }
                const int tokbase = (blk0 + jb + ls) * kBlk;
                if (M == 0 && (ls >= nsub || tokbase + row >= L)) z = NEG_INF;
                if (M == 2 && tokbase + row >= Lseg) z = NEG_INF;
                ks.z[0][0][0] = z;
            } else {
#pragma unroll
            for (int s = 0; s < kSub; ++s) {
                if (s < nsub) {
                    const uint32_t ss = st + s * dSC;
                    float sacc[NG][4];
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
                        const uint2 w0 = lds64(ss + offK0 + grp * 32);
                        const uint2 w1 = lds64(ss + offK0 + dK1 + grp * 32);
                        uint32_t u0[8], u1[8];
                        unpack_k(w0.x, u0);
                        unpack_k(w0.y, u0 + 4);
                        unpack_k(w1.x, u1);
                        unpack_k(w1.y, u1 + 4);
                        sacc[grp][0] = sacc[grp][1] = sacc[grp][2] = sacc[grp][3] = 0.f;
#pragma unroll
                        for (int kbl = 0; kbl < 4; ++kbl)
                            mma_16816(sacc[grp], u0[2 * kbl], u1[2 * kbl], u0[2 * kbl + 1],
                                      u1[2 * kbl + 1], qf[grp][kbl][0], qf[grp][kbl][1]);
                    }
                    const uint32_t sm = st + s * dSM + offKm0;
#pragma unroll
                    for (int r = 0; r < 2; ++r) {
                        const uint2 km = load_meta<NG>(sm + r * dM1);
                        float z0 = 0.f, z1 = 0.f;
#pragma unroll
                        for (int grp = 0; grp < NG; ++grp) {
                            const float2 f = meta_f2(grp == 0 ? km.x : km.y);
                            const float sk = f.y * zk;
                            const float mk = f.x * zs;
                            z0 = fmaf(sacc[grp][2 * r + 0], sk, fmaf(mk, qs[grp][0], z0));
                            z1 = fmaf(sacc[grp][2 * r + 1], sk, fmaf(mk, qs[grp][1], z1));
                        }
                        ks.z[s][r][0] = z0;
                        ks.z[s][r][1] = z1;
                    }
                    const int tokbase = (blk0 + jb + s) * kBlk;
                    if (M == 0 && tokbase + kBlk > L) {                 // ragged tail
                        if (tokbase + tk0 >= L) ks.z[s][0][0] = ks.z[s][0][1] = NEG_INF;
                        if (tokbase + tk1 >= L) ks.z[s][1][0] = ks.z[s][1][1] = NEG_INF;
                    }
                    if (M == 2) {
                        if (tokbase + tk0 >= Lseg) ks.z[s][0][0] = ks.z[s][0][1] = NEG_INF;
                        if (tokbase + tk1 >= Lseg) ks.z[s][1][0] = ks.z[s][1][1] = NEG_INF;
                    }
                } else {
                    ks.z[s][0][0] = ks.z[s][0][1] = ks.z[s][1][0] = ks.z[s][1][1] = NEG_INF;
                }
            }
            }
        };

        // softmax + V part of one stage, then hand the slot back to the producer
        auto stage_v = [&](auto full, int sl, int jb, const KState<D> &ks) {
            constexpr int M = (int)decltype(full)::value;
            constexpr bool F = M != 0;
            const uint32_t st = sl * GG::STAGE;
            const int nsub = F ? kSub : min(kSub, seg_n - jb);
            const bool tail = M == 2 || (M == 0 && (blk0 + jb + kSub) * kBlk > L);
            if constexpr (MHA) {
                // ---- one token per lane: warp-wide running max, p, V meta, w = p*scale
                const int ls = t >> 1, hi = t & 1;
                const int row = hi ? tk1 : tk0;
                const float z = ks.z[0][0][0];
                // the running max moves only if some lane's score exceeds it: one vote
                // instead of a 5-shuffle max chain on most stages (same result)
                if (!LMO_LAZY_MAX || __any_sync(0xffffffffu, z > m_run[0])) {
                float mb = z;
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) mb = fmaxf(mb, __shfl_xor_sync(0xffffffffu, mb, off));
                if (mb > m_run[0]) {                          // warp-uniform
                    const float a0 = fast_exp2(m_run[0] - mb);
                    m_run[0] = mb;
                    mE[0] = mb - (float)Ei;
                    l_run[0] *= a0;
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) pm[0][grp] *= a0;
#pragma unroll
                    for (int i = 0; i < NG * 4; ++i) {
                        acc[i][0] *= a0;
                        acc[i][1] *= a0;
                        acc[i][2] *= a0;
                        acc[i][3] *= a0;
                    }
                }
                }
                float p = fast_exp2(z - mE[0]);
                const uint2 vmw = load_meta<NG>(ring_u32 + st + ls * dSM + row * GG::ROW + GG::OVM);
                {
                    uint32_t vx = NG == 2 ? max(vmw.x, vmw.y) : vmw.x;
                    if (M != 1 && z == NEG_INF) vx = 0u;                  // stale meta of masked slots
                    if (__any_sync(0xffffffffu, vx >= vthr)) p *= v_exp(vx);
                }
                l_run[0] += p;
                float w[2] = {0.f, 0.f};
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    float2 f = meta_f2(grp == 0 ? vmw.x : vmw.y);
                    if (M != 1 && z == NEG_INF) f = make_float2(0.f, 0.f);     // stale meta of masked slots
                    pm[0][grp] = fmaf(p, f.x, pm[0][grp]);
                    w[grp] = p * f.y;
                }
                const uint32_t xw = pack_half2(w[0], w[1]);           // (group 0, group 1)
#pragma unroll
                for (int s = 0; s < kSub; ++s) {
                    if (s < nsub) {
                        // B = P^T: k = 2t, 2t+1 (rows 2t, 2t+1) and 2t+8, 2t+9 (rows +8), any column
                        const uint32_t x0 = __shfl_sync(0xffffffffu, xw, 8 * t + 2 * s);
                        const uint32_t x1 = __shfl_sync(0xffffffffu, xw, 8 * t + 4 + 2 * s);
                        const uint32_t x2 = __shfl_sync(0xffffffffu, xw, 8 * t + 2 * s + 1);
                        const uint32_t x3 = __shfl_sync(0xffffffffu, xw, 8 * t + 5 + 2 * s);
                        const uint32_t ss = st + s * dSC;
#pragma unroll
                        for (int grp = 0; grp < NG; ++grp) {
                            const uint32_t sel = grp == 0 ? 0x5410u : 0x7632u;
                            const uint32_t bp0 = prmt(x0, x1, sel), bp1 = prmt(x2, x3, sel);
                            const uint2 v0 = load_v2<NG>(ss + offV0 + grp * GG::ROW);
                            const uint2 v1 = load_v2<NG>(ss + offV0 + dK1 + grp * GG::ROW);
                            uint32_t j0[8], j1[8];
                            unpack_v(v0.x, v0.y, j0);
                            unpack_v(v1.x, v1.y, j1);
#pragma unroll
                            for (int mbl = 0; mbl < 4; ++mbl)
                                mma_16816(acc[grp * 4 + mbl], j0[2 * mbl], j0[2 * mbl + 1], j1[2 * mbl],
                                          j1[2 * mbl + 1], bp0, bp1);
                        }
                    }
                }
                __syncwarp();
                if (lane == 0 && !ctl.pdone) issue(sl);
#if LMO_ATTN_PROFILE
                ++prof_st;
#endif
                return;
            }
            float mb0 = fmaxf(fmaxf(ks.z[0][0][0], ks.z[0][1][0]), fmaxf(ks.z[kSub - 1][0][0], ks.z[kSub - 1][1][0]));
            float mb1 = fmaxf(fmaxf(ks.z[0][0][1], ks.z[0][1][1]), fmaxf(ks.z[kSub - 1][0][1], ks.z[kSub - 1][1][1]));
            // lazy: the running maxima move only if some lane's score exceeds them (one vote;
            // the shuffle reductions and the rescale run only then -- same result)
            if (!LMO_LAZY_MAX || __any_sync(0xffffffffu, (mb0 > m_run[0]) || (mb1 > m_run[1]))) {
            mb0 = max_over_g(mb0);
            mb1 = max_over_g(mb1);
            const float mn0 = fmaxf(m_run[0], mb0), mn1 = fmaxf(m_run[1], mb1);
            // (non-lazy builds: FULL stages rescale unconditionally, branch-free; GEN stages
            // skip it when no running max moved)
            if (LMO_LAZY_MAX || (F && !LMO_GQA_VOTE) || __any_sync(0xffffffffu, (mn0 > m_run[0]) || (mn1 > m_run[1]))) {
                const float a0 = fast_exp2(m_run[0] - mn0), a1 = fast_exp2(m_run[1] - mn1);
                m_run[0] = mn0;
                m_run[1] = mn1;
                mE[0] = mn0 - (float)Ei;
                mE[1] = mn1 - (float)Ei;
                l_run[0] *= a0;
                l_run[1] *= a1;
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    pm[0][grp] *= a0;
                    pm[1][grp] *= a1;
                }
#pragma unroll
                for (int i = 0; i < NG * 4; ++i) {
                    acc[i][0] *= a0;
                    acc[i][1] *= a1;
                    acc[i][2] *= a0;
                    acc[i][3] *= a1;
                }
            }
            }
            // V meta of the stage's rows (both sub-blocks) and ONE vote for the V operand
            // exponent before any p is formed (LMO_GQA_HOIST; else per sub-block)
            uint2 vmS[kSub][2];
#pragma unroll
            for (int s = 0; s < kSub; ++s) {
                const uint32_t sm = st + s * dSM;
                vmS[s][0] = (s < nsub) ? load_meta<NG>(sm + offVm0) : make_uint2(0u, 0u);
                vmS[s][1] = (s < nsub) ? load_meta<NG>(sm + offVm0 + dM1) : make_uint2(0u, 0u);
            }
            if (LMO_GQA_HOIST) {
                uint32_t vx = 0u;
#pragma unroll
                for (int s = 0; s < kSub; ++s)
#pragma unroll
                    for (int r = 0; r < 2; ++r) {
                        uint32_t v = NG == 2 ? max(vmS[s][r].x, vmS[s][r].y) : vmS[s][r].x;
                        if (tail && ks.z[s][r][0] == NEG_INF) v = 0u;   // masked: meta may be stale
                        vx = max(vx, v);
                    }
                if (__any_sync(0xffffffffu, vx >= vthr)) v_exp(vx);
            }
#pragma unroll
            for (int s = 0; s < kSub; ++s) {
                if (s < nsub) {
                    float p[2][2];
#pragma unroll
                    for (int r = 0; r < 2; ++r) {
                        p[r][0] = fast_exp2(ks.z[s][r][0] - mE[0]);
                        p[r][1] = fast_exp2(ks.z[s][r][1] - mE[1]);
                    }
                    const uint32_t ss = st + s * dSC;
                    const uint2 vmA = vmS[s][0];
                    const uint2 vmB = vmS[s][1];
                    if (!LMO_GQA_HOIST) {
                        uint32_t vxA = NG == 2 ? max(vmA.x, vmA.y) : vmA.x;
                        uint32_t vxB = NG == 2 ? max(vmB.x, vmB.y) : vmB.x;
                        if (tail) {                    // masked tail tokens: meta may be stale
                            if (ks.z[s][0][0] == NEG_INF) vxA = 0u;
                            if (ks.z[s][1][0] == NEG_INF) vxB = 0u;
                        }
                        const uint32_t vx = max(vxA, vxB);
                        if (__any_sync(0xffffffffu, vx >= vthr)) {
                            const float f = v_exp(vx);
                            p[0][0] *= f;
                            p[0][1] *= f;
                            p[1][0] *= f;
                            p[1][1] *= f;
                        }
                    }
                    l_run[0] += p[0][0] + p[1][0];
                    l_run[1] += p[0][1] + p[1][1];
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
                        float2 f0 = meta_f2(grp == 0 ? vmA.x : vmA.y);
                        float2 f1 = meta_f2(grp == 0 ? vmB.x : vmB.y);
                        if (tail) {                    // masked tail tokens: meta may be stale
                            if (ks.z[s][0][0] == NEG_INF) f0 = make_float2(0.f, 0.f);
                            if (ks.z[s][1][0] == NEG_INF) f1 = make_float2(0.f, 0.f);
                        }
                        pm[0][grp] = fmaf(p[0][0], f0.x, fmaf(p[1][0], f1.x, pm[0][grp]));
                        pm[1][grp] = fmaf(p[0][1], f0.x, fmaf(p[1][1], f1.x, pm[1][grp]));
                        // P^T: (token row, heads 2t..2t+1) -> transpose -> (head g, tokens 2t..2t+1)
                        const uint32_t bp0 = movmatrix_t(pack_half2(p[0][0] * f0.y, p[0][1] * f0.y));
                        const uint32_t bp1 = movmatrix_t(pack_half2(p[1][0] * f1.y, p[1][1] * f1.y));
                        const uint2 v0 = load_v2<NG>(ss + offV0 + grp * GG::ROW);
                        const uint2 v1 = load_v2<NG>(ss + offV0 + dK1 + grp * GG::ROW);
                        uint32_t j0[8], j1[8];
                        unpack_v(v0.x, v0.y, j0);
                        unpack_v(v1.x, v1.y, j1);
#pragma unroll
                        for (int mbl = 0; mbl < 4; ++mbl)
                            mma_16816(acc[grp * 4 + mbl], j0[2 * mbl], j0[2 * mbl + 1], j1[2 * mbl],
                                      j1[2 * mbl + 1], bp0, bp1);
                    }
                }
            }
            __syncwarp();
            if (lane == 0 && !ctl.pdone) issue(sl);
#if LMO_ATTN_PROFILE
            ++prof_st;
#endif
        };

        auto advance = [&](int &sl, uint32_t &ph) {
            if (++sl == ST) {
                sl = 0;
                ph ^= 1u;
            }
        };

        // software pipeline over the segment's stages: K part of stage i+1, then
        // softmax/V part of stage i.  Stages with all sub-blocks present and no
        // ragged tail take the branch-free FULL path (the hot loop); the rest
        // (at most the last one or two of a segment) take the general path.
        const int nst = (seg_n + kSub - 1) / kSub;
        KState<D> kC, kN;
        if constexpr (LMO_UNIFIED && MHA) {   // (measured: MHA gains, GQA loses)
        const std::integral_constant<int, 2> MK{};
        if (nst > 0) {
            wait_stage(slot, phase);
            stage_k(MK, slot, 0, kC);
        }
        int i = 0;
#pragma unroll 1
        for (; i + 1 < nst; ++i) {
            int slN = slot;
            uint32_t phN = phase;
            advance(slN, phN);
            wait_stage(slN, phN);
            stage_k(MK, slN, (i + 1) * kSub, kN);
            stage_v(MK, slot, i * kSub, kC);
            slot = slN;
            phase = phN;
            kC = kN;
        }
        if (nst > 0) {            // the last stage's V part (peeled: keeps the loop body branch-free)
            stage_v(MK, slot, i * kSub, kC);
            advance(slot, phase);
        }
        } else {
        const int nfull = max(0, min(seg_n / kSub, (L / kBlk - blk0) / kSub));
        const std::true_type FULL{};
        const std::false_type GEN{};
        if (nst > 0) {
            wait_stage(slot, phase);
            if (nfull > 0) stage_k(FULL, slot, 0, kC);
            else stage_k(GEN, slot, 0, kC);
        }
        int i = 0;
        // steady state: contiguous hot loop (FULL K part of i+1, FULL V part of i)
#pragma unroll 1
        for (; i + 1 < nfull; ++i) {
            int slN = slot;
            uint32_t phN = phase;
            advance(slN, phN);
            wait_stage(slN, phN);
            stage_k(FULL, slN, (i + 1) * kSub, kN);
            stage_v(FULL, slot, i * kSub, kC);
            slot = slN;
            phase = phN;
            kC = kN;
        }
        // remainder: at most the last two stages of the segment
#pragma unroll 1
        for (; i < nst; ++i) {
            int slN = slot;
            uint32_t phN = phase;
            advance(slN, phN);
            if (i + 1 < nst) {
                wait_stage(slN, phN);
                stage_k(GEN, slN, (i + 1) * kSub, kN);
            }
            if (i < nfull) stage_v(FULL, slot, i * kSub, kC);
            else stage_v(GEN, slot, i * kSub, kC);
            slot = slN;
            phase = phN;
            kC = kN;
        }
        }

        // ------------------------------------------------ segment end
#if LMO_ATTN_PROFILE
        prof_c0 = clock64();
#endif
        // heads 2t+e: reduce l and Pm over the 8 g-lanes; O = 2^24 acc(row g) / 2^20 acc(row g+8) + Pm
        float lt[2], pmt[2][NG];
        if constexpr (MHA) {      // per-lane tokens: full-warp sums; head 0 only
            float l = l_run[0];
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) l += __shfl_xor_sync(0xffffffffu, l, off);
            lt[0] = lt[1] = l;
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) {
                float v = pm[0][grp];
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
                pmt[0][grp] = pmt[1][grp] = v;
            }
        } else {
#pragma unroll
        for (int e = 0; e < 2; ++e) {
            lt[e] = sum_over_g(l_run[e]);
#pragma unroll
            for (int grp = 0; grp < NG; ++grp) pmt[e][grp] = sum_over_g(pm[e][grp]);
        }
        }
        float vo[2][NG][8];
#pragma unroll
        for (int grp = 0; grp < NG; ++grp)
#pragma unroll
            for (int mbl = 0; mbl < 4; ++mbl)
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    vo[e][grp][2 * mbl] = fmaf(acc[grp * 4 + mbl][e], 16777216.0f, pmt[e][grp]);
                    vo[e][grp][2 * mbl + 1] = fmaf(acc[grp * 4 + mbl][2 + e], 1048576.0f, pmt[e][grp]);
                }
        const SegDesc sd = ctl.seg;
        const int64_t rowbase = (int64_t)sd.b * a.Hq + (int64_t)sd.kvh * a.G;
        if (a.flex && sd.L > 0 && sd.blk0 + sd.sn == sd.nb) {
            // FlexGen-exact (NEXT-1; reading 13b): the new token's own K/V enter its
            // attention unquantized.  Lane (g, t) owns dims grp*64 + 8g .. +7 of heads 2t, 2t+1
            // (MHA: head 0): z_new = sigma*log2e * q.k_new (fp32, reduced over g), merged into
            // the running softmax with the same 2^Ei factor as l, Pm and acc.
            const int64_t pr = ((int64_t)sd.b * a.Hkv + sd.kvh) * D;
            float z[2];
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int h = MHA ? 0 : min(2 * t + e, a.G - 1);
                const __half *qp = a.q + (rowbase + h) * D;
                float dot = 0.f;
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    const uint4 qw = *reinterpret_cast<const uint4 *>(qp + grp * 64 + 8 * g);
                    const uint4 kw = *reinterpret_cast<const uint4 *>(a.raw_k + pr + grp * 64 + 8 * g);
                    const __half2 *qh = reinterpret_cast<const __half2 *>(&qw);
                    const __half2 *kh = reinterpret_cast<const __half2 *>(&kw);
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const float2 qf2 = __half22float2(qh[i]), kf2 = __half22float2(kh[i]);
                        dot = fmaf(qf2.x, kf2.x, fmaf(qf2.y, kf2.y, dot));
                    }
                }
                z[e] = sum_over_g(dot) * zs;
            }
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const float m2 = fmaxf(m_run[e], z[e]);
                const float sc = fast_exp2(mE[e] - (m2 - (float)Ei));     // old terms (0 if none)
                const float pn = fast_exp2(z[e] - m2) * exp2i(Ei);
                lt[e] = fmaf(lt[e], sc, pn);
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
                    const uint4 vw = *reinterpret_cast<const uint4 *>(a.raw_v + pr + grp * 64 + 8 * g);
                    const __half2 *vh = reinterpret_cast<const __half2 *>(&vw);
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const float2 v2 = __half22float2(vh[i]);
                        vo[e][grp][2 * i] = fmaf(vo[e][grp][2 * i], sc, pn * v2.x);
                        vo[e][grp][2 * i + 1] = fmaf(vo[e][grp][2 * i + 1], sc, pn * v2.y);
                    }
                }
                m_run[e] = m2;
                mE[e] = m2 - (float)Ei;
            }
        }
        const bool full = SCH == 1 || (SCH == 0 && (sd.blk0 == 0) && (sd.sn == sd.nb) && wms.T <= 1);
        if (SCH == 2 && sd.v + wms.n_teams >= a.B * a.Hkv) {
            // ---- pair team (T = 2 or 4), the team's LAST pair (the only pair when teams
            // outnumber pairs -- the regime teams are chosen for): A4 on chip.  The producers of
            // ranks 1..T-1 have issued nothing beyond this segment and every issued stage is
            // consumed, so their TMA rings are idle: each writes its partial (numerators, m, l
            // -- in the SAME lane layout) into its own ring and arrives on a named barrier; rank
            // 0 syncs, merges in registers and stores.  No L2 round trip, no atomics, no extra
            // shared memory.
            const int T = wms.T, ti = warp / T, rank = warp - ti * T;
            const uint32_t bar_full = 1 + ti, bar_n = 32 * T;
            auto part_of = [&](int r) {
                return reinterpret_cast<float *>(ring + (size_t)(ti * T + r) * ST * GG::STAGE);
            };
            if (rank != 0) {
                float *part = part_of(rank);
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const int h = 2 * t + e;
                    if (h < a.G) {
                        float *ph = part + h * (D + 4);             // (16-B aligned head records)
#pragma unroll
                        for (int grp = 0; grp < NG; ++grp) {
                            float4 *r4 = reinterpret_cast<float4 *>(ph + grp * 64 + 8 * g);
                            r4[0] = make_float4(vo[e][grp][0], vo[e][grp][1], vo[e][grp][2], vo[e][grp][3]);
                            r4[1] = make_float4(vo[e][grp][4], vo[e][grp][5], vo[e][grp][6], vo[e][grp][7]);
                        }
                        if (g == 0) {
                            ph[D] = m_run[e] == NEG_INF ? NEG_INF : mE[e];
                            ph[D + 1] = lt[e];
                        }
                    }
                }
                asm volatile("bar.arrive %0, %1;\n" ::"r"(bar_full), "r"(bar_n) : "memory");
            } else {
                asm volatile("bar.sync %0, %1;\n" ::"r"(bar_full), "r"(bar_n) : "memory");
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const int h = 2 * t + e;
                    const int hc = min(h, a.G - 1);
                    const float m0 = m_run[e] == NEG_INF ? NEG_INF : mE[e];
                    float M = m0;
                    for (int r = 1; r < T; ++r) M = fmaxf(M, part_of(r)[hc * (D + 4) + D]);
                    if (h >= a.G || M == NEG_INF) continue;      // (empty sequence: zero row written)
                    const float w0 = fast_exp2(m0 - M);
                    float l = lt[e] * w0;
                    float o[NG][8];
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp)
#pragma unroll
                        for (int i = 0; i < 8; ++i) o[grp][i] = vo[e][grp][i] * w0;
                    for (int r = 1; r < T; ++r) {
                        const float *ph = part_of(r) + hc * (D + 4);
                        const float wr = fast_exp2(ph[D] - M);
                        l = fmaf(ph[D + 1], wr, l);
#pragma unroll
                        for (int grp = 0; grp < NG; ++grp) {
                            const float4 *r4 = reinterpret_cast<const float4 *>(ph + grp * 64 + 8 * g);
                            const float4 x0 = r4[0], x1 = r4[1];
                            o[grp][0] = fmaf(x0.x, wr, o[grp][0]); o[grp][1] = fmaf(x0.y, wr, o[grp][1]);
                            o[grp][2] = fmaf(x0.z, wr, o[grp][2]); o[grp][3] = fmaf(x0.w, wr, o[grp][3]);
                            o[grp][4] = fmaf(x1.x, wr, o[grp][4]); o[grp][5] = fmaf(x1.y, wr, o[grp][5]);
                            o[grp][6] = fmaf(x1.z, wr, o[grp][6]); o[grp][7] = fmaf(x1.w, wr, o[grp][7]);
                        }
                    }
                    const float il = __frcp_rn(l);
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
#pragma unroll
                        for (int i = 0; i < 8; ++i) o[grp][i] *= il;
                        store_row8<D>(a, rowbase + h, grp * 64 + 8 * g, o[grp]);
                    }
                }
            }
            ++team_k;
        } else if ((SCH == 2 && !LMO_TEAM_RING_ONLY) || (SCH == 0 && wms.T > 1)) {
            // ---- pair team: partials through L2 scratch, named barrier, rank 0 merges
            const int T = wms.T;
            const int64_t myslot = 2 * (int64_t)gw + (team_k & 1);
            float *rec = a.partials + myslot * (int64_t)a.G * GG::REC;
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int h = 2 * t + e;
                if (h < a.G) {
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
                        float4 *r4 = reinterpret_cast<float4 *>(rec + h * GG::REC + grp * 64 + 8 * g);
                        __stcg(r4, make_float4(vo[e][grp][0], vo[e][grp][1], vo[e][grp][2], vo[e][grp][3]));
                        __stcg(r4 + 1, make_float4(vo[e][grp][4], vo[e][grp][5], vo[e][grp][6], vo[e][grp][7]));
                    }
                    if (g == 0) {
                        __stcg(rec + h * GG::REC + D, m_run[e] == NEG_INF ? NEG_INF : mE[e]);
                        __stcg(rec + h * GG::REC + D + 1, lt[e]);
                    }
                }
            }
            asm volatile("bar.sync %0, %1;\n" ::"r"(1 + warp / T), "r"(T * 32) : "memory");
            // every warp of the team merges heads h = rank, rank + T, ...; all loads of a
            // head are independent (one L2 round trip per head)
            {
                constexpr int DPL = D / 32;
                const int rank = gw % T, gw0 = gw - rank;
                const float *base = a.partials + (int64_t)(team_k & 1) * a.G * GG::REC;
                for (int h = rank; h < a.G; h += T) {
                    float mj[kWarps], lj[kWarps], oj[kWarps][DPL];   // (teams: T <= kWarps)
#pragma unroll
                    for (int j = 0; j < kWarps; ++j) {
                        if (j < T) {
                            const float *r = base + 2 * (int64_t)(gw0 + j) * a.G * GG::REC + h * GG::REC;
                            mj[j] = __ldcg(r + D);
                            lj[j] = __ldcg(r + D + 1);
                            if constexpr (DPL == 4) {
                                const float4 x = __ldcg(reinterpret_cast<const float4 *>(r) + lane);
                                oj[j][0] = x.x; oj[j][1] = x.y; oj[j][2] = x.z; oj[j][3] = x.w;
                            } else {
#pragma unroll
                                for (int i2 = 0; i2 < DPL; ++i2) oj[j][i2] = __ldcg(r + lane * DPL + i2);
                            }
                        }
                    }
                    float M = NEG_INF;
#pragma unroll
                    for (int j = 0; j < kWarps; ++j) if (j < T) M = fmaxf(M, mj[j]);
                    if (M == NEG_INF) continue;          // empty sequence: zero row already written
                    float l = 0.f, o[DPL];
#pragma unroll
                    for (int i2 = 0; i2 < DPL; ++i2) o[i2] = 0.f;
#pragma unroll
                    for (int j = 0; j < kWarps; ++j) {
                        if (j < T) {
                            const float w = fast_exp2(mj[j] - M);
                            l = fmaf(lj[j], w, l);
#pragma unroll
                            for (int i2 = 0; i2 < DPL; ++i2) o[i2] = fmaf(oj[j][i2], w, o[i2]);
                        }
                    }
                    const float il = __frcp_rn(l);
                    const int64_t row = rowbase + h;
                    if (a.out_f16) {
#pragma unroll
                        for (int i2 = 0; i2 < DPL; ++i2)
                            static_cast<__half *>(a.out)[row * D + lane * DPL + i2] = __float2half_rn(o[i2] * il);
                    } else if constexpr (DPL == 4) {
                        reinterpret_cast<float4 *>(static_cast<float *>(a.out) + row * D)[lane] =
                            make_float4(o[0] * il, o[1] * il, o[2] * il, o[3] * il);
                    } else {
#pragma unroll
                        for (int i2 = 0; i2 < DPL; ++i2) static_cast<float *>(a.out)[row * D + lane * DPL + i2] = o[i2] * il;
                    }
                }
            }
            ++team_k;
        } else if (full) {
            // (an empty sequence -- per-sequence length 0 -- keeps the zero row written at entry)
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int h = 2 * t + e;
                const float il = __frcp_rn(lt[e]);
                if (sd.L <= 0) break;
#pragma unroll
                for (int grp = 0; grp < NG; ++grp) {
#pragma unroll
                    for (int i = 0; i < 8; ++i) vo[e][grp][i] *= il;
                    if (h < a.G) store_row8<D>(a, rowbase + h, grp * 64 + 8 * g, vo[e][grp]);
                }
            }
        } else if constexpr (SCH == 0) {
            const WorkMap wm = wms;
            // pair start = global index of the pair's first block
            const int ps = wm.seq_start(sd.b) + sd.kvh * sd.nb;
            // partial record in slot (virtual warp, first/last) -- stream-K -- or (virtual warp)
            const int64_t rslot = wm.k == 0 ? 2 * (int64_t)sd.v + (sd.x0 < ps ? 1 : 0) : sd.v;
            float *rec = a.partials + rslot * (int64_t)a.G * GG::REC;
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int h = 2 * t + e;
                if (h < a.G) {
#pragma unroll
                    for (int grp = 0; grp < NG; ++grp) {
                        float4 *r4 = reinterpret_cast<float4 *>(rec + h * GG::REC + grp * 64 + 8 * g);
                        __stcg(r4, make_float4(vo[e][grp][0], vo[e][grp][1], vo[e][grp][2], vo[e][grp][3]));
                        __stcg(r4 + 1, make_float4(vo[e][grp][4], vo[e][grp][5], vo[e][grp][6], vo[e][grp][7]));
                    }
                    if (g == 0) {
                        __stcg(rec + h * GG::REC + D, m_run[e] == NEG_INF ? NEG_INF : mE[e]);
                        __stcg(rec + h * GG::REC + D + 1, lt[e]);
                    }
                }
            }
            if (wm.sm) {   // SM teams: merged once, after the CTA barrier at the end
                __syncwarp();
                continue;
            }
            __threadfence();
            __syncwarp();
            // segments of this pair = non-empty ranges of virtual warps v0..v1
            const int v0 = wm.vwarp_of(ps), v1 = wm.vwarp_of(ps + sd.nb - 1);
            int nseg = v1 - v0 + 1;
            if (wm.k != 0) {
                nseg = 0;
                for (int v = v0; v <= v1; ++v) nseg += (wm.R(v) < wm.R(v + 1)) ? 1 : 0;
            }
            const int pair = sd.b * a.Hkv + sd.kvh;
            int last = 0;
            if (lane == 0) last = (atomicAdd(&a.counters[pair], 1) == nseg - 1);
            last = __shfl_sync(0xffffffffu, last, 0);
            if (last) {
                __threadfence();
                // slot of the j-th segment; stream-K: only v0's range can start before the pair
                const int64_t s0 = wm.k == 0 ? 2 * (int64_t)v0 + (wm.R(v0) < ps ? 1 : 0) : v0;
                constexpr int DPL = D / 32;      // dims per lane
                for (int h = 0; h < a.G; ++h) {
                    // pass 1 (lanes over segments): max of the partial maxima
                    float M = NEG_INF;
                    for (int j = lane; j < v1 - v0 + 1; j += 32) {
                        const int v = v0 + j;
                        if (wm.k != 0 && !(wm.R(v) < wm.R(v + 1))) continue;
                        const int64_t sl = wm.k == 0 ? (j == 0 ? s0 : 2 * (int64_t)v) : v;
                        M = fmaxf(M, __ldcg(a.partials + sl * a.G * GG::REC + h * GG::REC + D));
                    }
#pragma unroll
                    for (int off = 16; off > 0; off >>= 1) M = fmaxf(M, __shfl_xor_sync(0xffffffffu, M, off));
                    float l = 0.f, o[DPL];
#pragma unroll
                    for (int i = 0; i < DPL; ++i) o[i] = 0.f;
                    // pass 2 (all lanes, each its own dims): weighted sums
                    for (int j = 0; j < v1 - v0 + 1; ++j) {
                        const int v = v0 + j;
                        if (wm.k != 0 && !(wm.R(v) < wm.R(v + 1))) continue;
                        const int64_t sl = wm.k == 0 ? (j == 0 ? s0 : 2 * (int64_t)v) : v;
                        const float *r = a.partials + sl * a.G * GG::REC + h * GG::REC;
                        const float w = exp2f(__ldcg(r + D) - M);
                        l = fmaf(__ldcg(r + D + 1), w, l);
                        if (DPL == 4) {
                            const float4 x = __ldcg(reinterpret_cast<const float4 *>(r) + lane);
                            o[0] = fmaf(x.x, w, o[0]);
                            o[1] = fmaf(x.y, w, o[1]);
                            o[2] = fmaf(x.z, w, o[2]);
                            o[3] = fmaf(x.w, w, o[3]);
                        } else {
#pragma unroll
                            for (int i = 0; i < DPL; ++i) o[i] = fmaf(__ldcg(r + lane * DPL + i), w, o[i]);
                        }
                    }
                    const float il = __frcp_rn(l);
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
        __syncwarp();
#if LMO_ATTN_PROFILE
        prof_ce += clock64() - prof_c0;
#endif
    }

#if LMO_ATTN_PROFILE
    prof_gf = gtimer();   // (slot 13 reused: end of the main loop)
#endif
    // ---- SM teams (A4): the CTA's pairs that were cut between warps are merged here,
    // once, after one CTA barrier (partials in L2 scratch; no fences or atomics).
    if (SCH == 0 && wms.sm) {
        __syncthreads();
        const WorkMap wm = wms;
        const int c = blockIdx.x;
        const int X0 = wm.X0, n = wm.n;
        const int p0 = X0 / wm.nbu, p1 = (X0 + n) / wm.nbu;
        // owner of block x = the largest warp w with X0 + floor(w n / NW) <= x
        auto owner = [&](int x) { return ((x - X0 + 1) * NW + n - 1) / n - 1; };
        constexpr int DPL = D / 32;
        for (int p = p0 + warp; p < p1; p += NW) {
            const int ps = p * wm.nbu;
            const int w0 = owner(ps), w1 = owner(ps + wm.nbu - 1);
            if (w0 == w1) continue;                         // one warp: written directly
            const int vb = c * NW;
            const int b = (int)wm.dHkv.div((uint32_t)p), kvh = p - b * a.Hkv;
            const int64_t rowbase = (int64_t)b * a.Hq + (int64_t)kvh * a.G;
            for (int h = 0; h < a.G; ++h) {
                // online merge over the pieces, 4 at a time (all loads of a chunk independent:
                // one L2 round trip per chunk; a pair rarely has more than 4 pieces)
                float M = NEG_INF, l = 0.f, o[DPL];
#pragma unroll
                for (int i = 0; i < DPL; ++i) o[i] = 0.f;
                for (int w = w0; w <= w1; w += 4) {
                    float mj[4], lj[4], oj[4][DPL];
                    bool ok[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int ww = w + u;
                        ok[u] = ww <= w1 && wm.R(vb + ww) < wm.R(vb + ww + 1);
                        mj[u] = NEG_INF;
                        lj[u] = 0.f;
#pragma unroll
                        for (int i = 0; i < DPL; ++i) oj[u][i] = 0.f;
                        if (ok[u]) {
                            const int64_t sl = 2 * (int64_t)(vb + ww) + (ww == w0 && wm.R(vb + ww) < ps ? 1 : 0);
                            const float *r = a.partials + sl * a.G * GG::REC + h * GG::REC;
                            mj[u] = __ldcg(r + D);
                            lj[u] = __ldcg(r + D + 1);
                            if constexpr (DPL == 4) {
                                const float4 x = __ldcg(reinterpret_cast<const float4 *>(r) + lane);
                                oj[u][0] = x.x; oj[u][1] = x.y; oj[u][2] = x.z; oj[u][3] = x.w;
                            } else {
#pragma unroll
                                for (int i = 0; i < DPL; ++i) oj[u][i] = __ldcg(r + lane * DPL + i);
                            }
                        }
                    }
                    float Mn = M;
#pragma unroll
                    for (int u = 0; u < 4; ++u) Mn = fmaxf(Mn, mj[u]);
                    const float sc = fast_exp2(M - Mn);      // (M = -inf on the first chunk: 0)
                    l *= sc;
#pragma unroll
                    for (int i = 0; i < DPL; ++i) o[i] *= sc;
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        if (!ok[u]) continue;
                        const float wgt = fast_exp2(mj[u] - Mn);
                        l = fmaf(lj[u], wgt, l);
#pragma unroll
                        for (int i = 0; i < DPL; ++i) o[i] = fmaf(oj[u][i], wgt, o[i]);
                    }
                    M = Mn;
                }
                const float il = __frcp_rn(l);
                const int64_t row = rowbase + h;
                if (a.out_f16) {
#pragma unroll
                    for (int i = 0; i < DPL; ++i)
                        static_cast<__half *>(a.out)[row * D + lane * DPL + i] = __float2half_rn(o[i] * il);
                } else if constexpr (DPL == 4) {
                    reinterpret_cast<float4 *>(static_cast<float *>(a.out) + row * D)[lane] =
                        make_float4(o[0] * il, o[1] * il, o[2] * il, o[3] * il);
                } else {
#pragma unroll
                    for (int i = 0; i < DPL; ++i) static_cast<float *>(a.out)[row * D + lane * DPL + i] = o[i] * il;
                }
            }
        }
    }
#if LMO_ATTN_PROFILE
    if (lane == 0 && g_attn_prof) {
        unsigned long long *pr = g_attn_prof + 16 * ((size_t)a.prof_slot * 148 * 64 + gw);
        unsigned smid, wid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
        pr[0] = prof_wait;
        pr[1] = clock64() - prof_t0;
        pr[2] = prof_st;
        pr[3] = ((unsigned long long)smid << 32) | ((unsigned long long)wid << 16) | (unsigned long long)prof_seg;
        pr[4] = prof_g0;
        pr[5] = prof_g1;
        pr[6] = prof_g2;
        pr[7] = gtimer();
        pr[8] = prof_gw;
        pr[9] = prof_gm;
        pr[10] = prof_gp;
        pr[11] = prof_ga;
        pr[12] = prof_gq;
        pr[13] = prof_gf;
        pr[14] = prof_gb;
        pr[15] = ((unsigned long long)prof_ce << 32) | (unsigned long long)(prof_cs & 0xffffffffull);
    }
#endif
}

#if LMO_ATTN_PROFILE
extern "C" int lmo_debug_attn_profile(void *buf) {
    return (int)cudaMemcpyToSymbol(g_attn_prof, &buf, sizeof(void *));
}
#endif

// ---------------------------------------------------------------- host side
cudaError_t launch_kv_append(const lmo_kv_cache &cache, const void *k_new, const void *v_new,
                             int n_new, int pos0, const int32_t *pos_dev, cudaStream_t st,
                             int pos_from_lens);
template <int D, int NW = kWarps, int ST = kStages>
static size_t smem_bytes(int B_prefix) {
    return bars_bytes<NW, ST>() + (size_t)NW * ST * Geo<D>::STAGE + (B_prefix > 0 ? (B_prefix + 1) * sizeof(int) : 0);
}


// SM teams: one CTA of kSmWarps warps per SM (the ring fills the SM's shared memory)
#ifndef LMO_SM_WARPS
#define LMO_SM_WARPS 16
#endif
constexpr int kSmWarps = LMO_SM_WARPS;
template <int D>
static bool sm_team_ok() {
    static std::atomic<int> ok[64];   // 0 unknown, 1 yes, 2 no (idempotent once-per-device probe)
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (ok[dev].load(std::memory_order_acquire) == 0) {
        int n = 0, n1 = 0;
        const int sz = (int)smem_bytes<D, kSmWarps>(0);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, true, kSmWarps>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, false, kSmWarps>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, decode_attn_q4_kernel<D, true, kSmWarps>, kSmWarps * 32, sz);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n1, decode_attn_q4_kernel<D, false, kSmWarps>, kSmWarps * 32, sz);
        ok[dev].store((n >= 1 && n1 >= 1) ? 1 : 2, std::memory_order_release);
        cudaGetLastError();
    }
    return ok[dev].load(std::memory_order_acquire) == 1;
}

template <int D>
static int ctas_per_sm(int B_prefix, bool mha) {   // (MHA and GQA instances differ in registers)
    static std::atomic<int> occ[64][2][2];   // idempotent once-per-device occupancy probe
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    const int mode = B_prefix > 0 ? 1 : 0;
    if (occ[dev][mode][mha].load(std::memory_order_acquire) == 0) {
        const int sz = (int)smem_bytes<D>(kMaxBatchSmem);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, true, kWarps, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, false, kWarps, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, true, kWarps, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, false, kWarps, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, true, kWarps, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        cudaFuncSetAttribute(decode_attn_q4_kernel<D, false, kWarps, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        int n = 0;
        const size_t smem = smem_bytes<D>(mode ? kMaxBatchSmem : 0);
        // the least occupancy over the schedule instances of this variant (same bound; SCH 0 is the largest)
        for (int k = 0; k < 3; ++k) {
            int m = 0;
            if (mha)
                cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                    &m, k == 0 ? decode_attn_q4_kernel<D, true, kWarps, 0> : k == 1 ? decode_attn_q4_kernel<D, true, kWarps, 1>
                                                                            : decode_attn_q4_kernel<D, true, kWarps, 2>,
                    kWarps * 32, smem);
            else
                cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                    &m, k == 0 ? decode_attn_q4_kernel<D, false, kWarps, 0> : k == 1 ? decode_attn_q4_kernel<D, false, kWarps, 1>
                                                                             : decode_attn_q4_kernel<D, false, kWarps, 2>,
                    kWarps * 32, smem);
            if (k == 0 || m < n) n = m;
        }
        occ[dev][mode][mha].store(n > 0 ? n : 1, std::memory_order_release);
    }
    return occ[dev][mode][mha].load(std::memory_order_acquire);
}

// resident CTAs per SM of the deep-ring GQA instance (d = 128, uniform length)
static int deep_ctas_per_sm() {
    static std::atomic<int> occ[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (occ[dev].load(std::memory_order_acquire) == 0) {
        const int sz = (int)smem_bytes<128, kWarps, kDeepStages>(0);
        cudaFuncSetAttribute(decode_attn_q4_kernel<128, false, kWarps, 1, kDeepStages>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, sz);
        int n = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, decode_attn_q4_kernel<128, false, kWarps, 1, kDeepStages>,
                                                      kWarps * 32, sz);
        cudaGetLastError();
        occ[dev].store(n > 0 ? n : -1, std::memory_order_release);
    }
    return occ[dev].load(std::memory_order_acquire);
}

int attn_max_warps_v(int head_dim, int B_prefix, bool mha) {
    const int occ = head_dim == 64 ? ctas_per_sm<64>(B_prefix, mha) : ctas_per_sm<128>(B_prefix, mha);
    return device_sm_count() * occ * kWarps;
}

int attn_max_warps(int head_dim, int B_prefix) {   // the larger of the MHA / GQA grids (scratch sizing)
    const int a = attn_max_warps_v(head_dim, B_prefix, true), b = attn_max_warps_v(head_dim, B_prefix, false);
    return a > b ? a : b;
}


size_t attn_workspace_bytes(int B, int Hkv, int Hq, int D, int num_splits) {
    const int G = Hq / Hkv;
    const size_t counters = ((size_t)B * Hkv * sizeof(int) + 255) / 256 * 256;
    size_t slots = 2 * (size_t)attn_max_warps(D, 0);               // stream-K and team scratch
    const size_t sm_slots = 2 * (size_t)device_sm_count() * kSmWarps;  // SM teams
    if (sm_slots > slots) slots = sm_slots;
    if (num_splits > 0 && (size_t)B * Hkv * num_splits > slots) slots = (size_t)B * Hkv * num_splits;
    return counters + slots * G * (D + 4) * sizeof(float);
}

// Work distribution: persistent pair teams -- each (b, kv-head) pair is
// processed by a team of T warps of one CTA; a warp's producer runs ahead
// across the pairs it processes, so a pair boundary costs no pipeline bubble.
// T = 1 when the pairs can keep a fair share of the resident warps busy, else
// 2 or 4 (few pairs: a pair's blocks are split over more warps).  Stream-K
// (balanced block ranges with a global last-arriver merge) is kept for
// explicit use; measured slower than teams on every BASELINE config.
static int choose_team(int64_t pairs, int64_t warps) {
    for (int T = 1; T < kWarps; T *= 2)
        if ((double)pairs * T >= 0.35 * (double)warps) return T;
    return kWarps;
}

cudaError_t launch_decode_attention(const lmo_kv_cache &c, const void *q, int Hq, int len,
                                    const int32_t *lens, float softmax_scale, int num_splits,
                                    void *out, int out_f16, void *ws, cudaStream_t st,
                                    const void *k_new, const void *v_new, unsigned flags) {
    AttnArgs a;
    // LMO_STEP_CACHE_STABLE: stream the first LMO_EARLY_STAGES stages of each warp before the
    // PDL wait.  Measured (fused step, us per layer, depth 0 / 1 / 2 / 3): c2 18.0 / 18.3 / 18.0 /
    // 18.2, c3 17.5 / 17.6 / 17.6 / 19.1, c4 59.4 / 59.3 / 58.3 / 58.7, c5 37.4 / 37.9 / 37.2 /
    // 37.2 -- a full ring ahead floods HBM while the previous launch drains (c3: 4-stage pairs).
    a.early = (flags & LMO_STEP_CACHE_STABLE) ? LMO_EARLY_STAGES : 0;
    a.flex = (k_new && (flags & LMO_STEP_FLEXGEN_EXACT)) ? 1 : 0;
    a.raw_k = static_cast<const __half *>(k_new);
    a.raw_v = static_cast<const __half *>(v_new);
    a.k_new = static_cast<const __half *>(k_new);
    a.v_new = static_cast<const __half *>(v_new);
    a.kv = c.kv;
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
#if LMO_ATTN_PROFILE
    static std::atomic<int> prof_launches{0};   // profile builds: launch i records into slot i % 16
    a.prof_slot = prof_launches.fetch_add(1) % 16;
#else
    a.prof_slot = 0;
#endif
    const size_t counters = ((size_t)c.batch * c.kv_heads * sizeof(int) + 255) / 256 * 256;
    a.counters = static_cast<int *>(ws);
    a.partials = reinterpret_cast<float *>(static_cast<uint8_t *>(ws) + counters);

    const int D = c.head_dim;
    const int Bp = lens ? c.batch : 0;
    const int max_ctas = attn_max_warps_v(D, Bp, a.G == 1) / kWarps;
    const int64_t pairs = (int64_t)c.batch * c.kv_heads;
    const int64_t nbu = lens ? 0 : (len + kBlk - 1) / kBlk;
    a.team = 0;
    bool sm = false;                          // SM teams (uniform length only)
    const bool sm_able = !lens && (D == 64 ? sm_team_ok<64>() : sm_team_ok<128>());
    if (num_splits == LMO_SPLITS_SMTEAM) {
        a.num_splits = num_splits = 0;
        sm = sm_able;
        if (!sm) a.team = choose_team(pairs, (int64_t)max_ctas * kWarps);
    } else if (num_splits == LMO_SPLITS_STREAMK) {
        a.num_splits = num_splits = 0;        // explicit stream-K
    } else if (num_splits == 1 || num_splits == 2 || num_splits == 4) {
        a.team = num_splits;                  // explicit team size (batch-independent results)
        a.num_splits = 0;
    } else if (num_splits == 0) {
        a.team = choose_team(pairs, (int64_t)max_ctas * kWarps);
#ifdef LMO_EXPERIMENTS
        static const char *sched = getenv("LMO_ATTN_SCHED");   // experiments: streamk | sm | team1|2|4
        if (sched && !strcmp(sched, "streamk")) a.team = 0;
        if (sched && !strcmp(sched, "sm") && sm_able) { a.team = 0; sm = true; }
        if (sched && sched[0] == 't') a.team = atoi(sched + 4);
#endif
    }
    if (a.k_new && !a.team && (lens || a.num_splits > 0)) {
        // fixed splits, or stream-K over per-sequence lengths: append with its own kernel first
        const cudaError_t e = launch_kv_append(c, k_new, v_new, 1, len - 1, lens, st, /*pos_from_lens=*/1);
        if (e != cudaSuccess) return e;
        a.k_new = a.v_new = nullptr;
        // the append kernel just enqueued writes slot L-1: the attention kernel must not
        // read any stage before griddepcontrol.wait (the early prologue only holds back
        // the append slot when it does the append itself)
        a.early = 0;
    }
    // Deep-ring GQA instance (measured): GQA at d = 128 with uniform length and
    // the automatic schedule, when the pairs fill more than one warp per SMSP of the default
    // grid but at most one warp each of a 2-CTA/SM grid (c5: 1024 pairs) -- T = 1 on a grid of
    // kDeepStages-deep rings, twice the bytes in flight per busy warp.
    bool deep = false;
    if (D == 128 && a.G > 1 && !lens && num_splits == 0 && !sm && a.team == 1 && LMO_DEEP_GQA) {
        const int occ = deep_ctas_per_sm();
        if (occ > 0 && pairs > (int64_t)max_ctas * kWarps / 4 && pairs <= (int64_t)device_sm_count() * occ * kWarps)
            deep = true;
    }
    int64_t want_warps;
    if (deep) {
        want_warps = (int64_t)device_sm_count() * deep_ctas_per_sm() * kWarps;
    } else if (a.team) {
        want_warps = (int64_t)max_ctas * kWarps;          // all CTAs; idle teams exit at once

#ifdef LMO_EXPERIMENTS
        static const char *tight = getenv("LMO_ATTN_TIGHT");   // experiments: grid = teams
        if (tight && tight[0] == '1') want_warps = pairs * a.team;
#endif
    } else if (lens) {
        want_warps = (int64_t)max_ctas * kWarps;
    } else {
        const int64_t N = pairs * nbu;
        want_warps = num_splits > 0 ? pairs * num_splits : N;
    }
    // Small batches (teams of T > 1, every team at most one pair, <= 2 working CTAs per SM):
    // cap the resident CTAs at 2 per SM (padded shared memory).  With 4 per SM and
    // programmatic dependent launch, the next launch's low CTA ids -- the ones with work --
    // land 2-4 to an SM in the slots the previous launch's idle CTAs free, leaving other SMs
    // idle (timeline: 128 working CTAs on 70 SMs); with 2 per SM a launch with <= 148
    // working CTAs gets one SM each and a landing slot for the next launch on every SM
    // (c5 at batch 16: 21.7 -> 14.4 us, c2 at batch 4: 10.9 -> 7.7 us).
    size_t pad_smem = 0;
    int64_t cap_ctas = max_ctas;
    const int64_t need_ctas = (pairs * a.team + kWarps - 1) / kWarps;
    const int per_sm_cap = LMO_SMALL_CTAS_PER_SM;
    const bool small = per_sm_cap > 0 && a.team > 1 && pairs <= (int64_t)max_ctas * kWarps / a.team &&
                       need_ctas <= (int64_t)device_sm_count() * per_sm_cap && per_sm_cap < max_ctas / device_sm_count();
    if (small) {
        cap_ctas = (int64_t)device_sm_count() * per_sm_cap;
        const size_t per_sm = 228 * 1024, want = per_sm / per_sm_cap - 2048;
        const size_t base = D == 64 ? smem_bytes<64>(Bp) : smem_bytes<128>(Bp);
        if (want > base) pad_smem = want - base;
        if (want_warps > cap_ctas * kWarps) want_warps = cap_ctas * kWarps;
    }
    int64_t ctas = (want_warps + kWarps - 1) / kWarps;
    if (ctas > cap_ctas && !deep) ctas = cap_ctas;
    if (ctas < 1) ctas = 1;
    // MHA launches in the same regime (T = 1, about one pair per warp of a 2-CTA/SM grid, c2's
    // 1024 pairs): launch 2 CTAs per SM of the default instance -- the free shared memory lets
    // the next PDL launch's CTAs become resident (and prefetch) beside them (c2 step 0.597 ->
    // 0.584 ms; c3, with more pairs than warps, loses: not applied there)
    if (!deep && LMO_HALF_GRID_MHA && a.G == 1 && a.team == 1 && !lens && num_splits == 0 && !sm &&
        pairs > (int64_t)max_ctas * kWarps / 4 && pairs <= (int64_t)device_sm_count() * 2 * kWarps &&
        max_ctas >= device_sm_count() * 4)
        ctas = device_sm_count() * 2;
#ifdef LMO_EXPERIMENTS
    static const char *cap_env = getenv("LMO_ATTN_MAX_CTAS");   // tuning / experiments only
    if (cap_env && atoi(cap_env) > 0 && ctas > atoi(cap_env)) ctas = atoi(cap_env);
#endif
    const int NW = sm ? kSmWarps : kWarps;
    if (sm) ctas = device_sm_count();
    {   // the work map (uniform-length fields; per-sequence ones are completed on device)
        WorkMap &wm = a.wm;
        wm.prefix = nullptr;
        wm.B = c.batch;
        wm.Hkv = c.kv_heads;
        wm.k = a.num_splits;
        wm.W = (int)ctas * NW;
        wm.nbu = lens ? 0 : (int)nbu;
        wm.N = lens ? 0 : (int)(pairs * nbu);
        wm.V = wm.k == 0 ? (wm.N < wm.W ? wm.N : wm.W) : (int)pairs * wm.k;
        wm.T = a.team;
        wm.n_teams = a.team ? wm.W / a.team : 0;
        wm.tsh = a.team == 4 ? 2 : a.team == 2 ? 1 : 0;
        wm.dHkv = FastDiv((uint32_t)c.kv_heads);
        wm.sm = sm ? 1 : 0;
        wm.P = (int)pairs;
        wm.C = (int)ctas;
        wm.NW = NW;
        if (sm) wm.V = wm.W;
    }
#ifdef LMO_EXPERIMENTS
    static const char *ed = getenv("LMO_EARLY_DEPTH");   // experiments: stages streamed before the wait
    if (ed && a.early) a.early = atoi(ed);
#endif
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)ctas);
    cfg.blockDim = dim3(NW * 32);
    cfg.dynamicSmemBytes = sm ? (D == 64 ? smem_bytes<64, kSmWarps>(0) : smem_bytes<128, kSmWarps>(0))
                         : deep ? smem_bytes<128, kWarps, kDeepStages>(0)
                              : (D == 64 ? smem_bytes<64>(Bp) : smem_bytes<128>(Bp)) + pad_smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const bool mha = a.G == 1;
    cudaError_t e;
    if (sm)
        e = D == 64 ? (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, true, kSmWarps>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, false, kSmWarps>, a))
                    : (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, true, kSmWarps>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, false, kSmWarps>, a));
    else if (deep)
        e = cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, false, kWarps, 1, kDeepStages>, a);
    else if (a.team == 1 && !LMO_NO_SCH)
        e = D == 64 ? (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, true, kWarps, 1>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, false, kWarps, 1>, a))
                    : (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, true, kWarps, 1>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, false, kWarps, 1>, a));
    else if (a.team > 1 && !LMO_NO_SCH && pairs <= (int64_t)a.wm.n_teams)
        e = D == 64 ? (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, true, kWarps, 2>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, false, kWarps, 2>, a))
                    : (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, true, kWarps, 2>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, false, kWarps, 2>, a));
    else
        e = D == 64 ? (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, true, kWarps>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<64, false, kWarps>, a))
                    : (mha ? cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, true, kWarps>, a)
                           : cudaLaunchKernelEx(&cfg, decode_attn_q4_kernel<128, false, kWarps>, a));
    if (e != cudaSuccess) return e;
    note_launch();
    return cudaGetLastError();
}

}  // namespace lmo
