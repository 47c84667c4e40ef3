// quant.cu -- K1 group-wise quantize (Alg 2 / Eq 10), K2 KV append-quantize
// (Eq 7), K5 group-wise dequantize (Eq 11).  sm_100a.
//
// All three are HBM-streaming kernels (2.5625 B/element moved for K1/K2,
// 2.5625 for K5): 128-bit coalesced loads/stores, 8 lanes per 64-group,
// warp-shuffle min/max, no shared memory.  The rounding chain lives in
// common.cuh (group_params / quant_code) and is the same for K1 and K2, so
// append is bit-identical to quantize on the same rows by construction.
#include "common.cuh"

namespace lmo {

__device__ __forceinline__ uint4 ldg_stream(const void *p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];\n"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

// K1 fast path: inner == 1, n % 64 == 0.  One 64-group per 4 lanes (16 elements
// each: two 128-bit loads in flight), grid-stride over groups.
__global__ void __launch_bounds__(256) quantize_vec_kernel(const __half *__restrict__ x,
                                                           int64_t ngroups_total,
                                                           uint8_t *__restrict__ codes,
                                                           uint32_t *__restrict__ meta) {
    const int lane4 = threadIdx.x & 3;
    const int64_t stride = (int64_t)gridDim.x * (blockDim.x / 4);
    for (int64_t g0 = (int64_t)blockIdx.x * (blockDim.x / 4); g0 < ngroups_total; g0 += stride) {
        const int64_t gid = g0 + (threadIdx.x >> 2);
        const bool valid = gid < ngroups_total;
        uint4 xa = make_uint4(0, 0, 0, 0), xb = xa;
        if (valid) {
            const __half *src = x + gid * kGroup + lane4 * 16;
            xa = ldg_stream(src);
            xb = ldg_stream(src + 8);
        }
        uint32_t mw;
        const uint2 w = quantize_group_lane4(xa, xb, mw);     // all lanes take part in shuffles
        if (valid) {
            reinterpret_cast<uint2 *>(codes + gid * (kGroup / 2))[lane4] = w;
            if (lane4 == 0) meta[gid] = mw;
        }
    }
}

// K1 general path: any (outer, n, inner); one thread per (o, group, i), i
// fastest so that inner > 1 (e.g. grouping a weight matrix along its output
// dim) is coalesced across threads.
__global__ void __launch_bounds__(256) quantize_generic_kernel(const __half *__restrict__ x,
                                                               int64_t outer, int64_t n,
                                                               int64_t inner,
                                                               uint8_t *__restrict__ codes,
                                                               uint32_t *__restrict__ meta) {
    const int64_t ng = (n + kGroup - 1) / kGroup;
    const int64_t total = outer * ng * inner;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx % inner;
        const int64_t g = (idx / inner) % ng;
        const int64_t o = idx / (inner * ng);
        float mn = INFINITY, mx = -INFINITY;
        for (int k = 0; k < kGroup; ++k) {
            const int64_t j = g * kGroup + k;
            const float v = (j < n) ? __half2float(x[(o * n + j) * inner + i]) : 0.0f;
            mn = fminf(mn, v);
            mx = fmaxf(mx, v);
        }
        const GroupParams p = group_params(mn, mx);
        const int64_t npad2 = ng * kGroup / 2;
        for (int k = 0; k < kGroup; k += 2) {
            const int64_t j = g * kGroup + k;
            const float v0 = (j < n) ? __half2float(x[(o * n + j) * inner + i]) : 0.0f;
            const float v1 = (j + 1 < n) ? __half2float(x[(o * n + j + 1) * inner + i]) : 0.0f;
            codes[(o * npad2 + j / 2) * inner + i] =
                (uint8_t)(quant_code(v0, p) | (quant_code(v1, p) << 4));
        }
        meta[(o * ng + g) * inner + i] = meta_word(p);
    }
}

// K2: quantize new K/V rows [B][Hkv][n_new][d] into cache slots pos_b + t.
// 4 lanes per 64-group, grid-stride over (row, K|V, group) units.
__global__ void __launch_bounds__(256) kv_append_kernel(lmo_kv_cache cache,
                                                        const __half *__restrict__ k_new,
                                                        const __half *__restrict__ v_new,
                                                        int n_new, FastDiv div_n, FastDiv div_h,
                                                        int pos0,
                                                        const int32_t *__restrict__ pos_dev,
                                                        int pos_from_lens) {
    asm volatile("griddepcontrol.wait;\n" ::: "memory");   // PDL: inputs of earlier kernels
    const int d = cache.head_dim;
    const int gpr = d / kGroup;
    const int RB = d / 2, MB = gpr * 4, ROW = 2 * (RB + MB);
    // unit u = (row r, half kv, group grp), kv-major inside a row so that a warp's 8
    // units cover whole compressed rows (K codes|K meta|V codes|V meta) contiguously
    const int lane4 = threadIdx.x & 3;
    const int upr = 2 * gpr;                                   // units per row
    const int nunits = cache.batch * cache.kv_heads * n_new * upr;
    const int stride = gridDim.x * (blockDim.x / 4);
    for (int u0 = blockIdx.x * (blockDim.x / 4); u0 < nunits; u0 += stride) {
        const int u = u0 + (threadIdx.x >> 2);
        bool valid = u < nunits;
        const int r = valid ? (u >> gpr) : 0;                  // upr = 2*gpr = 2 or 4: shift by gpr
        const int within = u - r * upr;                        // r = (b*Hkv + h)*n_new + t
        const int kv = within >= gpr;
        const int grp = within - kv * gpr;
        const int bh = (int)div_n.div((uint32_t)r);
        const int t = r - bh * n_new;
        const int b = (int)div_h.div((uint32_t)bh);
        int pos = pos_dev ? pos_dev[b] : pos0;
        if (pos_dev && pos_from_lens) pos = min(pos, cache.capacity) - 1;   // new token at L_b - 1
        if (pos < 0 || pos + n_new > cache.capacity) valid = false;
        uint4 xa = make_uint4(0, 0, 0, 0), xb = xa;
        if (valid) {
            const __half *src = (kv ? v_new : k_new) + (int64_t)r * d + grp * kGroup + lane4 * 16;
            xa = ldg_stream(src);
            xb = ldg_stream(src + 8);
        }
        uint32_t mw;
        const uint2 w = quantize_group_lane4(xa, xb, mw);
        if (valid) {
            const int64_t slot = (int64_t)bh * cache.capacity + pos + t;
            uint8_t *row = cache.kv + slot * ROW + kv * (RB + MB);
            if (kv == 0) {
                uint32_t *dst = reinterpret_cast<uint32_t *>(row + grp * 32 + lane4 * 8);
                dst[0] = w.x;
                dst[1] = w.y;
            } else {   // V codes: pair-interleaved 16-bit chunks (common.cuh, include/lmo.h)
                const int tok = pos + t;
                uint8_t *pr = cache.kv + ((int64_t)bh * cache.capacity + (tok & ~1)) * ROW;
                const int c = 16 * grp + 4 * lane4;
                store_v_chunk(pr, d, c, tok, w.x & 0xFFFFu);
                store_v_chunk(pr, d, c + 1, tok, w.x >> 16);
                store_v_chunk(pr, d, c + 2, tok, w.y & 0xFFFFu);
                store_v_chunk(pr, d, c + 3, tok, w.y >> 16);
            }
            if (lane4 == 0) reinterpret_cast<uint32_t *>(row + RB)[grp] = mw;
        }
    }
}

__device__ __forceinline__ __half dequant_one(uint32_t c, uint32_t mw) {
    const float mn = __half2float(__ushort_as_half((unsigned short)(mw & 0xffffu)));
    const float sc = __half2float(__ushort_as_half((unsigned short)(mw >> 16)));
    return __float2half_rn(__fmaf_rn((float)c, sc, mn));   // RN16(RN32(c*scale + min))
}

// K5 fast path: inner == 1, n % 64 == 0.  One 32-bit code word (8 elements) in, one
// 16-byte fp16 vector out per thread and item; consecutive lanes take consecutive
// words so every load and store instruction is fully coalesced; 4 items per thread
// in flight, grid-stride over tiles of 4*blockDim words.
__global__ void __launch_bounds__(256) dequantize_vec_kernel(const uint32_t *__restrict__ codes,
                                                             const uint32_t *__restrict__ meta,
                                                             int64_t n_words,
                                                             uint4 *__restrict__ y) {
    constexpr int kItems = 4;
    const int64_t tile = (int64_t)kItems * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * tile; base < n_words; base += (int64_t)gridDim.x * tile) {
        uint32_t w[kItems], mw[kItems];
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            const int64_t i = base + j * blockDim.x + threadIdx.x;
            w[j] = i < n_words ? __ldcs(codes + i) : 0u;
            mw[j] = i < n_words ? __ldg(meta + i / 8) : 0u;    // 8 words per 64-group
        }
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            const int64_t i = base + j * blockDim.x + threadIdx.x;
            const float mn = __half2float(__ushort_as_half((unsigned short)(mw[j] & 0xffffu)));
            const float sc = __half2float(__ushort_as_half((unsigned short)(mw[j] >> 16)));
            uint32_t o[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                // code -> float exactly via the 2^23 magic (0x4B000000 | c) - 2^23
                const float c0 = __uint_as_float(0x4B000000u | ((w[j] >> (8 * k)) & 0xfu)) - 8388608.0f;
                const float c1 = __uint_as_float(0x4B000000u | ((w[j] >> (8 * k + 4)) & 0xfu)) - 8388608.0f;
                const __half lo = __float2half_rn(__fmaf_rn(c0, sc, mn));   // RN16(RN32(c*scale + min))
                const __half hi = __float2half_rn(__fmaf_rn(c1, sc, mn));
                o[k] = (uint32_t)__half_as_ushort(lo) | ((uint32_t)__half_as_ushort(hi) << 16);
            }
            if (i < n_words) __stcs(y + i, make_uint4(o[0], o[1], o[2], o[3]));
        }
    }
}

// K5 general path: one thread per output element.
__global__ void __launch_bounds__(256) dequantize_generic_kernel(const uint8_t *__restrict__ codes,
                                                                 const uint32_t *__restrict__ meta,
                                                                 int64_t outer, int64_t n,
                                                                 int64_t inner,
                                                                 __half *__restrict__ y) {
    const int64_t ng = (n + kGroup - 1) / kGroup;
    const int64_t npad2 = ng * kGroup / 2;
    const int64_t total = outer * n * inner;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx % inner;
        const int64_t j = (idx / inner) % n;
        const int64_t o = idx / (inner * n);
        const uint8_t byte = codes[(o * npad2 + j / 2) * inner + i];
        const uint32_t c = (j & 1) ? (byte >> 4) : (byte & 0xf);
        y[idx] = dequant_one(c, meta[(o * ng + j / kGroup) * inner + i]);
    }
}

// ------------------------------------------------------------ host launch
static int grid_for(int64_t work, int per_block) {
    int64_t g = (work + per_block - 1) / per_block;
    const int64_t cap = (int64_t)device_sm_count() * 32;
    return (int)(g < 1 ? 1 : (g > cap ? cap : g));
}

cudaError_t launch_quantize(const void *x, int64_t outer, int64_t n, int64_t inner,
                            uint8_t *codes, lmo_qmeta *meta, cudaStream_t st) {
    const __half *xh = static_cast<const __half *>(x);
    uint32_t *mw = reinterpret_cast<uint32_t *>(meta);
    if (inner == 1 && n % kGroup == 0) {
        const int64_t groups = outer * (n / kGroup);
        const int64_t blocks = (groups + 63) / 64;
        quantize_vec_kernel<<<grid_for(blocks * 256, 256), 256, 0, st>>>(xh, groups, codes, mw);
    } else {
        const int64_t work = outer * ((n + kGroup - 1) / kGroup) * inner;
        quantize_generic_kernel<<<grid_for(work, 256), 256, 0, st>>>(xh, outer, n, inner, codes,
                                                                       mw);
    }
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_dequantize(const uint8_t *codes, const lmo_qmeta *meta, int64_t outer,
                              int64_t n, int64_t inner, void *y, cudaStream_t st) {
    const uint32_t *mw = reinterpret_cast<const uint32_t *>(meta);
    __half *yh = static_cast<__half *>(y);
    if (inner == 1 && n % kGroup == 0) {
        const int64_t n_words = outer * n / 8;
        dequantize_vec_kernel<<<grid_for((n_words + 3) / 4, 256), 256, 0, st>>>(
            reinterpret_cast<const uint32_t *>(codes), mw, n_words, reinterpret_cast<uint4 *>(yh));
    } else {
        dequantize_generic_kernel<<<grid_for(outer * n * inner, 256), 256, 0, st>>>(
            codes, mw, outer, n, inner, yh);
    }
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_kv_append(const lmo_kv_cache &cache, const void *k_new, const void *v_new,
                             int n_new, int pos0, const int32_t *pos_dev, cudaStream_t st,
                             int pos_from_lens) {
    const int64_t units = 2LL * cache.batch * cache.kv_heads * n_new * (cache.head_dim / kGroup);
    const int64_t blocks = (units + 63) / 64;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid_for(blocks * 256, 256));
    cfg.blockDim = dim3(256);
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const cudaError_t e = cudaLaunchKernelEx(&cfg, kv_append_kernel, cache,
                                             static_cast<const __half *>(k_new),
                                             static_cast<const __half *>(v_new), n_new,
                                             FastDiv((uint32_t)n_new),
                                             FastDiv((uint32_t)cache.kv_heads), pos0, pos_dev,
                                             pos_from_lens);
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace lmo
