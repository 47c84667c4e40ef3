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
// blockIdx.y: 0 = K, 1 = V; 4 lanes per 64-group, grid-stride over (row, group).
__global__ void __launch_bounds__(256) kv_append_kernel(lmo_kv_cache cache,
                                                        const __half *__restrict__ k_new,
                                                        const __half *__restrict__ v_new,
                                                        int n_new, int pos0,
                                                        const int32_t *__restrict__ pos_dev,
                                                        int pos_from_lens) {
    asm volatile("griddepcontrol.wait;\n" ::: "memory");   // PDL: inputs of earlier kernels
    const int d = cache.head_dim;
    const int gpr = d / kGroup;
    const int RB = d / 2, MB = gpr * 4, ROW = 2 * (RB + MB);
    const int kv = blockIdx.y;
    const __half *srcbase = kv == 0 ? k_new : v_new;
    const int lane4 = threadIdx.x & 3;
    const int rows = cache.batch * cache.kv_heads * n_new;     // (b*Hkv + h)*n_new + t
    const int ngroups = rows * gpr;
    const int stride = gridDim.x * (blockDim.x / 4);
    for (int g0 = blockIdx.x * (blockDim.x / 4); g0 < ngroups; g0 += stride) {
        const int gid = g0 + (threadIdx.x >> 2);
        bool valid = gid < ngroups;
        const int r = valid ? gid / gpr : 0;
        const int grp = gid - r * gpr;
        const int bh = r / n_new;
        const int t = r - bh * n_new;
        const int b = bh / cache.kv_heads;
        int pos = pos_dev ? pos_dev[b] : pos0;
        if (pos_dev && pos_from_lens) pos = min(pos, cache.capacity) - 1;   // new token at L_b - 1
        if (pos < 0 || pos + n_new > cache.capacity) valid = false;
        uint4 xa = make_uint4(0, 0, 0, 0), xb = xa;
        if (valid) {
            const __half *src = srcbase + (int64_t)r * d + grp * kGroup + lane4 * 16;
            xa = ldg_stream(src);
            xb = ldg_stream(src + 8);
        }
        uint32_t mw;
        const uint2 w = quantize_group_lane4(xa, xb, mw);
        if (valid) {
            // compressed row: K codes | K meta | V codes | V meta
            const int64_t slot = (int64_t)bh * cache.capacity + pos + t;
            uint8_t *row = cache.kv + slot * ROW + kv * (RB + MB);
            // the V half of a d=64 row starts at byte 36: only 4-byte alignment holds
            uint32_t *dst = reinterpret_cast<uint32_t *>(row + grp * 32 + lane4 * 8);
            dst[0] = w.x;
            dst[1] = w.y;
            if (lane4 == 0) reinterpret_cast<uint32_t *>(row + RB)[grp] = mw;
        }
    }
}

__device__ __forceinline__ __half dequant_one(uint32_t c, uint32_t mw) {
    const float mn = __half2float(__ushort_as_half((unsigned short)(mw & 0xffffu)));
    const float sc = __half2float(__ushort_as_half((unsigned short)(mw >> 16)));
    return __float2half_rn(__fmaf_rn((float)c, sc, mn));   // RN16(RN32(c*scale + min))
}

// K5 fast path: inner == 1, n % 64 == 0; 16 elements (8 code bytes in, 32 B out)
// per thread, grid-stride.
__global__ void __launch_bounds__(256) dequantize_vec_kernel(const uint8_t *__restrict__ codes,
                                                             const uint32_t *__restrict__ meta,
                                                             int64_t n_hex,
                                                             __half *__restrict__ y) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n_hex; idx += stride) {
        const uint2 w = __ldg(reinterpret_cast<const uint2 *>(codes) + idx);
        const uint32_t mw = __ldg(meta + idx / 4);
        const float mn = __half2float(__ushort_as_half((unsigned short)(mw & 0xffffu)));
        const float sc = __half2float(__ushort_as_half((unsigned short)(mw >> 16)));
        uint4 out[2];
        uint32_t *o = reinterpret_cast<uint32_t *>(out);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t word = k < 4 ? w.x : w.y;
            const int sh = 8 * (k & 3);
            // code -> float exactly via the 2^23 magic (0x4B000000 | c) - 2^23
            const float c0 = __uint_as_float(0x4B000000u | ((word >> sh) & 0xfu)) - 8388608.0f;
            const float c1 = __uint_as_float(0x4B000000u | ((word >> (sh + 4)) & 0xfu)) - 8388608.0f;
            const __half lo = __float2half_rn(__fmaf_rn(c0, sc, mn));   // RN16(RN32(c*scale + min))
            const __half hi = __float2half_rn(__fmaf_rn(c1, sc, mn));
            o[k] = (uint32_t)__half_as_ushort(lo) | ((uint32_t)__half_as_ushort(hi) << 16);
        }
        uint4 *dst = reinterpret_cast<uint4 *>(y) + 2 * idx;
        dst[0] = out[0];
        dst[1] = out[1];
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
        const int64_t n_hex = outer * n / 16;
        dequantize_vec_kernel<<<grid_for(n_hex, 256), 256, 0, st>>>(codes, mw, n_hex, yh);
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
    const int64_t groups = (int64_t)cache.batch * cache.kv_heads * n_new * (cache.head_dim / kGroup);
    const int64_t blocks = (groups + 63) / 64;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid_for(blocks * 256, 256), 2);
    cfg.blockDim = dim3(256);
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const cudaError_t e = cudaLaunchKernelEx(&cfg, kv_append_kernel, cache,
                                             static_cast<const __half *>(k_new),
                                             static_cast<const __half *>(v_new), n_new, pos0, pos_dev,
                                             pos_from_lens);
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace lmo
