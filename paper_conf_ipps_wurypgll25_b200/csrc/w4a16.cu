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
// 64-element steps (one quantization group = one 128-B swizzle atom):
//   warps 0-7 (256 threads)  producers: cp.async of the raw codes / meta / x
//                            kRaw steps ahead into a staging ring; dequant of
//                            their row-half into the SWIZZLE_128B K-major A
//                            stage; x copy into the B stage; then the epilogue
//                            (warps 0-3: TMEM lanes = output rows)
//   warp 8                   TMEM allocation, one elected lane issues
//                            tcgen05.mma (4 x K=16 per step) and commits the
//                            stage back to the producers.
// Split-K (grid.y) accumulates fp32 partial tiles with red.global.add.
#include "common.cuh"

namespace lmo {

namespace w4 {
constexpr int kM = 128;          // output features per CTA (UMMA M)
constexpr int kK = 64;           // K per stage (one group, one swizzle atom of fp16)
constexpr int kStages = 3;       // A/B operand stages
constexpr int kRaw = 4;          // cp.async staging depth (steps in flight)
constexpr int kProd = 256;       // producer threads
constexpr int kThreads = kProd + 32;

template <int BN>
struct Smem {
    static constexpr int A = kM * 128;                 // 16 KB
    static constexpr int B = BN * 128;                 // BN x 64 fp16
    static constexpr int STAGE = A + B;
    static constexpr int RAW_CODES = kM * 32;          // 4 KB
    static constexpr int RAW_META = kM * 8;          // one copy per row-half (thread-private)
    static constexpr int RAW_X = BN * 128;
    static constexpr int RAW = RAW_CODES + RAW_META + RAW_X;
    static constexpr int BYTES = kStages * STAGE + kRaw * RAW + 1024 /* align */ + 256 /* barriers */;
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
// byte is read in place as 1024 + 16c and scaled by scale/16.
__device__ __forceinline__ uint4 deq8(uint32_t w, __half2 sc, __half2 sc16, __half2 mn) {
    const __half2 k1024 = __half2half2(__ushort_as_half(0x6400));
    const uint32_t s8 = w >> 8;
    const uint32_t t0 = lop3_and_or(w, 0x000F000Fu, 0x64006400u);    // (c0, c4) + 1024
    const uint32_t t1 = lop3_and_or(w, 0x00F000F0u, 0x64006400u);    // 16 (c1, c5) + 1024
    const uint32_t t2 = lop3_and_or(s8, 0x000F000Fu, 0x64006400u);   // (c2, c6) + 1024
    const uint32_t t3 = lop3_and_or(s8, 0x00F000F0u, 0x64006400u);   // 16 (c3, c7) + 1024
    auto f = [&](uint32_t t, __half2 s) {
        const __half2 c = __hsub2(*reinterpret_cast<const __half2 *>(&t), k1024);
        const __half2 r = __hfma2(c, s, mn);
        return *reinterpret_cast<const uint32_t *>(&r);
    };
    const uint32_t p0 = f(t0, sc), p1 = f(t1, sc16), p2 = f(t2, sc), p3 = f(t3, sc16);
    return make_uint4(prmt(p0, p1, 0x5410u), prmt(p2, p3, 0x5410u), prmt(p0, p1, 0x7632u),
                      prmt(p2, p3, 0x7632u));
}

template <int BN>
__global__ void __launch_bounds__(kThreads, 1)
w4a16_kernel(const uint8_t *__restrict__ codes, const uint32_t *__restrict__ meta,
             const __half *__restrict__ x, float *__restrict__ y, int N, int K, int batch,
             int ksplit) {
    using S = Smem<BN>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *stages = smem;                                   // [kStages][A | B]
    uint8_t *raw = smem + kStages * S::STAGE;                 // [kRaw][codes | meta | x]
    uint64_t *bars = reinterpret_cast<uint64_t *>(raw + kRaw * S::RAW);
    uint64_t *full = bars, *empty = bars + kStages, *done = bars + 2 * kStages;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 2 * kStages + 1);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int n0 = blockIdx.x * kM;
    const int KB = K / kK;
    const int kb0 = (int)((long long)blockIdx.y * KB / ksplit), kb1 = (int)((long long)(blockIdx.y + 1) * KB / ksplit);
    const int nsteps = kb1 - kb0;
    constexpr int TCOLS = BN < 32 ? 32 : BN;                  // TMEM columns (power of 2 >= 32)

    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], kProd);
            mbar_init(&empty[s], 1);
        }
        mbar_init(done, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == kProd / 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                     "n"(TCOLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    const uint32_t tmem = *tmem_slot;

    if (tid < kProd) {
        // ------------------------------------------------------------ producers
        const int r = tid & (kM - 1), h = tid >> 7;             // row of the tile, half of the group
        const uint8_t *crow = codes + (int64_t)(n0 + r) * (K / 2) + h * 16;
        const uint32_t *mrow = meta + (int64_t)(n0 + r) * (K / kK);
        const uint32_t raw_u32 = smem_u32(raw);
        auto issue = [&](int j) {   // step j's raw data -> staging slot j % kRaw
            if (j < nsteps) {
                const int kb = kb0 + j;
                const uint32_t base = raw_u32 + (j % kRaw) * S::RAW;
                cp_async16(base + r * 32 + h * 16, crow + (int64_t)kb * 32, 16);
                cp_async4(base + S::RAW_CODES + (h * kM + r) * 4, mrow + kb);
                for (int c = tid; c < BN * 8; c += kProd) {       // x rows (zero beyond batch)
                    const int xr = c >> 3, xc = c & 7;
                    const bool ok = xr < batch;
                    const __half *src = x + (int64_t)(ok ? xr : 0) * K + kb * kK + xc * 8;
                    cp_async16(base + S::RAW_CODES + S::RAW_META + c * 16, src, ok ? 16 : 0);
                }
            }
            cp_commit();
        };
        for (int j = 0; j < kRaw - 1; ++j) issue(j);
        for (int j = 0; j < nsteps; ++j) {
            issue(j + kRaw - 1);
            cp_wait<kRaw - 1>();                                 // this thread's copies of step j
            const int st = j % kStages;
            if (j >= kStages) mbar_wait(&empty[st], ((j / kStages) - 1) & 1);
            const uint8_t *rs = raw + (j % kRaw) * S::RAW;
            uint8_t *A = stages + st * S::STAGE;
            uint8_t *Bs = A + S::A;
            // dequantize this thread's 32 weights (row r, k = 32h .. 32h+31)
            const uint4 cw = *reinterpret_cast<const uint4 *>(rs + r * 32 + h * 16);
            const uint32_t mw = *reinterpret_cast<const uint32_t *>(rs + S::RAW_CODES + (h * kM + r) * 4);
            const __half mnh = __ushort_as_half((unsigned short)(mw & 0xFFFFu));
            const __half sch = __ushort_as_half((unsigned short)(mw >> 16));
            const __half2 mn2 = __half2half2(mnh), sc2 = __half2half2(sch);
            const __half2 sc16 = __hmul2(sc2, __half2half2(__float2half_rn(0.0625f)));
            const uint32_t words[4] = {cw.x, cw.y, cw.z, cw.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const uint4 v = deq8(words[i], sc2, sc16, mn2);
                const int chunk = (h * 4 + i) ^ (r & 7);                 // SWIZZLE_128B
                *reinterpret_cast<uint4 *>(A + r * 128 + chunk * 16) = v;
            }
            // activations: raw [BN][8 chunks] -> swizzled B stage
            for (int c = tid; c < BN * 8; c += kProd) {
                const int xr = c >> 3, xc = c & 7;
                const uint4 v = *reinterpret_cast<const uint4 *>(rs + S::RAW_CODES + S::RAW_META + c * 16);
                *reinterpret_cast<uint4 *>(Bs + xr * 128 + ((xc ^ (xr & 7)) * 16)) = v;
            }
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            mbar_arrive(&full[st]);
        }
        cp_wait<0>();
    } else {
        // ------------------------------------------------------------ MMA issuer
        constexpr uint32_t idesc = umma_idesc<BN>();
        for (int j = 0; j < nsteps; ++j) {
            const int st = j % kStages;
            mbar_wait(&full[st], (j / kStages) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
            if (lane == 0) {
                const uint32_t a0 = smem_u32(stages + st * S::STAGE), b0 = a0 + S::A;
#pragma unroll
                for (int k = 0; k < kK / 16; ++k) {
                    const uint64_t da = umma_desc(a0 + k * 32), db = umma_desc(b0 + k * 32);
                    const uint32_t acc = (j > 0 || k > 0) ? 1u : 0u;
                    asm volatile(
                        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem),
                        "l"(da), "l"(db), "r"(idesc), "r"(acc));
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(&empty[st]))
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
    if (warp < 4) {
        const int row = warp * 32 + lane;                        // TMEM lane = output feature
        if (nsteps > 0) {
            mbar_wait(done, 0);
            asm volatile("tcgen05.fence::after_thread_sync;\n");
        }
#pragma unroll
        for (int c0 = 0; c0 < BN; c0 += 32) {
            uint32_t v[32];
            const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + c0;
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
                    if (ksplit > 1) atomicAdd(dst, val);
                    else *dst = val;
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    if (warp == kProd / 32) {
        asm volatile("tcgen05.fence::after_thread_sync;\n");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "n"(TCOLS));
    }
}

}  // namespace w4

int w4a16_auto_split(int N, int K) {
    const int tiles = N / w4::kM, KB = K / w4::kK;
    const int sms = device_sm_count();
    int s = 1;
    while (tiles * s < sms && s * 2 <= KB / 4) s *= 2;   // fill the SMs, keep >= 4 groups per split
    return s;
}

cudaError_t launch_w4a16(const uint8_t *codes, const void *meta, const void *x, float *y, int N, int K,
                         int batch, int ksplit, cudaStream_t st) {
    if (ksplit <= 0) ksplit = w4a16_auto_split(N, K);
    if (ksplit > K / w4::kK) ksplit = K / w4::kK;
    if (ksplit > 1) {
        const cudaError_t e = cudaMemsetAsync(y, 0, (size_t)batch * N * sizeof(float), st);
        if (e != cudaSuccess) return e;
    }
    dim3 grid(N / w4::kM, ksplit);
    cudaError_t e;
    if (batch <= 64) {
        const int sm = w4::Smem<64>::BYTES;
        cudaFuncSetAttribute(w4::w4a16_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        w4::w4a16_kernel<64><<<grid, w4::kThreads, sm, st>>>(codes, static_cast<const uint32_t *>(meta),
                                                              static_cast<const __half *>(x), y, N, K, batch, ksplit);
    } else {
        const int sm = w4::Smem<128>::BYTES;
        cudaFuncSetAttribute(w4::w4a16_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        w4::w4a16_kernel<128><<<grid, w4::kThreads, sm, st>>>(codes, static_cast<const uint32_t *>(meta),
                                                               static_cast<const __half *>(x), y, N, K, batch, ksplit);
    }
    e = cudaGetLastError();
    if (e == cudaSuccess) note_launch();
    return e;
}

}  // namespace lmo
