// Microbenchmark: per-SMSP throughput of the q4 attention inner loop pieces
// (nibble unpack LOP3/SHF/PRMT, HMMA m16n8k16, LDS) on smem-resident data, vs
// warps per SMSP.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ub scripts/ubench_unpack.cu
// One CTA per SM, W warps; each warp loops ITER "stages" over its own 4.5 KB of smem.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>

__device__ __forceinline__ void mma16816(float *c, uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
    asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                 : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
                 : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
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
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t s) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(s));
    return r;
}

constexpr int ROW = 144, STAGE = 32 * ROW;

__device__ __forceinline__ void imma16832(int *c, uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                          uint32_t b0, uint32_t b1) {
    asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.u8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                 : "+r"(c[0]), "+r"(c[1]), "+r"(c[2]), "+r"(c[3])
                 : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// MODE 4: K side as u8 x s8 IMMA (2 per 32 dims: q hi/lo bytes), nibble -> byte unpack (3 ops / 8 codes);
//         V side unchanged (f16 HMMA).  MODE 5: IMMA only (16 per stage, raw words).
template <int MODE>
__global__ void __launch_bounds__(1024, 1) ubi(int iters, unsigned long long *out, float *sink) {
    extern __shared__ __align__(128) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
    for (int i = threadIdx.x; i < blockDim.x / 32 * STAGE / 4; i += blockDim.x)
        reinterpret_cast<uint32_t *>(smem)[i] = (i * 2654435761u) ^ 0x5a5a5a5au;
    __syncthreads();
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(smem + warp * STAGE);
    const uint32_t offK = base + g * ROW + 16 * t, offV = base + (2 * t) * ROW + 64 + 8 + 4 * g;
    float acc[8][4] = {};
    int ci[2][2][4] = {};
    uint32_t x = 0, qh0 = 0x01020304u + lane, qh1 = 0x05060708u, ql0 = 0x7f7f7f7fu, ql1 = 0x11223344u;
    uint32_t qf0 = 0x3c003c00u + lane, qf1 = 0x38003800u;
    __syncwarp();
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        const uint32_t st = (it & 1) * 16;
#pragma unroll
        for (int s = 0; s < 2; ++s) {
            // K: 16 tokens x 128 dims = 4 k32 slices; lane holds rows g, g+8, 16 B (32 codes) each
            const uint4 w0 = *reinterpret_cast<const uint4 *>(smem + (offK - (uint32_t)__cvta_generic_to_shared(smem)) + st + s * 16 * ROW);
            const uint4 w1 = *reinterpret_cast<const uint4 *>(smem + (offK - (uint32_t)__cvta_generic_to_shared(smem)) + st + s * 16 * ROW + 8 * ROW);
            const uint32_t ww0[4] = {w0.x, w0.y, w0.z, w0.w}, ww1[4] = {w1.x, w1.y, w1.z, w1.w};
#pragma unroll
            for (int kb = 0; kb < 4; ++kb) {
                uint32_t a0, a1, a2, a3;
                if (MODE == 4) {
                    a0 = ww0[kb] & 0x0F0F0F0Fu; a2 = (ww0[kb] >> 4) & 0x0F0F0F0Fu;
                    a1 = ww1[kb] & 0x0F0F0F0Fu; a3 = (ww1[kb] >> 4) & 0x0F0F0F0Fu;
                } else {
                    a0 = ww0[kb]; a1 = ww1[kb]; a2 = ww0[kb] + 1; a3 = ww1[kb] + 1;
                }
                imma16832(ci[s][kb >> 1], a0, a1, a2, a3, qh0, qh1);
                imma16832(ci[s][kb >> 1], a0, a1, a2, a3, ql0 + it, ql1);
            }
            if (MODE == 4) {
#pragma unroll
                for (int grp = 0; grp < 2; ++grp) {
                    const uint32_t wa0 = lds32(offV + st + s * 16 * ROW + grp * 32);
                    const uint32_t wb0 = lds32(offV + st + s * 16 * ROW + ROW + grp * 32);
                    const uint32_t wa1 = lds32(offV + st + s * 16 * ROW + 8 * ROW + grp * 32);
                    const uint32_t wb1 = lds32(offV + st + s * 16 * ROW + 9 * ROW + grp * 32);
                    uint32_t j0[8], j1[8];
                    const uint32_t pa[2] = {wa0, wa1}, pb[2] = {wb0, wb1};
                    uint32_t *jj[2] = {j0, j1};
#pragma unroll
                    for (int k = 0; k < 2; ++k) {
                        const uint32_t lo = prmt(pa[k], pb[k], 0x5410u), hi = prmt(pa[k], pb[k], 0x7632u);
                        const uint32_t lo8 = lo >> 8, hi8 = hi >> 8;
                        jj[k][0] = lo & 0x000F000Fu; jj[k][1] = lo & 0x00F000F0u;
                        jj[k][2] = lo8 & 0x000F000Fu; jj[k][3] = lo8 & 0x00F000F0u;
                        jj[k][4] = hi & 0x000F000Fu; jj[k][5] = hi & 0x00F000F0u;
                        jj[k][6] = hi8 & 0x000F000Fu; jj[k][7] = hi8 & 0x00F000F0u;
                    }
#pragma unroll
                    for (int mb = 0; mb < 4; ++mb)
                        mma16816(acc[grp * 4 + mb], j0[2 * mb], j0[2 * mb + 1], j1[2 * mb], j1[2 * mb + 1], qf0 + it, qf1);
                }
            }
        }
    }
    const long long t1 = clock64();
    float sm = (float)x;
    for (int i = 0; i < 8; ++i) sm += acc[i][0] + acc[i][1] + acc[i][2] + acc[i][3];
    for (int i = 0; i < 16; ++i) sm += (float)(&ci[0][0][0])[i];
    if (sm == 123.456f) sink[threadIdx.x] = sm;
    if (lane == 0) out[blockIdx.x * 32 + warp] = (unsigned long long)(t1 - t0);
}

// MODE 0: full K+V unpack + 32 HMMA per stage (the kernel's MHA hot loop, minus softmax)
// MODE 1: unpack only (results XOR-folded)      MODE 2: HMMA only (raw words as A)
// MODE 3: LDS only
template <int MODE>
__global__ void __launch_bounds__(1024, 1) ub(int iters, unsigned long long *out, float *sink) {
    extern __shared__ __align__(128) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
    for (int i = threadIdx.x; i < blockDim.x / 32 * STAGE / 4; i += blockDim.x)
        reinterpret_cast<uint32_t *>(smem)[i] = (i * 2654435761u) ^ 0x5a5a5a5au;
    __syncthreads();
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(smem + warp * STAGE);
    const uint32_t offK = base + g * ROW + 8 * t, offV = base + (2 * t) * ROW + 64 + 8 + 4 * g;
    float acc[8][4] = {};
    float c2[4] = {};
    uint32_t x = 0, qf0 = 0x3c003c00u + lane, qf1 = 0x38003800u;
    __syncwarp();
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        const uint32_t st = (it & 1) * 16;   // wiggle addresses a bit (stay in bounds)
#pragma unroll
        for (int s = 0; s < 2; ++s) {
#pragma unroll
            for (int grp = 0; grp < 2; ++grp) {
                const uint2 w0 = lds64(offK + st + s * 16 * ROW + grp * 32);
                const uint2 w1 = lds64(offK + st + s * 16 * ROW + 8 * ROW + grp * 32);
                uint32_t u0[8], u1[8];
                if (MODE == 0 || MODE == 1) {
                    const uint32_t ww[4] = {w0.x, w0.y, w1.x, w1.y};
                    uint32_t *uu[4] = {u0, u0 + 4, u1, u1 + 4};
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const uint32_t sh = ww[k] >> 8;
                        uu[k][0] = ww[k] & 0x000F000Fu;
                        uu[k][1] = ww[k] & 0x00F000F0u;
                        uu[k][2] = sh & 0x000F000Fu;
                        uu[k][3] = sh & 0x00F000F0u;
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < 8; ++k) { u0[k] = w0.x + k; u1[k] = w1.y + k; }
                }
                if (MODE == 0 || MODE == 2) {
#pragma unroll
                    for (int kb = 0; kb < 4; ++kb)
                        mma16816(c2, u0[2 * kb], u1[2 * kb], u0[2 * kb + 1], u1[2 * kb + 1], qf0, qf1);
                } else if (MODE == 1) {
#pragma unroll
                    for (int k = 0; k < 8; ++k) x ^= u0[k] + u1[k];
                } else {
                    x ^= w0.x ^ w1.y ^ w0.y ^ w1.x;
                }
                // V side: 4 words (2 token pairs) -> 16 A registers
                const uint32_t wa0 = lds32(offV + st + s * 16 * ROW + grp * 32);
                const uint32_t wb0 = lds32(offV + st + s * 16 * ROW + ROW + grp * 32);
                const uint32_t wa1 = lds32(offV + st + s * 16 * ROW + 8 * ROW + grp * 32);
                const uint32_t wb1 = lds32(offV + st + s * 16 * ROW + 9 * ROW + grp * 32);
                uint32_t j0[8], j1[8];
                if (MODE == 0 || MODE == 1) {
                    const uint32_t pa[2] = {wa0, wa1}, pb[2] = {wb0, wb1};
                    uint32_t *jj[2] = {j0, j1};
#pragma unroll
                    for (int k = 0; k < 2; ++k) {
                        const uint32_t lo = prmt(pa[k], pb[k], 0x5410u), hi = prmt(pa[k], pb[k], 0x7632u);
                        const uint32_t lo8 = lo >> 8, hi8 = hi >> 8;
                        jj[k][0] = lo & 0x000F000Fu; jj[k][1] = lo & 0x00F000F0u;
                        jj[k][2] = lo8 & 0x000F000Fu; jj[k][3] = lo8 & 0x00F000F0u;
                        jj[k][4] = hi & 0x000F000Fu; jj[k][5] = hi & 0x00F000F0u;
                        jj[k][6] = hi8 & 0x000F000Fu; jj[k][7] = hi8 & 0x00F000F0u;
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < 8; ++k) { j0[k] = wa0 + k; j1[k] = wb1 + k; }
                }
                if (MODE == 0 || MODE == 2) {
#pragma unroll
                    for (int mb = 0; mb < 4; ++mb)
                        mma16816(acc[grp * 4 + mb], j0[2 * mb], j0[2 * mb + 1], j1[2 * mb], j1[2 * mb + 1], qf0 + it, qf1);
                } else if (MODE == 1) {
#pragma unroll
                    for (int k = 0; k < 8; ++k) x ^= j0[k] + j1[k];
                } else {
                    x ^= wa0 ^ wb0 ^ wa1 ^ wb1;
                }
            }
        }
    }
    const long long t1 = clock64();
    float s = c2[0] + c2[1] + c2[2] + c2[3] + (float)x;
    for (int i = 0; i < 8; ++i) s += acc[i][0] + acc[i][1] + acc[i][2] + acc[i][3];
    if (s == 123.456f) sink[threadIdx.x] = s;
    if (lane == 0) out[blockIdx.x * 32 + warp] = (unsigned long long)(t1 - t0);
}

template <int MODE>
void run(int W, unsigned long long *d_out, float *d_sink) {
    const int iters = 2000;
    const int smem = W * STAGE + 1024;
    if (MODE >= 4) {
        cudaFuncSetAttribute(ubi<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        ubi<MODE><<<148, W * 32, smem>>>(iters, d_out, d_sink);
        ubi<MODE><<<148, W * 32, smem>>>(iters, d_out, d_sink);
    } else {
    cudaFuncSetAttribute(ub<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    ub<MODE><<<148, W * 32, smem>>>(iters, d_out, d_sink);   // warm
    ub<MODE><<<148, W * 32, smem>>>(iters, d_out, d_sink);
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return; }
    unsigned long long h[148 * 32];
    cudaMemcpy(h, d_out, sizeof(h), cudaMemcpyDeviceToHost);
    double mx = 0, sum = 0;
    for (int b = 0; b < 148; ++b)
        for (int w = 0; w < W; ++w) { double c = (double)h[b * 32 + w]; sum += c; if (c > mx) mx = c; }
    const double per_warp = sum / (148 * W) / iters;       // cycles per stage per warp
    const double wps = W / 4.0;                            // warps per SMSP
    printf("MODE %d warps/SMSP %5.2f : %7.1f cyc/stage/warp (max %7.1f) -> SMSP %6.1f cyc/stage\n", MODE, wps,
           per_warp, mx / iters, mx / iters / wps);
}

int main() {
    unsigned long long *d_out;
    float *d_sink;
    cudaMalloc(&d_out, 148 * 32 * 8);
    cudaMalloc(&d_sink, 1024 * 4);
    const int Ws[] = {4, 8, 16, 32};
    for (int W : Ws) run<0>(W, d_out, d_sink);
    for (int W : Ws) run<2>(W, d_out, d_sink);
    for (int W : Ws) run<4>(W, d_out, d_sink);
    for (int W : Ws) run<5>(W, d_out, d_sink);
    return 0;
}
