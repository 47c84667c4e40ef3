// Microbenchmark: tcgen05.mma (kind::f16, cta_group::1, M = 128) issue throughput per SM
// for A from shared memory vs A from tensor memory, N = 64 / 128 / 256.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/ub_umma scripts/ubench_umma.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a) {
    return (uint64_t)((a & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)64 << 32) | ((uint64_t)1 << 46) |
           ((uint64_t)2 << 61);
}
template <int N, bool ATMEM>
__global__ void __launch_bounds__(128, 1) k(int iters, unsigned long long *out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;\n" ::"r"(su32(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n");
    const uint32_t tm = tslot;
    const uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    long long t0 = 0, t1 = 0;
    if (threadIdx.x == 0) {
        const uint32_t a = su32(sm), b = a + 16384;
        t0 = clock64();
        for (int i = 0; i < iters; ++i) {
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
                if (ATMEM)
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tm),
                                 "r"(tm + 256 + kk * 8), "l"(desc(b + kk * 32)), "r"(idesc), "r"(1));
                else
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm),
                                 "l"(desc(a + kk * 32)), "l"(desc(b + kk * 32)), "r"(idesc), "r"(1));
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(su32(&bar)));
        asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@P1 bra D;\nbra W;\nD:\n}\n" ::"r"(su32(&bar)));
        t1 = clock64();
        out[blockIdx.x] = (unsigned long long)(t1 - t0);
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n");
    __syncthreads();
    if (warp == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;\n");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;\n" ::"r"(tm));
    }
}
template <int N, bool ATMEM>
void run(unsigned long long *d) {
    const int iters = 4000, smem = 16384 + 256 * 128 + 1024;
    cudaFuncSetAttribute(k<N, ATMEM>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    k<N, ATMEM><<<148, 128, smem>>>(iters, d);
    k<N, ATMEM><<<148, 128, smem>>>(iters, d);
    if (cudaDeviceSynchronize() != cudaSuccess) { printf("err\n"); return; }
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
    const double per = mx / (iters * 4.0);                       // cycles per UMMA (128 x N x 16)
    const double macs = 128.0 * N * 16 / per;                    // MAC / cycle / SM
    printf("A %s N=%3d: %6.1f cyc per 128x%dx16 UMMA = %6.0f MAC/cyc/SM = %5.0f TFLOP/s @1.965GHz x148\n",
           ATMEM ? "tmem" : "smem", N, per, N, macs, macs * 2 * 148 * 1.965e9 / 1e12);
}
int main() {
    unsigned long long *d;
    cudaMalloc(&d, 148 * 8);
    run<64, false>(d); run<128, false>(d); run<256, false>(d);
    run<64, true>(d); run<128, true>(d); run<256, true>(d);
    return 0;
}
