// Where does the block scheduler put CTA i?  592 CTAs x 128 threads, 55 KB dynamic smem
// (the attention kernel's footprint: 4 CTAs / SM).  Prints smid of the first CTAs and the
// number of distinct SMs hosting CTAs [0, n) for several n.
#include <cstdio>
#include <set>
__global__ void k(int *out, int spin) {
    extern __shared__ char sm[];
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    if (threadIdx.x == 0) out[blockIdx.x] = smid;
    long long t0 = clock64();
    while (clock64() - t0 < spin) { sm[threadIdx.x] = (char)t0; }
}
int main() {
    int *d, h[592];
    cudaMalloc(&d, sizeof(h));
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 55424);
    for (int rep = 0; rep < 2; ++rep) {
        k<<<592, 128, 55424>>>(d, 200000);
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    }
    printf("first 40 CTAs -> smid:");
    for (int i = 0; i < 40; ++i) printf(" %d", h[i]);
    printf("\n");
    for (int n : {64, 128, 148, 256, 296, 512, 592}) {
        std::set<int> s(h, h + n);
        printf("CTAs [0,%d): %zu distinct SMs\n", n, s.size());
    }
    // strided picks
    for (int st : {2, 4}) {
        std::set<int> s;
        for (int i = 0; i < 128; ++i) s.insert(h[i * st]);
        printf("CTAs 0,%d,2*%d..(128 of them): %zu distinct SMs\n", st, st, s.size());
    }
    return 0;
}
