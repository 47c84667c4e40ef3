// gen.cu -- K6: seeded synthetic-input generator (bench/test support; holds no
// method arithmetic).  Device twin of paper_conf_ipps_wurypgll25_b200/inputs.py
// (splitmix64 counter -> Irwin-Hall(4) -> x8 outlier channels for K/q -> RN16),
// bit-identical to it (tests/test_gpu_parity.py::test_generator_matches_host).
#include "common.cuh"

namespace lmo {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void __launch_bounds__(256) gen_fill_kernel(__half *__restrict__ dst, int nb, int nh,
                                                       int npos, int dim, uint64_t seed, int stream,
                                                       int layer, int b0, int h0, int p0,
                                                       int group) {
    const int64_t total = (int64_t)nb * nh * npos * dim;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
         e += (int64_t)gridDim.x * blockDim.x) {
        const uint64_t i = (uint64_t)(e % dim);
        const uint64_t p = (uint64_t)(p0 + (e / dim) % npos);
        const uint64_t h = (uint64_t)(h0 + (e / ((int64_t)dim * npos)) % nh);
        const uint64_t b = (uint64_t)(b0 + e / ((int64_t)dim * npos * nh));
        const uint64_t idx = ((uint64_t)layer << 44) | (b << 32) | (h << 24) | (p << 12) | i;
        const uint64_t hs = splitmix64(seed ^ ((uint64_t)stream << 56) ^ idx);
        const int s = (int)(hs & 0xFFFF) + (int)((hs >> 16) & 0xFFFF) + (int)((hs >> 32) & 0xFFFF) +
                      (int)((hs >> 48) & 0xFFFF) - 131070;
        float v = (float)s * (1.0f / 32768.0f);   // exact
        if (stream == 1 || stream == 3) {           // K, q: outlier channels
            const uint64_t kvh = h / (uint64_t)group;
            const uint64_t key = seed ^ (0xA5ull << 56) ^ ((uint64_t)layer << 32) ^ (kvh << 16) ^ i;
            if (splitmix64(key) % 100ull == 0ull) v *= 8.0f;
        }
        dst[e] = __float2half_rn(v);
    }
}

cudaError_t launch_gen_fill(void *dst, int nb, int nh, int npos, int dim, uint64_t seed, int stream,
                            int layer, int b0, int h0, int p0, int group, cudaStream_t st) {
    const int64_t total = (int64_t)nb * nh * npos * dim;
    int64_t blocks = (total + 255) / 256;
    const int64_t cap = (int64_t)device_sm_count() * 16;
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    gen_fill_kernel<<<(unsigned)blocks, 256, 0, st>>>(static_cast<__half *>(dst), nb, nh, npos, dim,
                                                      seed, stream, layer, b0, h0, p0, group);
    note_launch();
    return cudaGetLastError();
}

}  // namespace lmo
