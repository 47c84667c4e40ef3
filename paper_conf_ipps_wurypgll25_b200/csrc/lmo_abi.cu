// lmo_abi.cu -- the extern "C" boundary (include/lmo.h): argument validation,
// status codes, launch bookkeeping.  No exceptions cross the ABI; nothing is
// launched or written when validation fails.
#include <atomic>
#include <cstdlib>
#include <mutex>

#include "common.cuh"

namespace lmo {

static std::atomic<uint64_t> g_launches{0};
void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

int device_sm_count() {
    static int cache[64] = {0};
    static std::mutex mu;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (cache[dev] == 0) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cache[dev] = n > 0 ? n : 1;
    }
    return cache[dev];
}

cudaError_t launch_quantize(const void *, int64_t, int64_t, int64_t, uint8_t *, lmo_qmeta *,
                            cudaStream_t);
cudaError_t launch_dequantize(const uint8_t *, const lmo_qmeta *, int64_t, int64_t, int64_t,
                              void *, cudaStream_t);
cudaError_t launch_kv_append(const lmo_kv_cache &, const void *, const void *, int, int,
                             const int32_t *, cudaStream_t, int pos_from_lens);
cudaError_t launch_decode_attention(const lmo_kv_cache &, const void *, int, int, const int32_t *,
                                    float, int, void *, int, void *, cudaStream_t, const void *,
                                    const void *, unsigned);

// Programmatic dependent launch for the hot-path kernels (always on in release
// builds; LMO_EXPERIMENTS builds read LMO_PDL=0 to disable it for measurements).
bool pdl_enabled() {
#ifdef LMO_EXPERIMENTS
    static const int v = [] {
        const char *e = getenv("LMO_PDL");
        return (e && e[0] == '0') ? 0 : 1;
    }();
    return v == 1;
#else
    return true;
#endif
}
cudaError_t launch_gen_fill(void *, int, int, int, int, uint64_t, int, int, int, int, int, int,
                            cudaStream_t);
size_t attn_workspace_bytes(int B, int Hkv, int Hq, int D, int num_splits);
cudaError_t launch_w4a16(const uint8_t *codes, const void *meta, const uint8_t *packed, const void *x, float *y,
                         int N, int K, int batch, int ksplit, cudaStream_t st);
cudaError_t launch_w4a16_pack(const uint8_t *codes, const void *meta, uint8_t *packed, int N, int K, cudaStream_t st);

cudaError_t launch_read_stream(const void *buf, size_t bytes, void *sink, cudaStream_t st);

static bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

static lmo_status check_cache(const lmo_kv_cache *c) {
    if (!c || !c->kv) return LMO_ERR_NULL;
    if (c->batch <= 0 || c->kv_heads <= 0 || c->capacity <= 0) return LMO_ERR_SHAPE;
    if (c->head_dim != 64 && c->head_dim != 128) return LMO_ERR_UNSUPPORTED;
    if (c->capacity % 16 != 0) return LMO_ERR_SHAPE;
    if (!aligned16(c->kv)) return LMO_ERR_ALIGN;
    return LMO_OK;
}

static lmo_status cuda_status(cudaError_t e) { return e == cudaSuccess ? LMO_OK : LMO_ERR_CUDA; }

}  // namespace lmo

using namespace lmo;

extern "C" {

lmo_status lmo_quantize_groupwise(const void *x, int64_t outer, int64_t n, int64_t inner, int bits,
                                  int group_size, uint8_t *codes, lmo_qmeta *meta, void *stream) {
    if (bits != 4 || group_size != kGroup) return LMO_ERR_UNSUPPORTED;
    if (outer < 0 || n < 0 || inner < 0) return LMO_ERR_SHAPE;
    if (outer == 0 || n == 0 || inner == 0) return LMO_OK;
    if (!x || !codes || !meta) return LMO_ERR_NULL;
    if (!aligned16(x) || !aligned16(codes) || !aligned16(meta)) return LMO_ERR_ALIGN;
    return cuda_status(
        launch_quantize(x, outer, n, inner, codes, meta, static_cast<cudaStream_t>(stream)));
}

lmo_status lmo_dequantize_groupwise(const uint8_t *codes, const lmo_qmeta *meta, int64_t outer,
                                    int64_t n, int64_t inner, int bits, int group_size, void *y,
                                    void *stream) {
    if (bits != 4 || group_size != kGroup) return LMO_ERR_UNSUPPORTED;
    if (outer < 0 || n < 0 || inner < 0) return LMO_ERR_SHAPE;
    if (outer == 0 || n == 0 || inner == 0) return LMO_OK;
    if (!codes || !meta || !y) return LMO_ERR_NULL;
    if (!aligned16(codes) || !aligned16(meta) || !aligned16(y)) return LMO_ERR_ALIGN;
    return cuda_status(
        launch_dequantize(codes, meta, outer, n, inner, y, static_cast<cudaStream_t>(stream)));
}

lmo_status lmo_kv_append_quant(const lmo_kv_cache *cache, const void *k_new, const void *v_new,
                               int32_t n_new, int32_t pos0, const int32_t *pos_dev, void *stream) {
    lmo_status s = check_cache(cache);
    if (s != LMO_OK) return s;
    if (!k_new || !v_new) return LMO_ERR_NULL;
    if (n_new < 0) return LMO_ERR_SHAPE;
    if (n_new == 0) return LMO_OK;
    if (!pos_dev && (pos0 < 0 || (int64_t)pos0 + n_new > cache->capacity)) return LMO_ERR_SHAPE;
    // the append kernel indexes (row, K|V, group) units in 32-bit
    if (2LL * cache->batch * cache->kv_heads * n_new * (cache->head_dim / kGroup) >= (1LL << 31))
        return LMO_ERR_SHAPE;
    if (!aligned16(k_new) || !aligned16(v_new)) return LMO_ERR_ALIGN;
    return cuda_status(launch_kv_append(*cache, k_new, v_new, n_new, pos0, pos_dev,
                                        static_cast<cudaStream_t>(stream), 0));
}

size_t lmo_decode_attention_workspace_bytes(int32_t batch, int32_t kv_heads, int32_t q_heads,
                                            int32_t head_dim, int32_t num_splits) {
    if (batch <= 0 || kv_heads <= 0 || q_heads <= 0 || q_heads % kv_heads != 0 || num_splits < LMO_SPLITS_SMTEAM ||
        (head_dim != 64 && head_dim != 128))
        return 0;
    return attn_workspace_bytes(batch, kv_heads, q_heads, head_dim, num_splits);
}

static lmo_status check_attention(const lmo_kv_cache *cache, const void *q, int32_t q_heads,
                                  int32_t len, const int32_t *seq_lens_dev, int32_t num_splits,
                                  void *out, lmo_dtype out_dtype, void *workspace,
                                  size_t workspace_bytes) {
    lmo_status s = check_cache(cache);
    if (s != LMO_OK) return s;
    if (!q || !out) return LMO_ERR_NULL;
    if (q_heads <= 0 || q_heads % cache->kv_heads != 0) return LMO_ERR_SHAPE;
    if (q_heads / cache->kv_heads > 8) return LMO_ERR_UNSUPPORTED;
    if (num_splits < LMO_SPLITS_SMTEAM) return LMO_ERR_SHAPE;
    if (out_dtype != LMO_F16 && out_dtype != LMO_F32) return LMO_ERR_UNSUPPORTED;
    if (!seq_lens_dev && (len < 1 || len > cache->capacity)) return LMO_ERR_SHAPE;
    if (seq_lens_dev && cache->batch > 1024) return LMO_ERR_UNSUPPORTED;
    if ((int64_t)cache->batch * cache->kv_heads * ((int64_t)cache->capacity / 16) > (1LL << 30))
        return LMO_ERR_SHAPE;
    if (!aligned16(q) || !aligned16(out)) return LMO_ERR_ALIGN;
    const size_t need = attn_workspace_bytes(cache->batch, cache->kv_heads, q_heads,
                                             cache->head_dim, num_splits);
    if (!workspace || workspace_bytes < need) return LMO_ERR_WORKSPACE;
    if (!aligned16(workspace)) return LMO_ERR_ALIGN;
    return LMO_OK;
}

lmo_status lmo_decode_attention_q4(const lmo_kv_cache *cache, const void *q, int32_t q_heads,
                                   int32_t len, const int32_t *seq_lens_dev, float softmax_scale,
                                   int32_t num_splits, void *out, lmo_dtype out_dtype,
                                   void *workspace, size_t workspace_bytes, void *stream) {
    const lmo_status s = check_attention(cache, q, q_heads, len, seq_lens_dev, num_splits, out,
                                         out_dtype, workspace, workspace_bytes);
    if (s != LMO_OK) return s;
    return cuda_status(launch_decode_attention(*cache, q, q_heads, len, seq_lens_dev,
                                               softmax_scale, num_splits, out,
                                               out_dtype == LMO_F16 ? 1 : 0, workspace,
                                               static_cast<cudaStream_t>(stream), nullptr,
                                               nullptr, 0u));
}

lmo_status lmo_decode_step_q4(const lmo_kv_cache *cache, const void *k_new_f16,
                              const void *v_new_f16, const void *q, int32_t q_heads, int32_t len,
                              const int32_t *seq_lens_dev, float softmax_scale, int32_t num_splits,
                              void *out, lmo_dtype out_dtype, void *workspace,
                              size_t workspace_bytes, uint32_t flags, void *stream) {
    const lmo_status s = check_attention(cache, q, q_heads, len, seq_lens_dev, num_splits, out,
                                         out_dtype, workspace, workspace_bytes);
    if (s != LMO_OK) return s;
    if (!k_new_f16 || !v_new_f16) return LMO_ERR_NULL;
    if (!aligned16(k_new_f16) || !aligned16(v_new_f16)) return LMO_ERR_ALIGN;
    return cuda_status(launch_decode_attention(*cache, q, q_heads, len, seq_lens_dev,
                                               softmax_scale, num_splits, out,
                                               out_dtype == LMO_F16 ? 1 : 0, workspace,
                                               static_cast<cudaStream_t>(stream), k_new_f16,
                                               v_new_f16, flags));
}

const char *lmo_status_string(lmo_status st) {
    switch (st) {
        case LMO_OK: return "LMO_OK";
        case LMO_ERR_NULL: return "LMO_ERR_NULL: required pointer is NULL";
        case LMO_ERR_SHAPE: return "LMO_ERR_SHAPE: invalid or inconsistent size";
        case LMO_ERR_UNSUPPORTED: return "LMO_ERR_UNSUPPORTED: unsupported bits/group/head_dim/ratio";
        case LMO_ERR_ALIGN: return "LMO_ERR_ALIGN: pointer not 16-byte aligned";
        case LMO_ERR_WORKSPACE: return "LMO_ERR_WORKSPACE: workspace missing or too small";
        case LMO_ERR_CUDA: return "LMO_ERR_CUDA: CUDA runtime/launch error";
    }
    return "LMO_ERR_UNKNOWN";
}

lmo_status lmo_gen_fill_f16(void *dst, int32_t nb, int32_t nh, int32_t npos, int32_t dim,
                            uint64_t seed, int32_t stream_id, int32_t layer, int32_t b0, int32_t h0,
                            int32_t p0, int32_t group, void *stream) {
    if (!dst) return LMO_ERR_NULL;
    if (nb < 0 || nh < 0 || npos < 0 || dim < 0 || group <= 0 || b0 < 0 || h0 < 0 || p0 < 0)
        return LMO_ERR_SHAPE;
    if ((int64_t)nb * nh * npos * dim == 0) return LMO_OK;
    if (layer < 0 || layer >= 256 || b0 + nb > 4096 || h0 + nh > 256 || p0 + npos > 4096 ||
        dim > 4096)
        return LMO_ERR_SHAPE;
    return cuda_status(launch_gen_fill(dst, nb, nh, npos, dim, seed, stream_id, layer, b0, h0, p0,
                                       group, static_cast<cudaStream_t>(stream)));
}

size_t lmo_kv_row_bytes(int32_t head_dim) {
    if (head_dim != 64 && head_dim != 128) return 0;
    return (size_t)2 * (head_dim / 2 + 4 * (head_dim / kGroup));
}

uint64_t lmo_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

lmo_status lmo_w4a16_linear(const uint8_t *codes, const lmo_qmeta *meta, int64_t N, int64_t K,
                            const void *x, int32_t batch, float *y, int32_t k_split, void *stream) {
    if (!codes || !meta || !x || !y) return LMO_ERR_NULL;
    if (N <= 0 || K <= 0 || batch <= 0 || k_split < 0) return LMO_ERR_SHAPE;
    if (N % 128 != 0 || K % kGroup != 0 || N > (1ll << 30) || K > (1ll << 30)) return LMO_ERR_SHAPE;
    if (batch > 128) return LMO_ERR_UNSUPPORTED;
    if (!aligned16(codes) || !aligned16(meta) || !aligned16(x) || !aligned16(y)) return LMO_ERR_ALIGN;
    return cuda_status(launch_w4a16(codes, meta, nullptr, x, y, (int)N, (int)K, batch, k_split,
                                    static_cast<cudaStream_t>(stream)));
}

size_t lmo_w4a16_packed_bytes(int64_t N, int64_t K) {
    if (N <= 0 || K <= 0 || N % 128 != 0 || K % kGroup != 0) return 0;
    return (size_t)(N / 128) * (size_t)(K / kGroup) * 4608u;
}

lmo_status lmo_w4a16_pack(const uint8_t *codes, const lmo_qmeta *meta, int64_t N, int64_t K, uint8_t *packed,
                          void *stream) {
    if (!codes || !meta || !packed) return LMO_ERR_NULL;
    if (N <= 0 || K <= 0 || N % 128 != 0 || K % kGroup != 0 || N > (1ll << 30) || K > (1ll << 30)) return LMO_ERR_SHAPE;
    if (!aligned16(codes) || !aligned16(meta) || !aligned16(packed)) return LMO_ERR_ALIGN;
    return cuda_status(launch_w4a16_pack(codes, meta, packed, (int)N, (int)K, static_cast<cudaStream_t>(stream)));
}

lmo_status lmo_w4a16_linear_packed(const uint8_t *packed, int64_t N, int64_t K, const void *x, int32_t batch,
                                   float *y, int32_t k_split, void *stream) {
    if (!packed || !x || !y) return LMO_ERR_NULL;
    if (N <= 0 || K <= 0 || batch <= 0 || k_split < 0) return LMO_ERR_SHAPE;
    if (N % 128 != 0 || K % kGroup != 0 || N > (1ll << 30) || K > (1ll << 30)) return LMO_ERR_SHAPE;
    if (batch > 128) return LMO_ERR_UNSUPPORTED;
    if (!aligned16(packed) || !aligned16(x) || !aligned16(y)) return LMO_ERR_ALIGN;
    return cuda_status(launch_w4a16(nullptr, nullptr, packed, x, y, (int)N, (int)K, batch, k_split,
                                    static_cast<cudaStream_t>(stream)));
}

lmo_status lmo_probe_read_stream(const void *buf, size_t bytes, void *sink, void *stream) {
    if (!buf || !sink) return LMO_ERR_NULL;
    if (bytes < 16 || bytes % 16 != 0) return LMO_ERR_SHAPE;
    if (!aligned16(buf) || !aligned16(sink)) return LMO_ERR_ALIGN;
    return cuda_status(launch_read_stream(buf, bytes, sink, static_cast<cudaStream_t>(stream)));
}

uint32_t lmo_version(void) { return (1u << 16) | 0u; }

}  // extern "C"
