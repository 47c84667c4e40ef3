// offload.cu -- NEXT-4: host-offloaded q4 KV cache executor (the paper's
// setting, Alg 1: per layer load_cache -> compute -> store_cache,
// the loads of the next layers overlapped with the current layer's compute).
//
// B200 design: the q4 cache rows of a layer are one strided copy
// (cudaMemcpy2DAsync: B*Hkv rows of (L-1)*row bytes, pitch cap*row) on a
// dedicated H2D stream into a device ring slot; the fused decode step
// (A2+A3+A4, decode_attn.cu) runs on the slot on the caller's stream; the new
// token's row pair (V codes are pair-interleaved) goes back with one strided D2H on a second copy stream (the two
// PCIe directions overlap).  Per-slot events order slot reuse.  All
// enqueue-only; no device allocation.
#include <new>

#include "common.cuh"

extern "C" lmo_status lmo_decode_step_q4(const lmo_kv_cache *, const void *, const void *,
                                         const void *, int32_t, int32_t, const int32_t *, float,
                                         int32_t, void *, lmo_dtype, void *, size_t, uint32_t,
                                         void *);
extern "C" size_t lmo_kv_row_bytes(int32_t head_dim);

struct lmo_offload {
    lmo_kv_cache shape;
    int layers, slots;
    uint8_t *host, *ring;
    size_t row, layer_bytes;
    cudaStream_t h2d, d2h;
    cudaEvent_t *loaded, *computed, *freed;   // [slots]
    cudaEvent_t done;
};

namespace {
bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
lmo_status cuda_ok(cudaError_t e) { return e == cudaSuccess ? LMO_OK : LMO_ERR_CUDA; }

lmo_status check_shape(const lmo_kv_cache *c) {
    if (!c) return LMO_ERR_NULL;
    if (c->batch <= 0 || c->kv_heads <= 0 || c->capacity <= 0 || c->capacity % 16) return LMO_ERR_SHAPE;
    if (c->head_dim != 64 && c->head_dim != 128) return LMO_ERR_UNSUPPORTED;
    return LMO_OK;
}
size_t layer_bytes(const lmo_kv_cache *c) {
    return (size_t)c->batch * c->kv_heads * c->capacity * lmo_kv_row_bytes(c->head_dim);
}
void destroy_events(lmo_offload *x) {
    for (int s = 0; s < x->slots; ++s) {
        if (x->loaded && x->loaded[s]) cudaEventDestroy(x->loaded[s]);
        if (x->computed && x->computed[s]) cudaEventDestroy(x->computed[s]);
        if (x->freed && x->freed[s]) cudaEventDestroy(x->freed[s]);
    }
    delete[] x->loaded;
    delete[] x->computed;
    delete[] x->freed;
    if (x->done) cudaEventDestroy(x->done);
    if (x->h2d) cudaStreamDestroy(x->h2d);
    if (x->d2h) cudaStreamDestroy(x->d2h);
}
}  // namespace

extern "C" {

size_t lmo_offload_ring_bytes(const lmo_kv_cache *shape, int32_t ring_slots) {
    if (check_shape(shape) != LMO_OK || ring_slots < 1) return 0;
    return layer_bytes(shape) * (size_t)ring_slots;
}

lmo_status lmo_offload_create(const lmo_kv_cache *shape, int32_t layers, uint8_t *host_kv,
                              uint8_t *ring_dev, int32_t ring_slots, lmo_offload_t *out) {
    const lmo_status st = check_shape(shape);
    if (st != LMO_OK) return st;
    if (!host_kv || !ring_dev || !out) return LMO_ERR_NULL;
    if (layers < 1 || ring_slots < 1) return LMO_ERR_SHAPE;
    if (!aligned16(host_kv) || !aligned16(ring_dev)) return LMO_ERR_ALIGN;
    lmo_offload *x = new (std::nothrow) lmo_offload();
    if (!x) return LMO_ERR_CUDA;
    x->shape = *shape;
    x->shape.kv = nullptr;
    x->layers = layers;
    x->slots = ring_slots;
    x->host = host_kv;
    x->ring = ring_dev;
    x->row = lmo_kv_row_bytes(shape->head_dim);
    x->layer_bytes = layer_bytes(shape);
    x->loaded = new (std::nothrow) cudaEvent_t[ring_slots]();
    x->computed = new (std::nothrow) cudaEvent_t[ring_slots]();
    x->freed = new (std::nothrow) cudaEvent_t[ring_slots]();
    bool ok = x->loaded && x->computed && x->freed;
    ok = ok && cudaStreamCreateWithFlags(&x->h2d, cudaStreamNonBlocking) == cudaSuccess;
    ok = ok && cudaStreamCreateWithFlags(&x->d2h, cudaStreamNonBlocking) == cudaSuccess;
    for (int s = 0; ok && s < ring_slots; ++s) {
        ok = cudaEventCreateWithFlags(&x->loaded[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&x->computed[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&x->freed[s], cudaEventDisableTiming) == cudaSuccess;
    }
    ok = ok && cudaEventCreateWithFlags(&x->done, cudaEventDisableTiming) == cudaSuccess;
    if (!ok) {
        destroy_events(x);
        delete x;
        return LMO_ERR_CUDA;
    }
    *out = x;
    return LMO_OK;
}

lmo_status lmo_offload_decode_step(lmo_offload_t x, const void *k_new, const void *v_new,
                                   const void *q, int32_t q_heads, int32_t len,
                                   float softmax_scale, int32_t num_splits, void *out,
                                   lmo_dtype out_dtype, void *workspace, size_t workspace_bytes,
                                   void *compute_stream) {
    if (!x) return LMO_ERR_NULL;
    if (!k_new || !v_new || !q || !out) return LMO_ERR_NULL;
    const lmo_kv_cache &c = x->shape;
    if (len < 1 || len > c.capacity) return LMO_ERR_SHAPE;
    if (q_heads <= 0 || q_heads % c.kv_heads) return LMO_ERR_SHAPE;
    // validate one layer's step up front (same shapes for every layer): nothing is
    // enqueued on an argument error
    {
        const size_t need = lmo_decode_attention_workspace_bytes(c.batch, c.kv_heads, q_heads,
                                                                 c.head_dim, num_splits);
        if (need == 0) return LMO_ERR_SHAPE;
        if (!workspace || workspace_bytes < need) return LMO_ERR_WORKSPACE;
    }
    if (!aligned16(k_new) || !aligned16(v_new) || !aligned16(q) || !aligned16(out) ||
        !aligned16(workspace))
        return LMO_ERR_ALIGN;
    cudaStream_t cs = static_cast<cudaStream_t>(compute_stream);
    const size_t pairs = (size_t)c.batch * c.kv_heads;
    const size_t pitch = (size_t)c.capacity * x->row;
    const size_t kv_layer = pairs * c.head_dim * 2;                 // fp16 [B][Hkv][d]
    const size_t q_layer = (size_t)c.batch * q_heads * c.head_dim * 2;
    const size_t o_layer = (size_t)c.batch * q_heads * c.head_dim * (out_dtype == LMO_F16 ? 2 : 4);
    // the step's inputs come from compute_stream's past: copies start after it
    if (cudaEventRecord(x->done, cs) != cudaSuccess) return LMO_ERR_CUDA;
    if (cudaStreamWaitEvent(x->h2d, x->done, 0) != cudaSuccess) return LMO_ERR_CUDA;
    for (int l = 0; l < x->layers; ++l) {
        const int s = l % x->slots;
        uint8_t *slot = x->ring + (size_t)s * x->layer_bytes;
        uint8_t *host = x->host + (size_t)l * x->layer_bytes;
        // load_cache: the old tokens [0, len-1) of every (b, kvh), as whole token pairs
        // (rows [0, len & ~1): an old token's pair partner row carries half its V codes)
        cudaError_t e = cudaStreamWaitEvent(x->h2d, x->freed[s], 0);
        const size_t nrows = (size_t)(len & ~1);
        if (e == cudaSuccess && nrows > 0)
            e = cudaMemcpy2DAsync(slot, pitch, host, pitch, nrows * x->row, pairs,
                                  cudaMemcpyHostToDevice, x->h2d);
        if (e == cudaSuccess) e = cudaEventRecord(x->loaded[s], x->h2d);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, x->loaded[s], 0);
        if (e != cudaSuccess) return LMO_ERR_CUDA;
        // compute: append the new token at len-1, attend over len (A2+A3+A4)
        lmo_kv_cache lc = c;
        lc.kv = slot;
        const lmo_status st = lmo_decode_step_q4(
            &lc, static_cast<const uint8_t *>(k_new) + l * kv_layer,
            static_cast<const uint8_t *>(v_new) + l * kv_layer,
            static_cast<const uint8_t *>(q) + l * q_layer, q_heads, len, nullptr, softmax_scale,
            num_splits, static_cast<uint8_t *>(out) + l * o_layer, out_dtype, workspace,
            workspace_bytes, 0u, cs);
        if (st != LMO_OK) return st;
        // store_cache: the new token back to host memory -- the two rows of its token pair
        // (the pair's V codes are interleaved across both rows, include/lmo.h)
        e = cudaEventRecord(x->computed[s], cs);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(x->d2h, x->computed[s], 0);
        const size_t r0 = (size_t)((len - 1) & ~1);
        if (e == cudaSuccess)
            e = cudaMemcpy2DAsync(host + r0 * x->row, pitch, slot + r0 * x->row, pitch, 2 * x->row, pairs,
                                  cudaMemcpyDeviceToHost, x->d2h);
        if (e == cudaSuccess) e = cudaEventRecord(x->freed[s], x->d2h);
        if (e != cudaSuccess) return LMO_ERR_CUDA;
    }
    // the caller's stream covers the whole step
    if (cudaEventRecord(x->done, x->d2h) != cudaSuccess) return LMO_ERR_CUDA;
    return cuda_ok(cudaStreamWaitEvent(cs, x->done, 0));
}

lmo_status lmo_offload_destroy(lmo_offload_t x) {
    if (!x) return LMO_ERR_NULL;
    cudaStreamSynchronize(x->h2d);
    cudaStreamSynchronize(x->d2h);
    destroy_events(x);
    delete x;
    return LMO_OK;
}

}  // extern "C"
