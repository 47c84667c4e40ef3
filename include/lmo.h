/*
 * lmo.h -- C ABI of the B200-native (sm_100a) LM-Offload hot path.
 *
 * Paper: "LM-Offload: Performance Model-Guided Generative Inference of Large
 * Language Models with Parallelism Control" (dblp/paper_conf_ipps_wurypgll25).
 * "P:n" cites line n of the paper text.
 *
 * Conventions (all entry points):
 *  - Every pointer except `cache` / status-string results is a DEVICE
 *    pointer owned by the caller.  The library never allocates, frees or
 *    synchronizes; it keeps no mutable global state except a launch counter
 *    and a once-initialised device-property cache.
 *  - `stream` is a cudaStream_t passed as void* (0 = legacy default stream).
 *    Every call only enqueues work on it and returns.
 *  - Argument errors are detected synchronously BEFORE any launch and nothing
 *    is written.  A failed launch returns LMO_ERR_CUDA (cudaGetLastError);
 *    asynchronous faults surface at the caller's next synchronization.
 *  - fp16 data is IEEE binary16.  Inputs must be finite (NaN/Inf: results
 *    unspecified).  No aliasing between inputs and outputs except the KV
 *    cache, which append updates in place.
 *  - Storage format ("compressed tensor", Alg 2): 4-bit codes, two
 *    per byte, LOW nibble = element 2j, HIGH nibble = element 2j+1; one
 *    lmo_qmeta {fp16 min, fp16 scale} per group of 64 consecutive elements
 *    along the quantize dimension.  Dequantized value = min + code*scale.
 */
#ifndef LMO_H_
#define LMO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    LMO_OK = 0,
    LMO_ERR_NULL = 1,         /* a required pointer is NULL                  */
    LMO_ERR_SHAPE = 2,        /* a size is negative/zero/inconsistent        */
    LMO_ERR_UNSUPPORTED = 3,  /* bits != 4, group != 64, head_dim not 64/128, */
                              /* group ratio > 8, ...                          */
    LMO_ERR_ALIGN = 4,        /* a pointer is not 16-byte aligned            */
    LMO_ERR_WORKSPACE = 5,    /* workspace missing or too small              */
    LMO_ERR_CUDA = 6          /* a CUDA runtime call or launch failed        */
} lmo_status;

typedef enum { LMO_F16 = 0, LMO_F32 = 1 } lmo_dtype;

/* Per-group metadata, 4 bytes: fp16 bit patterns of the group minimum and of
 * the quantization step scale = RU16(RN32(max - min) / 15).  scale == 0 iff
 * the group is constant (Eq 10's 0/0 case, reading 1). */
typedef struct {
    uint16_t min_f16;
    uint16_t scale_f16;
} lmo_qmeta;

/* ---------------------------------------------------------------------------
 * A1. Group-wise 4-bit quantization -- Alg 2 "Compress(tensor, target_bits,
 * quantize_dim)" with Eq 10:
 *     x_quant = round((x - min) / (max - min) * (2^b - 1)),
 * evaluated as code = min(15, rint(RN32(RN32(x - min) * RN32(1/scale)))).
 *
 * x_f16 : fp16 tensor viewed as (outer, n, inner), contiguous.  Groups are
 *         group_size consecutive elements along n (the quantize_dim); n is
 *         padded with +0 to n_pad = ceil(n/64)*64 and the pads take part in
 *         min/max (Alg 2 l.5-6 precede l.9-10).
 * codes : (outer, n_pad/2, inner) bytes; byte[o][j][i] packs elements 2j
 *         (low nibble) and 2j+1 (high nibble) of row (o, :, i).
 * meta  : (outer, n_pad/64, inner) lmo_qmeta.
 * bits must be 4 and group_size 64 (else LMO_ERR_UNSUPPORTED).  x, codes and
 * meta must be 16-byte aligned.  outer/n/inner == 0 is a no-op.
 * ------------------------------------------------------------------------- */
lmo_status lmo_quantize_groupwise(const void *x_f16, int64_t outer, int64_t n, int64_t inner,
                                  int bits, int group_size, uint8_t *codes, lmo_qmeta *meta,
                                  void *stream);

/* ---------------------------------------------------------------------------
 * A5. Group-wise dequantization -- Eq 11 in step form:
 *     y = RN16(RN32(code * scale + min)),
 * bit-exact with the oracle.  Same (outer, n, inner) view as above; y_f16 is
 * (outer, n, inner) fp16 (padding dropped).  Weights are quantized once and
 * only dequantized afterwards (Eq 4).
 * ------------------------------------------------------------------------- */
lmo_status lmo_dequantize_groupwise(const uint8_t *codes, const lmo_qmeta *meta, int64_t outer,
                                    int64_t n, int64_t inner, int bits, int group_size,
                                    void *y_f16, void *stream);

/* One layer's q4 KV cache (caller-owned device memory): one contiguous
 * "compressed row" per (sequence, kv head, token slot):
 *   kv : [batch][kv_heads][capacity][row_bytes]        row_bytes = lmo_kv_row_bytes(head_dim)
 *   row: K codes (head_dim/2 B) | K meta (head_dim/64 lmo_qmeta) |
 *        V area  (head_dim/2 B) | V meta (head_dim/64 lmo_qmeta)
 * (144 B per token at head_dim 128, 72 B at 64).  K codes and both metas are
 * exactly what lmo_quantize_groupwise(outer=1, n=head_dim, inner=1) produces for
 * that token's K (resp. V) row.  The V codes of a token PAIR (slots 2p, 2p+1)
 * are stored interleaved in 16-bit chunks of 4 dims: 32-bit word c of the pair =
 * [token 2p chunk c (low half) | token 2p+1 chunk c (high half)], where chunk c
 * holds the quantize_groupwise code bytes of dims 4c .. 4c+3; words 0 ..
 * head_dim/8-1 fill the V area of row 2p, the rest that of row 2p+1.  (One word
 * is then a tensor-core operand "(token, token) x 4 dims" without byte shuffles.)
 * A token's V codes therefore live in both rows of its pair; appends write only
 * the token's own 16-bit halves.  Token-major rows make a run of tokens of one
 * (sequence, kv head) a single contiguous span, i.e. one bulk copy.  Groups lie
 * along head_dim (reading 8), so every token's groups are
 * self-contained.  head_dim must be 64 or 128; capacity must be a multiple of
 * 16 (callers round up; the 16-token block is the kernels' unit of work); kv
 * must be 16-byte aligned. */
typedef struct {
    uint8_t *kv;
    int32_t batch;
    int32_t kv_heads;
    int32_t capacity;
    int32_t head_dim;
} lmo_kv_cache;

/* Bytes of one compressed K+V token row for head_dim (0 if unsupported). */
size_t lmo_kv_row_bytes(int32_t head_dim);

/* ---------------------------------------------------------------------------
 * A2. KV append-quantize -- "The KV cache is updated by concatenating the
 * current token's key and value vectors with the existing ones"; "the
 * newly generated KV cache is quantized" each token, each layer (P:235,
 * Eq 7; "new KV cache is compressed, old ... only decompressed").
 *
 * k_new_f16, v_new_f16 : [batch][kv_heads][n_new][head_dim] fp16.
 * Row (b, h, t) is quantized exactly as lmo_quantize_groupwise(outer=1,
 * n=head_dim, inner=1) would, and written to cache slot pos_b + t, where
 * pos_b = pos_dev[b] if pos_dev != NULL (device int32[batch]) else pos0.
 * Only slots [pos_b, pos_b + n_new) of each (b, h) are written.
 * Host-checked: 0 <= pos0, pos0 + n_new <= capacity (when pos_dev == NULL);
 * 2*batch*kv_heads*n_new*(head_dim/64) < 2^31 (else LMO_ERR_SHAPE).
 * With pos_dev, out-of-range rows (pos_b < 0 or pos_b + n_new > capacity)
 * are skipped on the device.
 * ------------------------------------------------------------------------- */
lmo_status lmo_kv_append_quant(const lmo_kv_cache *cache, const void *k_new_f16,
                               const void *v_new_f16, int32_t n_new, int32_t pos0,
                               const int32_t *pos_dev, void *stream);

/* Workspace bytes lmo_decode_attention_q4 needs for this shape.  The first
 * 4*batch*kv_heads bytes are per-(sequence, kv head) arrival counters that
 * MUST be zero before the first call on a workspace (e.g. cudaMemsetAsync);
 * every call leaves them zero again.  One call in flight per workspace. */
size_t lmo_decode_attention_workspace_bytes(int32_t batch, int32_t kv_heads, int32_t q_heads,
                                            int32_t head_dim, int32_t num_splits);

/* ---------------------------------------------------------------------------
 * A3+A4. Decode-step attention over the q4 cache with dequantization fused
 * ("QK^T/sqrt(d_k) ... A softmax function is then applied"; the old
 * cache is only dequantized, Eq 6):
 *   o[b][h] = softmax(softmax_scale * q[b][h] . K[b][kvh][0:L_b]^T) V[b][kvh][0:L_b]
 * with kvh = h / (q_heads / kv_heads) and K/V the dequantized cache rows
 * (min + code*scale).  fp32 accumulation, numerically stable softmax.
 *
 * q_f16       : [batch][q_heads][head_dim] fp16.
 * len         : L_b for every sequence when seq_lens_dev == NULL
 *               (1 <= len <= capacity, host-checked).
 * seq_lens_dev: optional device int32[batch]; L_b = min(seq_lens_dev[b],
 *               capacity); L_b <= 0 writes a zero output row.
 * num_splits  : 0 = auto: "pair teams" (each (b, kvh) pair processed by a
 *               team of 1, 2 or 4 warps of one CTA, combined on chip) when
 *               there are enough pairs to fill the GPU, else "stream-K" (the
 *               16-token blocks of all pairs divided evenly over the resident
 *               warps; partial results merged in-kernel by the last arriving
 *               warp).  1, 2, 4 = pair teams of that size; other k > 0 = each
 *               pair split into k contiguous parts merged in-kernel.  With
 *               k > 0 results do not depend on batch composition.
 *               LMO_SPLITS_STREAMK (-1) = stream-K explicitly.
 *               LMO_SPLITS_SMTEAM (-2) = "SM teams" (uniform length only,
 *               else auto): one CTA per SM owns a contiguous equal share of
 *               the (b, kvh) pairs, its warps split that share into equal
 *               block ranges, and pairs cut between warps are merged once
 *               per CTA after a CTA barrier.
 * out         : [batch][q_heads][head_dim], LMO_F32 or LMO_F16.
 * q_heads/kv_heads must be in 1..8.
 * ------------------------------------------------------------------------- */
#define LMO_SPLITS_STREAMK (-1)
#define LMO_SPLITS_SMTEAM (-2)
lmo_status lmo_decode_attention_q4(const lmo_kv_cache *cache, const void *q_f16, int32_t q_heads,
                                   int32_t len, const int32_t *seq_lens_dev, float softmax_scale,
                                   int32_t num_splits, void *out, lmo_dtype out_dtype,
                                   void *workspace, size_t workspace_bytes, void *stream);

/* ---------------------------------------------------------------------------
 * A2+A3+A4 fused: one decode step of one layer -- append-quantize the new
 * token's K/V (Eq 7) at slot L_b - 1, then attend over L_b tokens
 * (the new token through its quantized form, reading 13).
 * k_new_f16, v_new_f16 : [batch][kv_heads][head_dim] fp16 (the new token).
 * len / seq_lens_dev give L_b as in lmo_decode_attention_q4 (new token
 * included; L_b <= 0 appends nothing and writes a zero row).  Equivalent to
 * lmo_kv_append_quant(pos = L_b - 1, n_new = 1) followed by
 * lmo_decode_attention_q4 on the same stream, in one launch when the pair-team
 * schedule is used (else two).  Other arguments as lmo_decode_attention_q4.
 * flags: LMO_STEP_CACHE_STABLE = the kernel issued immediately before this
 *        call on `stream` does not write this cache's slots [0, L_b - 1) (true
 *        in a layer-by-layer decode loop).  The kernel may then start streaming
 *        those old-token blocks before the previous kernel has finished
 *        (programmatic dependent launch), overlapping its pipeline fill with
 *        the previous kernel's tail.  Ignored with seq_lens_dev.  0 = none.
 *        LMO_STEP_FLEXGEN_EXACT = the new token enters its OWN step's attention
 *        with its raw fp16 K/V (FlexGen's semantics, reading 13b:
 *        "the new KV cache is compressed, old only decompressed", P:159,
 *        P:235-243); it is still appended quantized at slot L_b - 1 for later
 *        steps.  Default (0): the new token is attended through its quantized
 *        form (reading 13).  Flags combine with |.
 * ------------------------------------------------------------------------- */
#define LMO_STEP_CACHE_STABLE 1u
#define LMO_STEP_FLEXGEN_EXACT 2u
lmo_status lmo_decode_step_q4(const lmo_kv_cache *cache, const void *k_new_f16,
                              const void *v_new_f16, const void *q_f16, int32_t q_heads,
                              int32_t len, const int32_t *seq_lens_dev, float softmax_scale,
                              int32_t num_splits, void *out, lmo_dtype out_dtype, void *workspace,
                              size_t workspace_bytes, uint32_t flags, void *stream);

/* ---------------------------------------------------------------------------
 * NEXT-4: host-offloaded q4 KV cache -- the paper's setting.
 * LM-Offload keeps the KV cache in CPU memory and, per layer, loads the cache
 * to the GPU, computes, and stores the new token's K/V back, overlapping the
 * loads of the next layers with the current layer's compute (Alg 1,
 * load_cache / compute / store_cache; Eq 6-7).
 *
 * host_kv   : pinned host memory (caller-owned, e.g. cudaHostAlloc or
 *             torch pin_memory), `layers` consecutive q4 caches each laid out
 *             exactly like a device lmo_kv_cache: [B][Hkv][cap][row] bytes.
 *             `shape` gives B, Hkv, cap, head_dim (its kv field is ignored).
 * ring_dev  : device staging ring, caller-owned, >= lmo_offload_ring_bytes();
 *             slot s is a full device cache of the same shape.
 * ring_slots: >= 1; layer l uses slot l % ring_slots, so up to ring_slots - 1
 *             layers are loaded ahead of the one being computed.
 * The executor owns two copy streams (H2D, D2H) and per-slot events; it never
 * allocates device memory.  Destroy with lmo_offload_destroy.
 * ------------------------------------------------------------------------- */
typedef struct lmo_offload *lmo_offload_t;
size_t lmo_offload_ring_bytes(const lmo_kv_cache *shape, int32_t ring_slots);
lmo_status lmo_offload_create(const lmo_kv_cache *shape, int32_t layers, uint8_t *host_kv,
                              uint8_t *ring_dev, int32_t ring_slots, lmo_offload_t *out);

/* One decode step of all layers at length L = len (the new token goes to slot
 * len-1 of every layer's cache).  For each layer l:
 *   H2D   rows [0, len & ~1) of every (b, kvh) of host layer l -> ring slot
 *         (the old tokens [0, len-1) as whole row pairs, see lmo_kv_cache)
 *         (one strided copy; waits until the slot's previous user is stored),
 *   A2-A4 lmo_decode_step_q4 on the slot with k_new/v_new/q of layer l
 *         (on compute_stream, after the H2D),
 *   D2H   the row pair of token len-1 (rows (len-1) & ~1 and +1) of every
 *         (b, kvh) of the slot -> host layer l.
 * k_new, v_new : device [layers][B][Hkv][head_dim] fp16; q device
 * [layers][B][q_heads][head_dim] fp16; out device [layers][B][q_heads][head_dim]
 * (out_dtype).  Other arguments as lmo_decode_step_q4 (num_splits, workspace).
 * Enqueues only; compute_stream is made to wait for the last D2H, so a
 * synchronize on compute_stream covers the whole step.  Host-side argument
 * errors are reported before anything is enqueued. */
lmo_status lmo_offload_decode_step(lmo_offload_t ex, const void *k_new_f16, const void *v_new_f16,
                                   const void *q_f16, int32_t q_heads, int32_t len,
                                   float softmax_scale, int32_t num_splits, void *out,
                                   lmo_dtype out_dtype, void *workspace, size_t workspace_bytes,
                                   void *compute_stream);
lmo_status lmo_offload_destroy(lmo_offload_t ex);

/* ---------------------------------------------------------------------------
 * NEXT-3. Linear layer over group-wise q4 weights (W4A16), dequantization fused
 * into the GEMM.  The paper dequantizes the q4 weights on the GPU every decode
 * step before the layer's matmuls ("load_weight + dequan_wgt", Eq 4
 * P:228-233; Eq 11); here the q4 codes stream from HBM
 * and are expanded only in shared memory:
 *     y[b][n] = sum_k x[b][k] * RN16(c[n][k] * scale[n][k/64] + min[n][k/64]).
 *
 * codes : W [N][K] quantized along K (lmo_quantize_groupwise with outer = N,
 *         n = K, inner = 1): [N][K/2] bytes, low nibble = even k.
 * meta  : [N][K/64] lmo_qmeta.
 * x_f16 : activations [batch][K] fp16, row-major.
 * y_f32 : output [batch][N] fp32, row-major (overwritten).
 * N % 128 == 0, K % 64 == 0, 1 <= batch <= 128 (else LMO_ERR_SHAPE /
 * LMO_ERR_UNSUPPORTED).  k_split: K-dimension split (0 = auto: split-K over
 * one wave of resident CTAs, or -- packed path, batch <= 64, when that wave is
 * poorly filled -- stream-K, equal ranges of the tile-steps of all tiles that
 * may cross a tile boundary); with a split (k_split > 1 or an auto split) y is
 * zeroed on `stream` by a kernel of this library and the partial tiles are
 * added atomically (summation order then varies: results agree within fp32
 * rounding; k_split = 1 is deterministic).  All
 * pointers 16-byte aligned.  Device memory is caller-owned; enqueued on
 * `stream`, asynchronous.
 * ------------------------------------------------------------------------- */
lmo_status lmo_w4a16_linear(const uint8_t *codes, const lmo_qmeta *meta, int64_t N, int64_t K,
                            const void *x_f16, int32_t batch, float *y_f32, int32_t k_split,
                            void *stream);

/* NEXT-3, streaming layout.  The paper quantizes the weights once at load
 * time; lmo_w4a16_pack rearranges them once into the layout the GEMM
 * streams: for each 128-row tile t and group g, one contiguous 4608-byte block
 * at offset (t * K/64 + g) * 4608 holding the tile's 128 rows x 32 code bytes
 * followed by their 128 lmo_qmeta.  Each 32-bit code word (8 consecutive k,
 * k-th code at nibble k) is stored k-interleaved: nibbles 0-3 hold k 0, 2, 4, 6
 * and nibbles 4-7 hold k 1, 3, 5, 7 (the dequantizer's masks then yield
 * k-ordered fp16 pairs directly).  A tile-step is then one 1-D bulk copy of
 * whole DRAM pages instead of 128 scattered 32-byte row pieces.
 * lmo_w4a16_packed_bytes gives the size (0 for an invalid shape);
 * lmo_w4a16_linear_packed computes exactly what lmo_w4a16_linear computes on
 * the unpacked codes/meta (same arithmetic, same shapes and errors). */
size_t lmo_w4a16_packed_bytes(int64_t N, int64_t K);
lmo_status lmo_w4a16_pack(const uint8_t *codes, const lmo_qmeta *meta, int64_t N, int64_t K,
                          uint8_t *packed, void *stream);
lmo_status lmo_w4a16_linear_packed(const uint8_t *packed, int64_t N, int64_t K, const void *x_f16,
                                   int32_t batch, float *y_f32, int32_t k_split, void *stream);

/* Human-readable name of a status code (static string). */
const char *lmo_status_string(lmo_status status);

/* ---------------------------------------------------------------------------
 * Support entry points (not steps of the method).
 * ------------------------------------------------------------------------- */

/* Seeded synthetic inputs (bench/test support, no method arithmetic): fills
 * dst [nb][nh][npos][dim] fp16 with the counter-based generator documented in
 * paper_conf_ipps_wurypgll25_b200/inputs.py, at global coordinates
 * (layer, b0+ib, h0+ih, p0+ip, i).  `group` maps a head to its kv head for
 * the outlier-channel mask (q: q_heads/kv_heads, K/V: 1).  Bit-identical to
 * inputs.gen_f16. */
lmo_status lmo_gen_fill_f16(void *dst, int32_t nb, int32_t nh, int32_t npos, int32_t dim,
                            uint64_t seed, int32_t stream_id, int32_t layer, int32_t b0,
                            int32_t h0, int32_t p0, int32_t group, void *stream);

/* Read-only HBM stream (measurement support for the bench's roofline
 * denominators): reads `bytes` (a multiple of 16, >= 16)
 * of device memory at buf with 128-bit streaming loads over a persistent
 * grid; sink is a device buffer of >= 4 * 4 * SM-count bytes that is written
 * only on an impossible XOR sentinel (keeps the loads live).  buf and sink
 * 16-byte aligned. */
lmo_status lmo_probe_read_stream(const void *buf, size_t bytes, void *sink, void *stream);

/* Number of kernels this library has launched in this process. */
uint64_t lmo_launch_count(void);

/* ABI version: (major << 16) | minor. */
uint32_t lmo_version(void);

#ifdef __cplusplus
}
#endif

#endif /* LMO_H_ */
