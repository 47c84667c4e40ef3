/*
 * lmo_oracle.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * Plain, slow, obviously-correct CPU oracle for the LM-Offload hot path
 * (dblp/paper_conf_ipps_wurypgll25).  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * under paper_conf_ipps_wurypgll25_b200/csrc/ and never calls it.
 *
 * Built with: gcc -O2 -std=c11 -fno-fast-math -ffp-contract=off -shared -fPIC
 * (no SIMD intrinsics, no OpenMP; the only threading is a plain pthread
 * fan-out over independent (b, head) rows in the _mt attention entry).
 *
 * Citations: "P:n" = /root/reference/PAPER.md line n.
 *   - Group-wise quantization: Alg 2, Eq 10, the prose
 *     "pads ... partitions all elements into groups along a certain
 *     dimension ... finds the minimum and maximum ... normalizes each element
 *     to the range (0, 2^b-1) using Equation 10 ... packed".
 *   - Dequantization: Eq 11.
 *   - KV append: "The KV cache is updated by concatenating the current
 *     token's key and value vectors with the existing ones"; "the
 *     newly generated KV cache is quantized" (Eq 7).
 *   - Attention: "attention score ... QK^T/sqrt(d_k) ... A softmax function
 *     is then applied"; P.V per the standard definition (reading 14).
 *
 * Readings of the paper:
 *   Q0 pad with +0 to a multiple of G=64; pads take part in min/max (Alg 2
 *      l.5-6 precede l.9-10).
 *   Q1 -0 is read as +0.
 *   Q2 mn/mx = min/max of the group (exact fp16 values).
 *   Q3 range = RN32(mx - mn).
 *   Q4 scale = RU16(range / 15)  (step form of Eq 10's (max-min)/(2^b-1),
 *      rounded up so that (x-mn)/scale <= 15 and |x - deq| <= scale/2).
 *   Q5 inv = scale == 0 ? 0 : RN32(1/scale).
 *   Q6 code = min(15, rint_half_even(RN32(RN32(x - mn) * inv))).
 *   Q7 meta = {fp16 mn, fp16 scale}.
 *   Q8 byte[j] = code[2j] | code[2j+1] << 4 (low nibble = even element).
 *   D1 y = RN16(RN32(code * scale + mn))  (Eq 11 in step form).
 *   T1-T5 attention in fp64 on the exact dequantized reals mn + c*scale.
 *   T6 (reading 13b, FlexGen-exact, optional): the newest token L_b-1 of each
 *      (b, kv head) enters its own step's attention with its raw fp16 K/V
 *      (k_last/v_last), not its quantized form -- "the newly generated KV cache
 *      is quantized" for later steps while the current step computes with it
 *      (P:159).
 * Each RN32 step is emulated by computing in fp64 and casting to float: the
 * fp64 result of +,-,*,/ on fp32/fp16 operands is either exact or a single
 * RN64 rounding, and RN32(RN64(r)) == RN32(r) because 53 >= 2*24+2.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define LMO_ORACLE_OK 0
#define LMO_ORACLE_EINVAL 1

/* ------------------------------------------------------------------ fp16 */

/* Exact value of a binary16 bit pattern. */
double lmo_oracle_h2d(uint16_t h) {
    int sign = (h >> 15) & 1;
    int e = (h >> 10) & 0x1f;
    int m = h & 0x3ff;
    double v;
    if (e == 0) {
        v = ldexp((double)m, -24);                 /* subnormal / zero */
    } else if (e == 31) {
        v = m ? NAN : INFINITY;
    } else {
        v = ldexp((double)(m + 1024), e - 25);     /* 1.m * 2^(e-15) */
    }
    return sign ? -v : v;
}

/* Encode a value that is exactly representable as binary16 (|a| finite). */
static uint16_t encode_exact_half(double a, int sign) {
    uint16_t s = (uint16_t)(sign ? 0x8000 : 0);
    if (a == 0.0) return s;
    if (a >= 65536.0) return (uint16_t)(s | 0x7c00);           /* overflowed */
    if (a < ldexp(1.0, -14)) {
        return (uint16_t)(s | (uint16_t)(a / ldexp(1.0, -24)));   /* subnormal */
    }
    int E;
    double f = frexp(a, &E);            /* a = f * 2^E, f in [0.5, 1) */
    int e = E - 1;                      /* a = (2f) * 2^e, 2f in [1, 2) */
    int mant = (int)((2.0 * f - 1.0) * 1024.0);
    return (uint16_t)(s | (uint16_t)((e + 15) << 10) | (uint16_t)mant);
}

/* Round-to-nearest-even to binary16 (subnormals kept, overflow -> inf). */
uint16_t lmo_oracle_rn16(double x) {
    if (isnan(x)) return 0x7e00;
    int sign = signbit(x) ? 1 : 0;
    double a = fabs(x);
    if (a >= 65520.0) return (uint16_t)((sign ? 0x8000 : 0) | 0x7c00);
    double quantum;
    if (a < ldexp(1.0, -14)) {
        quantum = ldexp(1.0, -24);
    } else {
        int E;
        frexp(a, &E);
        quantum = ldexp(1.0, E - 1 - 10);
    }
    double r = nearbyint(a / quantum);  /* default rounding mode: half-even */
    return encode_exact_half(r * quantum, sign);
}

/* Round toward +infinity to binary16, for x >= 0: RN16, then one ulp up if
 * the rounded value is below x. */
uint16_t lmo_oracle_ru16(double x) {
    uint16_t h = lmo_oracle_rn16(x);
    if (lmo_oracle_h2d(h) < x) h = (uint16_t)(h + 1);  /* x >= 0: next up */
    return h;
}

/* --------------------------------------------------------- quantization */

/* Alg 2 "Compress" with target_bits = 4 and a user group size. x is
 * viewed as (outer, n, inner) fp16 bit patterns; groups are `group`
 * consecutive elements along n (the quantize_dim).  Outputs:
 *   codes: (outer, n_pad/2, inner) bytes, n_pad = ceil(n/group)*group
 *   meta : (outer, n_pad/group, inner) pairs {min bits, scale bits}. */
int lmo_oracle_quantize_groupwise(const uint16_t *x, int64_t outer, int64_t n, int64_t inner,
                                  int bits, int group, uint8_t *codes, uint16_t *meta) {
    if (bits != 4 || group <= 0 || group % 2 != 0 || outer < 0 || n < 0 || inner < 0)
        return LMO_ORACLE_EINVAL;
    const int qmax = (1 << bits) - 1;                     /* 2^b - 1 = 15 */
    int64_t ngroups = (n + group - 1) / group;
    int64_t npad = ngroups * group;
    double *vals = (double *)malloc(sizeof(double) * (size_t)group);
    int *c = (int *)malloc(sizeof(int) * (size_t)group);
    if (!vals || !c) { free(vals); free(c); return LMO_ORACLE_EINVAL; }
    for (int64_t o = 0; o < outer; ++o) {
        for (int64_t g = 0; g < ngroups; ++g) {
            for (int64_t i = 0; i < inner; ++i) {
                /* Q0/Q1: pad with +0 (Alg 2 l.5-6), read -0 as +0 */
                for (int k = 0; k < group; ++k) {
                    int64_t j = g * group + k;
                    double v = 0.0;
                    if (j < n) v = lmo_oracle_h2d(x[(o * n + j) * inner + i]);
                    vals[k] = v + 0.0;                     /* -0 + 0 = +0 */
                }
                /* Q2: min / max along quantize_dim (Alg 2 l.9-10) */
                double mn = vals[0], mx = vals[0];
                for (int k = 1; k < group; ++k) {
                    if (vals[k] < mn) mn = vals[k];
                    if (vals[k] > mx) mx = vals[k];
                }
                /* Q3-Q5: Eq 10's (max-min)/(2^b-1) as a rounded-up fp16 step */
                float range = (float)(mx - mn);
                uint16_t scale_bits = lmo_oracle_ru16((double)range / (double)qmax);
                double scale = lmo_oracle_h2d(scale_bits);
                float inv = (scale == 0.0) ? 0.0f : (float)(1.0 / scale);
                /* Q6: min-max normalisation (Alg 2 l.12, Eq 10) + clamp (l.14) */
                for (int k = 0; k < group; ++k) {
                    float d = (float)(vals[k] - mn);
                    float t = (float)((double)d * (double)inv);
                    double r = nearbyint((double)t);
                    if (r > qmax) r = qmax;
                    if (r < 0) r = 0;
                    c[k] = (int)r;
                }
                /* Q7: meta */
                uint16_t *mt = meta + ((o * ngroups + g) * inner + i) * 2;
                mt[0] = lmo_oracle_rn16(mn);
                mt[1] = scale_bits;
                /* Q8: pack (Alg 2 l.16), low nibble = even element */
                for (int k = 0; k < group; k += 2) {
                    int64_t jb = (g * group + k) / 2;
                    codes[(o * (npad / 2) + jb) * inner + i] =
                        (uint8_t)((c[k] & 0xf) | ((c[k + 1] & 0xf) << 4));
                }
            }
        }
    }
    free(vals);
    free(c);
    return LMO_ORACLE_OK;
}

/* Eq 11 in step form: y = RN16(RN32(code * scale + min)); padding dropped. */
int lmo_oracle_dequantize_groupwise(const uint8_t *codes, const uint16_t *meta, int64_t outer,
                                    int64_t n, int64_t inner, int bits, int group, uint16_t *y) {
    if (bits != 4 || group <= 0 || group % 2 != 0) return LMO_ORACLE_EINVAL;
    int64_t ngroups = (n + group - 1) / group;
    int64_t npad = ngroups * group;
    for (int64_t o = 0; o < outer; ++o)
        for (int64_t j = 0; j < n; ++j)
            for (int64_t i = 0; i < inner; ++i) {
                uint8_t byte = codes[(o * (npad / 2) + j / 2) * inner + i];
                int c = (j % 2 == 0) ? (byte & 0xf) : (byte >> 4);
                const uint16_t *mt = meta + ((o * ngroups + j / group) * inner + i) * 2;
                double mn = lmo_oracle_h2d(mt[0]);
                double scale = lmo_oracle_h2d(mt[1]);
                double exact = (double)c * scale + mn;   /* exact in fp64 (<= 41 bits) */
                y[(o * n + j) * inner + i] = lmo_oracle_rn16((double)(float)exact);
            }
    return LMO_ORACLE_OK;
}

/* ----------------------------------------------------------- KV append */

/* Quantize k_new/v_new [B][Hkv][n_new][d] (fp16 bits) row by row (groups
 * along head_dim) into cache slots pos[b]..pos[b]+n_new-1 of the cache
 * layout [B][Hkv][cap][d/2] codes, [B][Hkv][cap][d/64][2] meta. */
int lmo_oracle_kv_append_quant(uint8_t *k_codes, uint16_t *k_meta, uint8_t *v_codes,
                               uint16_t *v_meta, int B, int Hkv, int cap, int d,
                               const uint16_t *k_new, const uint16_t *v_new, int n_new,
                               const int32_t *pos) {
    if (d % 64 != 0) return LMO_ORACLE_EINVAL;
    int ng = d / 64;
    for (int b = 0; b < B; ++b) {
        if (pos[b] < 0 || pos[b] + n_new > cap) return LMO_ORACLE_EINVAL;
        for (int h = 0; h < Hkv; ++h)
            for (int t = 0; t < n_new; ++t) {
                int64_t src = (((int64_t)b * Hkv + h) * n_new + t) * d;
                int64_t slot = ((int64_t)b * Hkv + h) * cap + pos[b] + t;
                int rc = lmo_oracle_quantize_groupwise(k_new + src, 1, d, 1, 4, 64,
                                                       k_codes + slot * (d / 2),
                                                       k_meta + slot * ng * 2);
                if (rc) return rc;
                rc = lmo_oracle_quantize_groupwise(v_new + src, 1, d, 1, 4, 64,
                                                   v_codes + slot * (d / 2),
                                                   v_meta + slot * ng * 2);
                if (rc) return rc;
            }
    }
    return LMO_ORACLE_OK;
}

/* ------------------------------------------------------------ attention */

typedef struct {
    const uint8_t *k_codes, *v_codes;
    const uint16_t *k_meta, *v_meta;
    int B, Hkv, cap, d, Hq;
    const uint16_t *q;
    const int32_t *lens;
    const uint16_t *k_last, *v_last;   /* T6: raw new-token K/V [B][Hkv][d] or NULL */
    double sigma;
    double *out;
    int64_t row_begin, row_end;  /* rows = b*Hq + h */
    int rc;
} attn_job;

/* T2: exact dequantized element i of token j of (b, kvh): mn + c*scale. */
static double deq_elem(const uint8_t *codes, const uint16_t *meta, int64_t slot, int d, int i) {
    uint8_t byte = codes[slot * (d / 2) + i / 2];
    int c = (i % 2 == 0) ? (byte & 0xf) : (byte >> 4);
    const uint16_t *mt = meta + (slot * (d / 64) + i / 64) * 2;
    return lmo_oracle_h2d(mt[0]) + (double)c * lmo_oracle_h2d(mt[1]);
}

static void attn_rows(attn_job *jb) {
    int G = jb->Hq / jb->Hkv;
    int d = jb->d;
    double *z = NULL;
    int zcap = 0;
    for (int64_t row = jb->row_begin; row < jb->row_end; ++row) {
        int b = (int)(row / jb->Hq), h = (int)(row % jb->Hq);
        int kvh = h / G;                                    /* T1 */
        int L = jb->lens[b];
        if (L < 1 || L > jb->cap) { jb->rc = LMO_ORACLE_EINVAL; break; }
        if (L > zcap) { free(z); z = (double *)malloc(sizeof(double) * (size_t)L); zcap = L; }
        const uint16_t *qr = jb->q + row * d;
        int64_t base = ((int64_t)b * jb->Hkv + kvh) * jb->cap;
        double m = -INFINITY;
        const uint16_t *kl = jb->k_last ? jb->k_last + ((int64_t)b * jb->Hkv + kvh) * d : NULL;
        const uint16_t *vl = jb->v_last ? jb->v_last + ((int64_t)b * jb->Hkv + kvh) * d : NULL;
        for (int j = 0; j < L; ++j) {                       /* T3 */
            double acc = 0.0;
            for (int i = 0; i < d; ++i)
                acc += lmo_oracle_h2d(qr[i]) * ((kl && j == L - 1) ? lmo_oracle_h2d(kl[i])        /* T6 */
                                                                  : deq_elem(jb->k_codes, jb->k_meta, base + j, d, i));
            z[j] = jb->sigma * acc;
            if (z[j] > m) m = z[j];
        }
        double l = 0.0;                                     /* T4 */
        for (int j = 0; j < L; ++j) { z[j] = exp(z[j] - m); l += z[j]; }
        double *o = jb->out + row * d;                      /* T5 */
        for (int i = 0; i < d; ++i) {
            double acc = 0.0;
            for (int j = 0; j < L; ++j)
                acc += z[j] * ((vl && j == L - 1) ? lmo_oracle_h2d(vl[i])                          /* T6 */
                                                  : deq_elem(jb->v_codes, jb->v_meta, base + j, d, i));
            o[i] = acc / l;
        }
    }
    free(z);
}

static void *attn_thread(void *arg) { attn_rows((attn_job *)arg); return NULL; }

/* o[b][h] = softmax(sigma * q[b][h] . K[b][h/G][0:L_b]) @ V[b][h/G][0:L_b],
 * over the exact dequantized q4 cache.  q: [B][Hq][d] fp16 bits, lens: [B],
 * out: [B][Hq][d] doubles.  nthreads >= 1 splits rows across pthreads.
 * k_last/v_last (T6, FlexGen-exact): NULL, or raw fp16 K/V [B][Hkv][d] used for
 * token L_b - 1 instead of its cache slot. */
int lmo_oracle_decode_attention_q4_ext(const uint8_t *k_codes, const uint16_t *k_meta,
                                       const uint8_t *v_codes, const uint16_t *v_meta, int B,
                                       int Hkv, int cap, int d, const uint16_t *q, int Hq,
                                       const int32_t *lens, const uint16_t *k_last,
                                       const uint16_t *v_last, double sigma, double *out,
                                       int nthreads) {
    if (d % 64 != 0 || Hkv <= 0 || Hq % Hkv != 0 || nthreads < 1) return LMO_ORACLE_EINVAL;
    int64_t rows = (int64_t)B * Hq;
    if (nthreads > rows) nthreads = (int)(rows > 0 ? rows : 1);
    attn_job *jobs = (attn_job *)calloc((size_t)nthreads, sizeof(attn_job));
    pthread_t *th = (pthread_t *)calloc((size_t)nthreads, sizeof(pthread_t));
    if (!jobs || !th) { free(jobs); free(th); return LMO_ORACLE_EINVAL; }
    for (int t = 0; t < nthreads; ++t) {
        attn_job j = {k_codes, v_codes, k_meta, v_meta, B, Hkv, cap, d, Hq, q, lens, k_last, v_last,
                      sigma, out, rows * t / nthreads, rows * (t + 1) / nthreads, 0};
        jobs[t] = j;
    }
    for (int t = 1; t < nthreads; ++t) pthread_create(&th[t], NULL, attn_thread, &jobs[t]);
    attn_rows(&jobs[0]);
    int rc = jobs[0].rc;
    for (int t = 1; t < nthreads; ++t) {
        pthread_join(th[t], NULL);
        if (jobs[t].rc) rc = jobs[t].rc;
    }
    free(jobs);
    free(th);
    return rc;
}

int lmo_oracle_decode_attention_q4_mt(const uint8_t *k_codes, const uint16_t *k_meta,
                                      const uint8_t *v_codes, const uint16_t *v_meta, int B,
                                      int Hkv, int cap, int d, const uint16_t *q, int Hq,
                                      const int32_t *lens, double sigma, double *out,
                                      int nthreads) {
    return lmo_oracle_decode_attention_q4_ext(k_codes, k_meta, v_codes, v_meta, B, Hkv, cap, d, q,
                                              Hq, lens, NULL, NULL, sigma, out, nthreads);
}

int lmo_oracle_decode_attention_q4(const uint8_t *k_codes, const uint16_t *k_meta,
                                   const uint8_t *v_codes, const uint16_t *v_meta, int B, int Hkv,
                                   int cap, int d, const uint16_t *q, int Hq, const int32_t *lens,
                                   double sigma, double *out) {
    return lmo_oracle_decode_attention_q4_mt(k_codes, k_meta, v_codes, v_meta, B, Hkv, cap, d, q,
                                             Hq, lens, sigma, out, 1);
}

/* ------------------------------------------------- W4A16 linear (NEXT-3) */

/* A linear layer over group-wise q4 weights: the paper quantizes the weights
 * once and dequantizes them on the GPU each decode step before the layer's
 * matmuls ("load_weight + dequan_wgt", Eq 4; "weights only cause
 * de-quantization overhead on GPU" P:293-295; Eq 11).  The plain
 * definition of that step is
 *     y[b][n] = sum_k x[b][k] * W~[n][k],   W~ = D1 dequantization of W,
 * with W quantized along k (groups of `group` consecutive input features of
 * one output row: outer = N, n = K, inner = 1 in quantize_groupwise terms).
 * Computed here in fp64 on the D1 fp16 values, k ascending.  x is fp16 bits
 * [B][K]; codes [N][Kpad/2]; meta [N][Kpad/group][2]; y double [B][N]. */
int lmo_oracle_w4a16_linear(const uint8_t *codes, const uint16_t *meta, int64_t N, int64_t K,
                            int group, const uint16_t *x, int64_t B, double *y) {
    if (N <= 0 || K <= 0 || B <= 0 || group <= 0 || group % 2 != 0) return LMO_ORACLE_EINVAL;
    uint16_t *w = (uint16_t *)malloc((size_t)(N * K) * sizeof(uint16_t));
    if (!w) return LMO_ORACLE_EINVAL;
    int rc = lmo_oracle_dequantize_groupwise(codes, meta, N, K, 1, 4, group, w);   /* D1, Eq 11 */
    if (rc) {
        free(w);
        return rc;
    }
    for (int64_t b = 0; b < B; ++b)
        for (int64_t n = 0; n < N; ++n) {
            double s = 0.0;
            for (int64_t k = 0; k < K; ++k)
                s += lmo_oracle_h2d(x[b * K + k]) * lmo_oracle_h2d(w[n * K + k]);
            y[b * N + n] = s;
        }
    free(w);
    return LMO_ORACLE_OK;
}
