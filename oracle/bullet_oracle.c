/*
 * bullet_oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU reference of the computation on the
 * Bullet co-run hot path (one Llama-style decoder layer, run for a prefill
 * batch and a decode batch).  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product (paper_conf_asplos_0001xc0l026_b200/, libbullet.so) never does,
 * and this file shares no code, header, table or constant with it.
 *
 * Paper passages followed (PAPER.md line numbers, "P:Lnnn"):
 *   - layer = QKV-projection, self-attention, O-projection, MLP; GEMMs with
 *     element-wise ops between them ............................. P:L40 (§2.1)
 *   - prefill builds the KV cache with full attention over its inputs; decode
 *     consumes one token and reads the KV cache ................. P:L42 (§2.1)
 *   - KV cache and index table shared between phases, copy-free
 *     hand-off ................................................. P:L227
 * The block internals (pre-RMSNorm, RoPE rotate-half with llama3 scaling,
 * GQA, SwiGLU, optional QKV bias) are not in the paper; DESIGN.md "Readings"
 * R-1..R-10 state the reading taken (public Llama-3.1 / Qwen2.5 configs).
 *
 * Arithmetic: everything in fp64 from the exact stored inputs (bf16 or fp32
 * values held in float), with the bf16 storage points of the bf16 model
 * mirrored by round-to-nearest-even (reading R-3):
 *   R1 h  = RMSNorm(x)          -> bf16
 *   R2 q,k,v after RoPE         -> bf16 (k,v are what the KV pool stores)
 *   R3 o  = attention output    -> bf16
 *   R4 h2 = RMSNorm(x1)         -> bf16
 *   R5 a  = silu(g) * u         -> bf16
 * x1 and out (the residual stream) are not rounded here.
 * In fp32 mode (bf16_mirror == 0) nothing is rounded except what the pool
 * stores (float).  Loops run in the definition's order; no blocking, no
 * fusion, no online softmax.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int d_model, n_heads, n_kv_heads, head_dim, d_ff;
  double rms_eps;
  double rope_theta;
  int rope_llama3;          /* 1: apply the llama3 inv_freq rescaling */
  double rope_factor, rope_low_freq, rope_high_freq;
  int rope_orig_max_pos;
  int bf16_mirror;          /* 1: bf16 model (round at R1..R5); 0: fp32 model */
} orc_cfg;

typedef struct {
  const float *w_qkv;     /* [(H+2Hkv)*hd][d]  rows: q heads, k heads, v heads */
  const float *b_qkv;     /* [(H+2Hkv)*hd] or NULL */
  const float *w_o;       /* [d][H*hd] */
  const float *w_gate_up; /* [2*I][d]  rows [0,I) gate, [I,2I) up */
  const float *w_down;    /* [d][I] */
  const float *g_attn;    /* [d] */
  const float *g_mlp;     /* [d] */
} orc_weights;

/* ---------------------------------------------------------------- rounding */

/* Round a real number to the nearest bfloat16 value, ties to even.
 * bf16 = 1 sign, 8 exponent, 7 fraction bits (same exponent range as fp32). */
double orc_round_bf16(double x) {
  if (x == 0.0 || !isfinite(x)) return x;
  int e;
  frexp(x, &e);                 /* |x| in [2^(e-1), 2^e) */
  int lead = e - 1;
  if (lead < -126) lead = -126; /* subnormal range: fixed spacing 2^-133 */
  double ulp = ldexp(1.0, lead - 7);
  double r = nearbyint(x / ulp) * ulp;      /* default mode: ties to even */
  if (fabs(r) >= ldexp(1.0, 128)) return copysign(INFINITY, x);
  return r;
}

static double store_point(const orc_cfg *c, double v) {
  return c->bf16_mirror ? orc_round_bf16(v) : v;
}

/* ------------------------------------------------------------ primitives */

/* RMSNorm of one row: h_j = x_j / sqrt(mean_k x_k^2 + eps) * g_j. */
void orc_rmsnorm_row(const double *x, const float *g, int d, double eps, double *h) {
  double ss = 0.0;
  for (int k = 0; k < d; ++k) ss += x[k] * x[k];
  double inv = 1.0 / sqrt(ss / d + eps);
  for (int j = 0; j < d; ++j) h[j] = x[j] * inv * (double)g[j];
}

/* y_j = sum_k h_k W[j][k] (+ b_j) for one row; W stored [N][K]. */
void orc_linear_row(const double *h, const float *W, const float *b, int K, int N, double *y) {
  for (int j = 0; j < N; ++j) {
    const float *w = W + (size_t)j * K;
    double acc = 0.0;
    for (int k = 0; k < K; ++k) acc += h[k] * (double)w[k];
    y[j] = acc + (b ? (double)b[j] : 0.0);
  }
}

/* RoPE inverse frequencies inv_freq_i = theta^(-2i/hd), i < hd/2, followed
 * (Llama-3.1) by the llama3 band rescaling of the public config:
 * wavelength lambda = 2*pi/inv_freq; lambda < L/high -> unchanged;
 * lambda > L/low -> inv_freq/factor; otherwise a linear blend with
 * smooth = (L/lambda - low)/(high - low). */
void orc_rope_inv_freq(const orc_cfg *c, double *inv_freq) {
  int hd = c->head_dim;
  for (int i = 0; i < hd / 2; ++i) {
    double f = pow(c->rope_theta, -2.0 * i / hd);
    if (c->rope_llama3) {
      double L = (double)c->rope_orig_max_pos;
      double lam = 2.0 * M_PI / f;
      double hi_wav = L / c->rope_high_freq, lo_wav = L / c->rope_low_freq;
      if (lam < hi_wav) {
        /* high-frequency band: unchanged */
      } else if (lam > lo_wav) {
        f = f / c->rope_factor;
      } else {
        double smooth = (L / lam - c->rope_low_freq) / (c->rope_high_freq - c->rope_low_freq);
        f = (1.0 - smooth) * f / c->rope_factor + smooth * f;
      }
    }
    inv_freq[i] = f;
  }
}

/* Rotate-half RoPE of one head vector u[hd] at position pos:
 * (a, b) = (u_i, u_{i+hd/2}) -> (a cos t - b sin t, b cos t + a sin t),
 * t = pos * inv_freq_i. */
void orc_rope_apply(double *u, int hd, int pos, const double *inv_freq) {
  for (int i = 0; i < hd / 2; ++i) {
    double t = (double)pos * inv_freq[i];
    double a = u[i], b = u[i + hd / 2];
    u[i] = a * cos(t) - b * sin(t);
    u[i + hd / 2] = b * cos(t) + a * sin(t);
  }
}

/* Pool slot of token position p of a request with block-table row bt:
 * block bt[p / B], offset p % B.  Returns the element offset of
 * pool[blk][kvh][p % B][0] in a [n_blocks][Hkv][B][hd] pool. */
size_t orc_slot_offset(const int *bt, int p, int B, int Hkv, int hd, int kvh) {
  size_t blk = (size_t)bt[p / B];
  return ((blk * Hkv + kvh) * (size_t)B + (size_t)(p % B)) * hd;
}

/* Attention of one query head vector q[hd] over keys 0..last (inclusive)
 * of one request, K/V gathered through the block table from the pool:
 *   s_j = q.k_j / sqrt(hd);  p_j = exp(s_j - max s) / sum exp(...);
 *   o = sum_j p_j v_j.   (causal: key j <= query position; DESIGN R-8) */
void orc_attend_paged(const double *q, const float *pool_k, const float *pool_v,
                      const int *bt, int B, int Hkv, int hd, int kvh, int last,
                      double *o) {
  int nk = last + 1;
  double *s = (double *)malloc(sizeof(double) * (size_t)nk);
  double scale = 1.0 / sqrt((double)hd);
  double mx = -INFINITY;
  for (int j = 0; j < nk; ++j) {
    const float *k = pool_k + orc_slot_offset(bt, j, B, Hkv, hd, kvh);
    double acc = 0.0;
    for (int t = 0; t < hd; ++t) acc += q[t] * (double)k[t];
    s[j] = acc * scale;
    if (s[j] > mx) mx = s[j];
  }
  double den = 0.0;
  for (int j = 0; j < nk; ++j) { s[j] = exp(s[j] - mx); den += s[j]; }
  for (int t = 0; t < hd; ++t) o[t] = 0.0;
  for (int j = 0; j < nk; ++j) {
    const float *v = pool_v + orc_slot_offset(bt, j, B, Hkv, hd, kvh);
    double p = s[j] / den;
    for (int t = 0; t < hd; ++t) o[t] += p * (double)v[t];
  }
  free(s);
}

static double silu(double z) { return z / (1.0 + exp(-z)); }

/* ------------------------------------------------------------ the layer */

/*
 * One decoder layer for a batch of requests.  Request r has ctx_lens[r]
 * tokens already in the pool and q_lens[r] new tokens at positions
 * ctx_lens[r] .. ctx_lens[r]+q_lens[r]-1 (prefill: ctx = 0; decode: q = 1).
 * Rows of x/out are the new tokens, request-major.
 *
 * Steps (DESIGN.md §"Oracle"):
 *  1 h = RMSNorm(x) g_attn                                      (R1)
 *  2 qkv = h W_qkv^T (+b)
 *  3 RoPE(q), RoPE(k) at the token position                      (R2)
 *  4 k, v -> pool slot bt[r][p/B]*B + p%B  (ALL rows, also unsampled)
 *  5 o = softmax(q k^T / sqrt(hd), keys <= position) v, GQA g=h/(H/Hkv) (R3)
 *  6 x1 = x + o W_o^T
 *  7 h2 = RMSNorm(x1) g_mlp                                     (R4)
 *  8 a = silu(h2 W_g^T) * (h2 W_u^T)                            (R5)
 *  9 out = x1 + a W_down^T
 * Steps 5-9 run only for rows with row_mask[row] != 0 (row_mask NULL: all).
 * Steps 1-4 run for every row: the pool must hold every new key before any
 * query reads it.  Optional diagnostics (NULL to skip): q_out [rows][H*hd],
 * o_out [rows][H*hd], a_out [rows][I] (rows outside the mask are left 0).
 * Returns 0, or -1 on an invalid argument (block id out of range, etc.).
 */
int orc_layer_forward(const orc_cfg *c, const orc_weights *w,
                      float *pool_k, float *pool_v, int n_blocks, int B,
                      int n_reqs, const int *q_lens, const int *ctx_lens,
                      const int *block_table, int max_blocks,
                      const double *x, double *out, const unsigned char *row_mask,
                      double *q_out, double *o_out, double *a_out) {
  const int d = c->d_model, H = c->n_heads, Hkv = c->n_kv_heads, hd = c->head_dim;
  const int I = c->d_ff, NQKV = (H + 2 * Hkv) * hd, grp = H / Hkv;
  if (H % Hkv != 0 || hd % 2 != 0) return -1;

  int n_rows = 0;
  for (int r = 0; r < n_reqs; ++r) {
    int last = ctx_lens[r] + q_lens[r] - 1;
    if (q_lens[r] < 0 || ctx_lens[r] < 0) return -1;
    if (q_lens[r] > 0 && last / B >= max_blocks) return -1;
    for (int p = 0; p <= last && q_lens[r] > 0; p += 1) {
      int blk = block_table[(size_t)r * max_blocks + p / B];
      if (blk < 0 || blk >= n_blocks) return -1;
    }
    n_rows += q_lens[r];
  }
  int *row_req = (int *)malloc(sizeof(int) * (size_t)(n_rows + 1));
  int *row_pos = (int *)malloc(sizeof(int) * (size_t)(n_rows + 1));
  for (int r = 0, row = 0; r < n_reqs; ++r)
    for (int i = 0; i < q_lens[r]; ++i, ++row) { row_req[row] = r; row_pos[row] = ctx_lens[r] + i; }

  double *inv_freq = (double *)malloc(sizeof(double) * (size_t)(hd / 2));
  orc_rope_inv_freq(c, inv_freq);
  double *q_all = (double *)malloc(sizeof(double) * (size_t)n_rows * H * hd + 1);

  /* steps 1-4 for every row */
#pragma omp parallel for schedule(dynamic, 4)
  for (int row = 0; row < n_rows; ++row) {
    double *h = (double *)malloc(sizeof(double) * (size_t)d);
    double *qkv = (double *)malloc(sizeof(double) * (size_t)NQKV);
    orc_rmsnorm_row(x + (size_t)row * d, w->g_attn, d, c->rms_eps, h);
    for (int j = 0; j < d; ++j) h[j] = store_point(c, h[j]);                 /* R1 */
    orc_linear_row(h, w->w_qkv, w->b_qkv, d, NQKV, qkv);
    int r = row_req[row], pos = row_pos[row];
    const int *bt = block_table + (size_t)r * max_blocks;
    for (int hh = 0; hh < H + Hkv; ++hh) orc_rope_apply(qkv + (size_t)hh * hd, hd, pos, inv_freq);
    for (int j = 0; j < NQKV; ++j) qkv[j] = store_point(c, qkv[j]);          /* R2 */
    memcpy(q_all + (size_t)row * H * hd, qkv, sizeof(double) * (size_t)H * hd);
    for (int g = 0; g < Hkv; ++g) {
      size_t off = orc_slot_offset(bt, pos, B, Hkv, hd, g);
      for (int t = 0; t < hd; ++t) {
        pool_k[off + t] = (float)qkv[(size_t)(H + g) * hd + t];
        pool_v[off + t] = (float)qkv[(size_t)(H + Hkv + g) * hd + t];
      }
    }
    free(h); free(qkv);
  }

  /* steps 5-9 for the sampled rows */
#pragma omp parallel for schedule(dynamic, 1)
  for (int row = 0; row < n_rows; ++row) {
    if (row_mask && !row_mask[row]) continue;
    int r = row_req[row], pos = row_pos[row];
    const int *bt = block_table + (size_t)r * max_blocks;
    const double *q = q_all + (size_t)row * H * hd;
    double *o = (double *)malloc(sizeof(double) * (size_t)H * hd);
    double *x1 = (double *)malloc(sizeof(double) * (size_t)d);
    double *h2 = (double *)malloc(sizeof(double) * (size_t)d);
    double *gu = (double *)malloc(sizeof(double) * (size_t)2 * I);
    double *a = (double *)malloc(sizeof(double) * (size_t)I);
    for (int hh = 0; hh < H; ++hh)
      orc_attend_paged(q + (size_t)hh * hd, pool_k, pool_v, bt, B, Hkv, hd, hh / grp, pos,
                       o + (size_t)hh * hd);
    for (int j = 0; j < H * hd; ++j) o[j] = store_point(c, o[j]);            /* R3 */
    orc_linear_row(o, w->w_o, NULL, H * hd, d, x1);
    for (int j = 0; j < d; ++j) x1[j] += x[(size_t)row * d + j];             /* step 6 */
    orc_rmsnorm_row(x1, w->g_mlp, d, c->rms_eps, h2);
    for (int j = 0; j < d; ++j) h2[j] = store_point(c, h2[j]);               /* R4 */
    orc_linear_row(h2, w->w_gate_up, NULL, d, 2 * I, gu);
    for (int j = 0; j < I; ++j) a[j] = store_point(c, silu(gu[j]) * gu[I + j]); /* R5 */
    orc_linear_row(a, w->w_down, NULL, I, d, out + (size_t)row * d);
    for (int j = 0; j < d; ++j) out[(size_t)row * d + j] += x1[j];           /* step 9 */
    if (q_out) memcpy(q_out + (size_t)row * H * hd, q, sizeof(double) * (size_t)H * hd);
    if (o_out) memcpy(o_out + (size_t)row * H * hd, o, sizeof(double) * (size_t)H * hd);
    if (a_out) memcpy(a_out + (size_t)row * I, a, sizeof(double) * (size_t)I);
    free(o); free(x1); free(h2); free(gu); free(a);
  }
  free(row_req); free(row_pos); free(inv_freq); free(q_all);
  return 0;
}

/* Thread count for the OpenMP loops above (timing only: the 1-core run of
 * the CPU baseline, SURVEY §8d "Oracle timing"); n <= 0 restores all cores.
 * Results do not depend on it: every parallel loop writes disjoint rows. */
#ifdef _OPENMP
#include <omp.h>
#endif
int orc_set_threads(int n) {
#ifdef _OPENMP
  omp_set_num_threads(n > 0 ? n : omp_get_num_procs());
  return omp_get_max_threads();
#else
  (void)n;
  return 1;
#endif
}
