/*
 * bullet.h — C ABI of the Bullet co-run hot path on B200 (sm_100a).
 *
 * Bullet runs a prefill batch and a decode batch of an LLM at the same time
 * on disjoint SM partitions of one GPU, re-deciding the partition every
 * layer-level scheduling cycle with a roofline performance model
 * (§3.1).  This library is the data-parallel
 * hot path of that method:
 *
 *   bullet_create          model + KV pool, SM probe            (§3.5.2; §3.4)
 *   bullet_step            one co-run layer step, both phases   (§3.1 step 5 P:L131; §3.3.1)
 *   bullet_model_predict   Eq. 1 + Eq. 2 + T_m
 *   bullet_choose_split    Alg. 1 + §3.3.3 search
 *
 * Conventions (every call):
 *   - Returns BULLET_OK (0) or a negative BULLET_E* code; bullet_last_error()
 *     gives a thread-local message.  Argument validation happens before any
 *     work is enqueued; a failed call enqueues nothing.
 *   - Pointers named d_* / documented "device" are CUDA device pointers;
 *     h_* / "host" are host pointers.  No C++ types, exceptions or torch
 *     types cross this boundary.  Streams are cudaStream_t passed as void*.
 *   - Ownership: the caller owns weights, KV pools, hidden buffers, block
 *     tables and streams, and keeps them alive while the handle uses them.
 *     The handle owns its workspace, work counters, RoPE table and NCCL
 *     communicators.
 *   - Element types: dtype BULLET_DTYPE_BF16 -> weights, KV pool and
 *     activations are bf16; BULLET_DTYPE_FP32 -> all fp32 (tiny config).
 *     The residual stream `hidden` is always fp32.
 *   - The library has no CPU fallback: without a usable sm_100 device
 *     bullet_create fails with BULLET_ECUDA / BULLET_EUNSUPPORTED.
 */
#ifndef BULLET_H
#define BULLET_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bullet_handle bullet_handle;

enum {
  BULLET_OK = 0,
  BULLET_EINVAL = -1,        /* bad argument / shape */
  BULLET_ECUDA = -2,         /* CUDA runtime or driver error */
  BULLET_ENCCL = -3,         /* NCCL error (tensor parallel) */
  BULLET_ESMRANGE = -4,      /* prefill_sm_count out of [0, N] or off-granularity */
  BULLET_EKV = -5,           /* block id out of range / request exceeds its block table */
  BULLET_ENOMEM = -6,        /* workspace allocation failed or batch exceeds max_* */
  BULLET_EUNSUPPORTED = -7   /* shape the kernels do not support (see bullet_create) */
};

enum { BULLET_DTYPE_FP32 = 0, BULLET_DTYPE_BF16 = 1 };

/* bullet_step flags */
enum {
  BULLET_CORUN = 0,          /* phases concurrently on disjoint SM ranges (the method) */
  BULLET_TIMESLICED = 1,     /* same kernels on all SMs, prefill then decode (baseline) */
  BULLET_UNGATED = 2,        /* both phases concurrently on all SMs ("Naive") */
  BULLET_SMID_LOG = 4,       /* record (launch, tile, smid) of every work unit */
  BULLET_PROFILE = 8,        /* CUDA events around every kernel (bullet_profile_read) */
  BULLET_UNFUSED = 16,       /* run S3 (RoPE + KV append) as its own kernel instead of the
                                QKV GEMM epilogue (bf16, head_dim 128); A/B tests only */
  BULLET_UNFUSED_NORM = 32,  /* run S6 / the next layer's S1 (RMSNorm) as their own kernels
                                instead of the tail of the O-proj / down GEMM; A/B tests only */
  BULLET_CHECK_KV = 128,     /* validation (host, before enqueue): EKV if a KV block used by a
                                prefill request is also used by a decode request (the
                                phases run concurrently: shared blocks would race) */
  BULLET_DEVICE_SPLIT = 64   /* CORUN: kernels read the phases' SM sets from device memory
                                (bullet_set_split) instead of kernel arguments, so one CUDA
                                graph captured from the step follows any later split
                                (SURVEY §8f NEXT-4); prefill_sm_count / the ranges still size
                                the GEMM plans */
};

/* Kernel kinds reported by bullet_profile_read. */
enum {
  BULLET_K_PLAN = 0, BULLET_K_RMSNORM1 = 1, BULLET_K_QKV = 2, BULLET_K_ROPE_KV = 3,
  BULLET_K_ATTN = 4, BULLET_K_OPROJ = 5, BULLET_K_RMSNORM2 = 6, BULLET_K_GATE_UP = 7,
  BULLET_K_DOWN = 8, BULLET_K_ALLREDUCE = 9
};

/* Model shape (per GPU under tensor parallelism: n_heads, n_kv_heads and
 * d_ff are the LOCAL counts; d_model is the full hidden size).  The layer is
 * the Llama pre-norm block (reading R-1; the paper names only
 * QKV-projection, attention, O-projection and MLP). */
typedef struct {
  int n_layers;              /* layers whose weights/pools are registered */
  int d_model, n_heads, n_kv_heads, head_dim, d_ff;
  float rms_eps;
  double rope_theta;
  int rope_llama3;           /* 1: llama3 inv_freq rescaling (Llama-3.1) */
  float rope_factor, rope_low_freq, rope_high_freq;
  int rope_orig_max_pos;
  int max_position;          /* RoPE table length (max token position + 1) */
  int qkv_bias;              /* 1: b_qkv present (Qwen2.5) */
  int dtype;                 /* BULLET_DTYPE_* */
  int tp_size, tp_rank;      /* 1, 0 without tensor parallelism */
  int max_prefill_tokens;    /* workspace sizing, prefill phase */
  int max_decode_tokens;     /* workspace sizing, decode phase */
} bullet_model_cfg;

/* KV pool: one K and one V array per layer, each
 * [n_blocks][n_kv_heads][block_size][head_dim] of dtype, row-major.  Token
 * position p of a request lives in block block_table[r][p / block_size] at
 * offset p % block_size (index table shared by both phases; a request
 * moving from prefill to decode keeps its block-table row — copy-free). */
typedef struct {
  void *const *d_k;          /* host array of n_layers device pointers */
  void *const *d_v;
  int n_blocks, block_size;
} bullet_kv_pool;

/* Weights of one layer, device pointers, row-major [out][in] (nn.Linear):
 *   w_qkv     [(H+2Hkv)*hd][d]   rows: q heads, then k heads, then v heads
 *   b_qkv     [(H+2Hkv)*hd]      or NULL when qkv_bias == 0
 *   w_o       [d][H*hd]
 *   w_gate_up [2*I][d]           rows [0,I) gate, [I,2I) up
 *   w_down    [d][I]
 *   g_attn, g_mlp [d]            RMSNorm gains
 * bf16 (or fp32 for BULLET_DTYPE_FP32); b_qkv and gains also of dtype. */
typedef struct {
  const void *w_qkv, *b_qkv, *w_o, *w_gate_up, *w_down, *g_attn, *g_mlp;
} bullet_layer_weights;

/* One phase's batch.  Request r has ctx_lens[r] tokens cached and
 * q_len_r = cu_seqlens[r+1] - cu_seqlens[r] new tokens at positions
 * ctx_lens[r] .. ctx_lens[r] + q_len_r - 1.  Prefill: ctx 0 (any ctx works);
 * decode: q_len 1.  `hidden` rows are the new tokens, request-major; it is
 * read as x and overwritten with the layer output (fp32 residual stream).
 * The batch runs layers [layer_begin, layer_end) in order.
 * Hybrid (chunked-prefill) batches: requests with q_len > 1 first (prefill
 * chunks, any ctx), then requests with q_len 1 (decodes); attention then runs
 * the prefill kernel over the chunks and the decode kernel over the rest
 * (the SARATHI-style baseline of SURVEY §8(f) NEXT-3: pass it as the
 * prefill batch with mode TIMESLICED and no decode batch). */
typedef struct {
  int n_reqs, n_tokens, max_blocks_per_req;
  const int32_t *d_cu_seqlens;   /* device [n_reqs+1] */
  const int32_t *d_ctx_lens;     /* device [n_reqs] */
  const int32_t *d_block_table;  /* device [n_reqs][max_blocks_per_req] */
  const int32_t *h_cu_seqlens;   /* host mirrors (validation, planning) */
  const int32_t *h_ctx_lens;
  const int32_t *h_block_table;  /* host mirror; NULL skips block-id validation */
  float *d_hidden;               /* device [n_tokens][d_model] fp32, in/out */
  int layer_begin, layer_end;
} bullet_batch;

/* Batch shape for the performance model (host arrays). */
typedef struct {
  int n_reqs;
  const int32_t *q_lens;         /* new tokens per request */
  const int32_t *ctx_lens;       /* cached tokens per request */
} bullet_batch_shape;

/* Scheduler state S_k = (P_k, D_k, R_k), P:L193 (§3.3.2); host arrays. */
typedef struct {
  int layers_done, total_layers;          /* l_k, total_layers (Alg. 1 l.3) */
  int n_prefill;                          /* running prefill requests */
  const int32_t *prefill_lens;
  const double *prefill_waited_ms;        /* q_i */
  int n_pending;                          /* w_k */
  const int32_t *pending_lens;
  const double *pending_waited_ms;
  int n_decode;                           /* n_d */
  const int32_t *decode_tokens;           /* o_i: tokens generated so far */
  const double *decode_elapsed_ms;        /* d_i: decode time so far */
  double decode_mean_ctx;
  int u_k, v_k;                           /* current prefill / decode SMs */
} bullet_sched_state;

/* SLOs (Table 2) and search bounds. */
typedef struct {
  double ttft_norm_ms_per_tok;   /* normalized TTFT: Gamma_ttft(r) = value * input_len_r */
  double tpot_ms;
  int w_max;                     /* W_max, Alg. 1 l.18 */
  int v_min;                     /* minimum decode SMs when co-running */
  double percentile;             /* 0.9 (Alg. 1 "P90") */
  int objective;                 /* 0: Alg. 1 as read (DESIGN R-14..R-17); 1: when both SLOs hold,
                                    the split with the most predicted tokens/s among the SLO-feasible
                                    ones instead of the fewest decode SMs, or the time-sliced cycle
                                    if it beats them (R-21, R-22); 2: when both SLOs hold, the
                                    SLO-feasible split and decode layer-steps k with the largest
                                    predicted gain of the co-run cycle over the same work
                                    time-sliced, or the time-sliced cycle (prefill_sm_count = N,
                                    k > 0) when no split gains (R-23) */
} bullet_slo;

/* Create a handle on the current CUDA device.  Probes the live SM ids
 * (%smid) and orders them (sigma).  `nccl_uids`: for tp_size > 1, 2 x 128
 * bytes (ncclUniqueId of the prefill and the decode communicator, same on
 * every rank) for the NCCL all-reduce, or NULL for the fused peer-memory
 * all-reduce (PEER mode, bullet_tp_connect below); NULL if tp_size = 1.  `perf_params_json`: fitted perf-model
 * parameters, or NULL for the unfitted roofline (d = p = 1).
 * Unsupported shapes (BULLET_EUNSUPPORTED): bf16 with d_model, H*hd or d_ff
 * not multiples of 64; (H+2Hkv)*hd, d_model or d_ff not multiples of 64;
 * head_dim != 128 for bf16 (64 or 128 for fp32); block_size not in {16}. */
int bullet_create(const bullet_model_cfg *cfg, const bullet_kv_pool *pool,
                  const void *nccl_uids, const char *perf_params_json,
                  bullet_handle **out);

/* Host-only handle for the performance model (no GPU, no allocations):
 * bullet_model_predict and bullet_choose_split behave as on a full handle
 * with N = n_sms SMs; every GPU call on it returns BULLET_EUNSUPPORTED.
 * For planning on a host without a GPU and for CPU tests. */
int bullet_perf_create(const bullet_model_cfg *cfg, int n_sms, const char *perf_params_json,
                       bullet_handle **out);

/* Register the weights of one layer (pointers are kept, not copied). */
int bullet_set_layer_weights(bullet_handle *h, int layer, const bullet_layer_weights *w);

/* SM count N of the device and the split granularity (2 = one TPC). */
int bullet_num_sms(const bullet_handle *h, int *n_sms, int *granularity);

/* Copy the probed ordered SM list sigma (host int32 [N]) — prefill gets
 * sigma[0:p), decode sigma[p:N) for prefill_sm_count p.  Order (SURVEY §8a
 * SG; env BULLET_SIGMA read at create): "sorted" smid order (default; TPC
 * pairs adjacent), "die" (the TPCs of one die, then the other's) or
 * "interleave" (alternating dies TPC by TPC), dies from the die probe. */
int bullet_sm_order(const bullet_handle *h, int32_t *h_sigma, int cap);

/* Die (0 / 1) of each SM of sigma, in sigma order (host int32 [N]), from the
 * die probe at create: an L2 hit on an SM's own die is faster than one on
 * the other die; -1 everywhere when the probe was inconclusive. */
int bullet_sm_dies(const bullet_handle *h, int32_t *h_die, int cap);

/* Number of kernel launches so far whose last CTA found every other CTA of
 * its grid outside the phase's SM range and did the work where it landed
 * (gate_enter's liveness guard: correct, but off-range).  0 in a healthy
 * run; synchronizes the device. */
int bullet_gate_fallbacks(bullet_handle *h, long long *n);

/* One layer step: the prefill batch runs its layers on stream s_prefill and
 * the decode batch runs its layers on stream s_decode.  With BULLET_CORUN
 * every kernel of the prefill phase claims work only on the first
 * prefill_sm_count SMs of sigma and every decode kernel only on the rest
 * (smid-gated persistent kernels; replaces libsmctrl masks over MPS,
 * P:L212).  prefill_sm_count = N pauses decode; 0 requires an empty
 * prefill.  Either batch may be NULL.  Asynchronous: enqueue only.
 * Ordering is the caller's: everything the step reads (hidden, tables,
 * pools, weights) must already be complete or ordered before s_prefill /
 * s_decode (e.g. cudaStreamWaitEvent); the step orders only its own kernels
 * (back to back on each stream).
 * Errors: EINVAL (shapes), ESMRANGE (split), EKV (block table), ENOMEM
 * (batch larger than cfg max_*). */
int bullet_step(bullet_handle *h, const bullet_batch *prefill, const bullet_batch *decode,
                int prefill_sm_count, int flags, void *s_prefill, void *s_decode);

/* bullet_step (BULLET_CORUN only) with explicit SM ranges of sigma: the
 * prefill phase claims work on sigma[pre_lo, pre_hi), decode on
 * sigma[dec_lo, dec_hi).  The ranges may overlap (non-strict partition,
 * SURVEY §8(f) NEXT-4): an SM in both ranges runs whichever
 * phase's CTA it receives, so a phase that finishes its kernels early leaves
 * the shared band to the other.  Bounds on the TPC granularity within [0, N];
 * a non-empty batch needs a non-empty range.  Errors as bullet_step. */
int bullet_step_ranges(bullet_handle *h, const bullet_batch *prefill, const bullet_batch *decode,
                       int pre_lo, int pre_hi, int dec_lo, int dec_hi, int flags, void *s_prefill,
                       void *s_decode);

/* BULLET_DEVICE_SPLIT: enqueue on `stream` the write of the device-resident
 * SM sets — prefill on sigma[pre_lo, pre_hi), decode on sigma[dec_lo, dec_hi)
 * (granularity and bounds as bullet_step_ranges; the ranges may overlap).
 * Steps (or replays of graphs captured from steps) with BULLET_DEVICE_SPLIT
 * that are ordered after it on the device use these sets.  Not captured into
 * a graph by itself: call it outside capture, before each replay that needs
 * a new split.  Initially every SM belongs to both phases.  A phase whose
 * set holds none of its CTAs still completes (the grid's last CTA works
 * wherever it landed — correct, slow).  Errors: ESMRANGE. */
int bullet_set_split(bullet_handle *h, int pre_lo, int pre_hi, int dec_lo, int dec_hi, void *stream);

/* Eq. 2 / T_m: predicted time (microseconds) of one layer of the given
 * batch on sm_count SMs; corun_sm_count > 0 applies the co-location factors
 * p_c, p_b. */
int bullet_model_predict(const bullet_handle *h, const bullet_batch_shape *shape, int sm_count,
                         int corun_sm_count, double *t_layer_us);

/* Online estimator feedback ("correlating deviations between
 * predicted latency and observed execution times across scheduling cycles,
 * using the inter-cycle duration t_{k+1} - t_k as dynamic feedback"): read /
 * replace the scale applied to the fitted co-location factors p_c(m), p_b(m)
 * of Eq. 2 (default 1) that every co-run prediction (corun_sm_count > 0) and
 * bullet_choose_split use.  Errors: EINVAL (non-positive factors). */
int bullet_get_colocation(const bullet_handle *h, double *p_c, double *p_b);
int bullet_set_colocation(bullet_handle *h, double p_c, double p_b);

/* The same feedback for the model's level: every predicted layer
 * time of a prefill-shaped batch (some request with more than one new
 * token) is multiplied by `pre`, of a decode-shaped batch by `dec` (default
 * 1; e.g. measured / predicted full-GPU layer time of the live batch).
 * Errors: EINVAL (non-positive scales). */
int bullet_get_phase_scale(const bullet_handle *h, double *pre, double *dec);
int bullet_set_phase_scale(bullet_handle *h, double pre, double dec);

/* Alg. 1 and the §3.3.3 search under the readings
 * of DESIGN.md §3 (R-14..R-17): returns the prefill SM count for the next
 * cycle (N = decode paused) and the number of decode layer-steps to co-run
 * with one prefill layer-step. */
int bullet_choose_split(const bullet_handle *h, const bullet_sched_state *s, const bullet_slo *slo,
                        int *prefill_sm_count, int *decode_layer_steps);

/* Device buffer for the smid log used with BULLET_SMID_LOG: int32
 * [1 + 4*capacity]; entry i = {launch_id, unit, smid, phase}; element 0 is
 * the entry counter (caller zeroes it).  NULL disables. */
int bullet_set_smid_log(bullet_handle *h, int32_t *d_log, int capacity);

/* Per-kernel device times of every launch made by bullet_step calls with
 * BULLET_PROFILE since the last read (oldest first): kind (BULLET_K_*),
 * phase (0 prefill, 1 decode), layer, milliseconds between CUDA events
 * recorded on the launching stream around the kernel.  Synchronizes on the
 * events; *n = number written (<= cap); the list is then cleared. */
int bullet_profile_read(bullet_handle *h, int32_t *kind, int32_t *phase, int32_t *layer, float *ms,
                        int cap, int *n);

/* Total kernels this handle has launched (all entry points). */
int bullet_launch_count(const bullet_handle *h, long long *n);

/* Diagnostics (DESIGN.md §5 "where the time goes"): per-CTA device
 * timestamps (%globaltimer, ns) of the next `max_launches` kernel launches
 * of this handle.  Each launch gets BULLET_TRACE_CTAS records of 16 uint64:
 * {smid, entry, first operand stage ready, MMA issue done, epilogue done,
 * exit, work units, last partial stored, first fixup start, last fixup end,
 * fixups, 0...}; CTAs that left their SM range (or kernels that only record
 * entry / exit) leave zeros.  max_launches = 0 disables (default).
 * The handle owns the device buffer.  BULLET_ENOMEM if it cannot be
 * allocated. */
enum { BULLET_TRACE_CTAS = 2368 };
int bullet_trace_enable(bullet_handle *h, int max_launches);

/* Copy the recorded launches (oldest first, *n <= cap) to host memory:
 * rec [cap][BULLET_TRACE_CTAS][16], meta [cap][4] = {kind (BULLET_K_*),
 * phase, layer, grid}; then restart recording.  Synchronizes the device. */
int bullet_trace_read(bullet_handle *h, uint64_t *rec, int32_t *meta, int cap, int *n);

/* Block until all work the handle enqueued has finished; surfaces
 * asynchronous CUDA / NCCL errors and peer all-reduce timeouts (ENCCL). */
int bullet_sync(bullet_handle *h);

/* ncclGetUniqueId into out (128 bytes), for tensor-parallel setup. */
int bullet_nccl_unique_id(void *out128);

/* ---- Fused tensor-parallel all-reduce over peer memory (
 * north_star (4): "an NCCL all-reduce over NVLink after the attention-out and
 * MLP-down projections", here fused into those GEMMs and smid-gated).
 * A handle created with tp_size > 1 and nccl_uids == NULL is in PEER mode:
 * bullet_create allocates one symmetric device region (same layout on every
 * rank: per phase two fp32 partial buffers [max_tokens][d_model], the fp32
 * residual stream `hidden` [max_tokens][d_model], ready / done counters).
 * Before the first step every rank connects to all ranks' regions (its own
 * included) with bullet_tp_connect (device addresses valid in this process:
 * same-process ranks, e.g. ranks simulated on SM partitions of one GPU) or
 * bullet_tp_connect_ipc (cudaIpcMemHandle_t of every rank, one process per
 * GPU; rank order).  In a step, the O-proj and down GEMMs of rank r write
 * fp32 partials into r's region and the same kernels then reduce rank r's
 * column slab [r d/n, (r+1) d/n) of every 16-row chunk as soon as all ranks'
 * partials of its 128-row block are ready (x + partial_0 + ... +
 * partial_{n-1}, fixed rank order: deterministic), store it into every
 * rank's hidden and return once all slabs have arrived.
 * Every batch passed to bullet_step must use the phase's symmetric hidden
 * (bullet_tp_hidden) as its `d_hidden` (else EINVAL); all ranks must make the
 * same sequence of steps with the same batch shapes (as with NCCL).  bf16
 * only.  A peer that never arrives makes the waiting kernels give up after
 * 20 s; bullet_sync then returns BULLET_ENCCL. */

/* Device address of this handle's symmetric region (PEER mode). */
int bullet_tp_base(const bullet_handle *h, void **d_base);

/* cudaIpcMemHandle_t (64 bytes) of this handle's symmetric region. */
int bullet_tp_ipc_handle(const bullet_handle *h, void *out64);

/* Connect to the tp_size regions `d_bases` (rank order; d_bases[tp_rank]
 * must be this handle's own).  Errors: EINVAL (not PEER mode, wrong own
 * base, null), EUNSUPPORTED (tp_size > 8). */
int bullet_tp_connect(bullet_handle *h, void *const *d_bases);

/* Open the other ranks' regions from tp_size x 64 bytes of IPC handles (rank
 * order, as gathered from every rank's bullet_tp_ipc_handle) and connect.
 * The handle closes them in bullet_destroy.  Errors: ECUDA (open failed). */
int bullet_tp_connect_ipc(bullet_handle *h, const void *handles);

/* The phase's (0 prefill, 1 decode) symmetric residual stream, fp32
 * [cfg max tokens of the phase][d_model]: the `d_hidden` of PEER-mode steps. */
int bullet_tp_hidden(const bullet_handle *h, int phase, float **d_hidden);

const char *bullet_last_error(void);
void bullet_destroy(bullet_handle *h);

/* ---- op-level entry points (the same kernels bullet_step launches), for
 * per-kernel parity tests.  All run on `stream` over the SMs of sigma[lo:hi)
 * (lo = 0, hi = N for the whole GPU). ---- */

/* C = A B^T with the epilogue `epi` (bf16 A [M][K], B [rowsB][K] for
 * BULLET_DTYPE_BF16 handles; fp32 otherwise):
 *   0 F32:      out_f32[M][N] = acc (+ bias[N])                (QKV)
 *   1 RESID:    out_f32[M][N] = resid[M][N] + acc (in place OK) (O-proj, down)
 *   2 SILU_MUL: out[M][N/2] = silu(acc[:, j]) * acc[:, silu_half + ... ]:
 *               B rows [0, N/2) gate, [silu_half, silu_half + N/2) up;
 *               out of dtype                                    (gate_up)
 * N = number of B rows used (2 x output columns for SILU_MUL). */
/* epi | BULLET_GEMM_PACKED: first repack B into the pre-swizzled tile layout
 * that bullet_step uses for weights (kernels.h), then run the bulk-copy path. */
enum { BULLET_GEMM_PACKED = 256 };
int bullet_op_gemm(bullet_handle *h, int epi, const void *d_A, int M, int K, const void *d_B,
                   int N, int silu_half, const void *d_bias, const float *d_resid, void *d_out,
                   int lo, int hi, void *stream);

/* KI2 microbenchmark: stream `bytes` (multiple of 64 KB) from d_src on the
 * SMs sigma[lo:hi) and discard them; mode 0 LDG.128, 1 cp.async.bulk (TMA
 * bulk copies), 2 cp.async 16 B; mode | (param << 8): LDG with `param` warps
 * per SM, cp.async with `param` 64 KB units in flight.  KI2, DESIGN.md §5. */
int bullet_op_stream(bullet_handle *h, const void *d_src, size_t bytes, int mode, int lo, int hi,
                     void *stream);

/* KI3 microbenchmark (not gated; n_ctas CTAs in clusters of 2, one per SM):
 * stream `bytes` (multiple of 32 KB) into shared memory in 32 KB stages; mc = 1:
 * each CTA fetches half of every stage with a .multicast::cluster bulk copy
 * into both CTAs, mc = 0: each CTA fetches the whole stage.  Measures whether
 * multicast lifts the per-SM async-copy ceiling. */
int bullet_op_stream_mc(bullet_handle *h, const void *d_src, size_t bytes, int mc, int n_ctas, void *stream);

int bullet_op_rmsnorm(bullet_handle *h, const float *d_x, int n, const void *d_g, void *d_out,
                      int lo, int hi, void *stream);

/* RoPE + KV append for `batch` rows: qkv fp32 [n_tokens][(H+2Hkv)*hd] in,
 * q out [n_tokens][H*hd] (dtype), k/v written to the pool of `layer`. */
int bullet_op_rope_kv(bullet_handle *h, const bullet_batch *batch, int layer, const float *d_qkv,
                      void *d_q, int lo, int hi, void *stream);

/* Attention for `batch` rows reading K/V of `layer` through the block
 * table: q [n_tokens][H*hd] in, o [n_tokens][H*hd] out (dtype).
 * kind 0: automatic (what bullet_step uses), 1: SIMT kernel, 2: mma.sync
 * prefill kernel, 3: tensor-core decode kernel, 4: tcgen05 prefill kernel
 * (2-4: bf16, head_dim 128). */
int bullet_op_attention(bullet_handle *h, const bullet_batch *batch, int layer, const void *d_q,
                        void *d_o, int kind, int lo, int hi, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* BULLET_H */
