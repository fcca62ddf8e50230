// kernels.h — argument structs and launchers of the Bullet sm_100a kernels.
#pragma once
#include "common.cuh"
#include <utility>

namespace bl {

enum { EPI_F32 = 0, EPI_RESID = 1, EPI_SILU = 2, EPI_QKV = 3 };

// Per-token position and KV slot of a phase's batch (plan kernel, once per
// step): x = position p = ctx[r] + (t - cu[r]), y = slot = bt[r][p / B] * B + p % B.
typedef int2 TokInfo;

// Fused tensor-parallel all-reduce over peer memory (SURVEY §8f NEXT-2,
// DESIGN.md §8).  A row-parallel GEMM (O-proj, down) of rank `rank` writes its
// fp32 partial into its symmetric partial buffer and, per finished 128-row
// block, adds the block's column count to ready[rank][rb] on every rank.
// When its own tiles run out, each CTA turns to reduce units: 16 rows of
// this rank's column slab [rank N/n, (rank+1) N/n) — wait until every rank's
// partial of the block is ready, sum x + partial_0 + ... + partial_{n-1} in
// rank order (deterministic), store the result into every rank's hidden and
// count the chunk in done[rb] on every rank — then to wait units (one per
// row block) that return once all n slabs of the block have landed here.  The
// kernel ends with hidden = x + sum of partials on every rank.  Counters only
// grow; `base` holds the values expected before this all-reduce
// ([0, max_rb): ready, [max_rb, 2 max_rb): done), advanced by the wait units.
constexpr int AR_MAX_RANKS = 8, AR_ROWS = 16;
struct ArArgs {
  int n, rank, max_rb;                              // n = 0: off
  float* part[AR_MAX_RANKS];                        // rank s's partial buffer [M][N] (this all-reduce's parity)
  float* hid[AR_MAX_RANKS];                         // rank s's hidden [M][N]
  unsigned long long* ready[AR_MAX_RANKS];          // rank s's ready counters [n][max_rb]
  unsigned long long* done[AR_MAX_RANKS];           // rank s's done counters [max_rb]
  unsigned long long* base;                         // local [2][max_rb]
  int* ctr;                                         // reduce / wait unit counter (zero at launch)
  int* err;                                         // set on a peer timeout
};

// RMSNorm fused into the tail of a residual GEMM (EPI_RESID; S6 after the
// O-proj, the next layer's S1 after down): every finished tile adds its
// column count to rb_ctr[128-row block]; once a CTA's GEMM units run out it
// claims rows from unit_ctr, waits until the row's block holds all N columns
// and normalises the row exactly as k_rmsnorm does (same reduction order:
// bit-identical), out = bf16(x * rsqrt(mean x^2 + eps) * g).
struct NormFuse {
  const void* g; void* out;   // out == nullptr: off
  float eps;
  int* rb_ctr;                // [ceil(M / 128)], zero at launch
  int* unit_ctr;              // zero at launch
  int rows;                   // rows per claim (1, 2, 4): several rows' loads in flight per CTA
};

// C[M x N] = A[M x K] . B[N x K]^T with a fused epilogue (all row-major).
struct GemmArgs {
  int M, N, K;        // N = B rows used (2 x output cols for EPI_SILU)
  int bn;             // tile width in B rows (tcgen05: 64/128/256; SIMT: 64)
  int mh;             // tcgen05: 128-row halves per unit (1, or 2 = 256 rows sharing each B stage)
  int n_full;         // tcgen05: units [0, n_full) are whole tiles over all of K ...
  int sk_tiles;       // ... the remaining sk_tiles tiles are streamed: their k-block iterations
  int sk_chunks;      //     cut into sk_chunks equal ranges (units n_full + c), gemm_tc.cu
  int band;           // tcgen05: M tiles per rasterisation band (see tile_coords)
  int epi;
  int silu_half;      // row offset of the "up" rows in B (EPI_SILU)
  const void* bias;   // [N] of the element type, or null (EPI_F32)
  const float* resid; // [M][ldo] (EPI_RESID; may alias out_f32)
  float* out_f32;     // [M][ldo] (EPI_F32, EPI_RESID)
  void* out_t;        // [M][ldo] of the element type (EPI_SILU)
  int ldo;
  float* partials;    // stream part: [2 sk_chunks slots][mh][bn/4][128][4] (float4 groups interleaved by row)
  int* tile_sems;     // stream part: [2][2048] segments stored per streamed tile; launch L
  int sk_parity;      // counts in slice sk_parity and zeroes the other one for launch L + 1
  int* fix_ctr;       // stream part: fixup item counter, zero at launch
  const uint8_t* b_packed;  // B pre-packed by pack_weight (else B comes through mapB)
  int b_evict_first;        // one M tile: the weight stream is used once (L2 evict-first)
  int b_rows;               // rows of B (packed layout stride)
  int split_b;              // 1: warp 3 issues the B tiles (second copy issuer), warp 0 the A tiles
  int b_pf;                 // warp 3 prefetches packed B k-block kb + b_pf into L2 (0 = off)
  int epi_coal;             // EPI_RESID / EPI_SILU whole tiles: rows transposed through shared memory so the
                            // warp's global loads / stores cover whole row segments (1 = on)
  int epi_pf;               // epilogue warps L2-prefetch their tile's inputs (residual rows, RoPE rows)
                            // when they learn the unit, i.e. while the mainloop streams (1 = on)
  int epi_dbg;              // diagnostics (BULLET_GEMM_EPI_DBG; wrong results): bit 0 no SiLU math,
                            // bit 1 no output stores, bit 2 no residual loads, bit 3 no RoPE-table loads,
                            // bit 4 no two-level-accumulation merge, bit 5 one accumulation chunk per tile
  int kcb;                  // two-level accumulation (DESIGN R-4e): K chunk in k-blocks (0 = off);
                            // each chunk accumulates in TMEM, the chunks are summed in fp32
                            // registers by the epilogue (requires mh == 1, bn == 128, whole tiles)
  // EPI_QKV (bf16, head_dim 128; fuses SURVEY §8a S3 into S2): the epilogue
  // adds the bias, rotates q / k heads (rotate-half RoPE from the (cos, sin)
  // table), rounds to bf16 (point R2) and stores q -> q_out[t][H][128],
  // k / v -> the paged pool slot of token t.  Tiles cover whole heads.
  void* q_out; void* pool_k; void* pool_v;
  const float2* cs;         // [max_pos][64] (cos, sin)
  const TokInfo* tok;       // [M]
  int H, Hkv, kvB;
  ArArgs ar;                // EPI_F32 into ar.part[ar.rank] + the fused all-reduce (ar.n > 1)
  NormFuse nf;              // EPI_RESID + RMSNorm of the finished rows (nf.out != nullptr)
  Launch L;
};

// Packed weight layout: W[R][K] bf16 -> [K/64][R/64] tiles of 64 rows x 64 k
// (8 KB), each stored as the 128-byte-swizzled shared-memory image a TMA
// SWIZZLE_128B load would produce (16-byte chunk c of row r at c ^ (r & 7)).
// A B-operand stage of bn rows at k-block kb is then one or two contiguous
// bulk copies.
cudaError_t launch_pack_weight(const __nv_bfloat16* W, int R, int K, uint8_t* out, cudaStream_t st);

struct NormArgs {
  const float* x; const void* g; void* out;
  int n, d; float eps;
  Launch L;
};

struct RopeArgs {
  const float* qkv; void* q_out; void* pool_k; void* pool_v;
  const float2* cs;   // [max_pos][hd/2] (cos, sin)
  const int32_t* cu; const int32_t* ctx; const int32_t* bt;
  int n_reqs, max_blocks, n_tok, H, Hkv, hd, B, max_pos;
  Launch L;
};

struct AttnArgs {
  const void* q; void* o; const void* pool_k; const void* pool_v;
  const int32_t* cu; const int32_t* ctx; const int32_t* bt;
  int n_reqs, max_blocks, n_tok, H, Hkv, hd, B;
  float scale;
  const int2* tiles;      // prefill tensor-core kernel: (request, q-tile) list
  const int* n_tiles;     // device count of `tiles`
  int dbg;                // diagnostics (BULLET_DBG env): bit0 = decode consumers skip math
  int tok_base;           // decode kernel: its rows are tokens [tok_base, n_tok) (mixed batches)
  const int4* order;      // decode kernel (nullable): unit row i -> (token - tok_base, request, position, -),
                          // longest context first; saves the claimer its per-unit request search
  int kv_chunks;          // decode kernel: KV chunks of attn_decode_max_blocks() blocks per unit (split-KV
                          // for longer contexts; 1 = none); partial (O, m, l) per chunk merged in order
  float* kv_part;         // [units][kv_chunks][8][128 + 2] (kv_chunks > 1)
  int* kv_tick;           // [units], zero between launches (self-resetting)
  int dec_pf;             // decode kernel: L2 prefetch distance (blocks of a warp's stream; 0 = off)
  int kv_tma;             // tcgen05 prefill: Q and full K/V tiles by TMA; decode: K/V blocks by TMA (else cp.async)
  Launch L;
};

struct StreamArgs {   // KI2 streaming microbenchmark
  const uint8_t* src; size_t bytes; int mode; int param; uint32_t* sink;
  size_t wrap;        // offsets masked by wrap (window - 1): re-read an L2-resident window
  Launch L;
};

struct PlanArgs {
  int* counters; int n_counters;
  const int32_t* cu; int n_reqs; int bq;
  int n_tile_reqs;    // prefill attention tiles cover requests [0, n_tile_reqs)
  int2* tiles; int* n_tiles;
  // per-token (position, slot) table (nullable): needs ctx, bt, max_blocks, B
  TokInfo* tok; const int32_t* ctx; const int32_t* bt; int max_blocks, B, n_tok;
  int* zero2; int n_zero2;   // second array zeroed per step (fused-norm row-block counters)
  // decode rows [order_base, n_tok) in descending context length (nullable): LPT order of the
  // decode attention's units (the longest rows start first, the tail is short)
  int4* order; int order_base;
};

// Launch helper: `pdl` = programmatic stream serialization (common.cuh
// pdl_wait / pdl_trigger) so the kernel may start while its predecessor on
// the stream drains.
template <typename... P, typename... A>
inline cudaError_t launch_ex(void (*k)(P...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, bool pdl,
                             A&&... args) {
  cudaLaunchConfig_t c = {};
  c.gridDim = grid; c.blockDim = block; c.dynamicSmemBytes = smem; c.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  c.attrs = at; c.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&c, k, std::forward<A>(args)...);
}

// launchers (return cudaError_t of the launch)
cudaError_t launch_gemm_tc(const CUtensorMap& mapA, const CUtensorMap& mapB, const GemmArgs& a,
                           int grid, cudaStream_t st);
size_t gemm_tc_smem_bytes(int bn, int mh);
int gemm_tc_stages(int bn, int mh);
template <typename T>
cudaError_t launch_gemm_simt(const T* A, const T* B, const GemmArgs& a, int grid, cudaStream_t st);
template <typename T>
cudaError_t launch_rmsnorm(const NormArgs& a, int grid, cudaStream_t st);
template <typename T>
cudaError_t launch_rmsnorm_warp(const NormArgs& a, int grid, cudaStream_t st);
template <typename T>
cudaError_t launch_rope_kv(const RopeArgs& a, int grid, cudaStream_t st);
template <typename T>
cudaError_t launch_attn_simt(const AttnArgs& a, int grid, cudaStream_t st);
cudaError_t launch_attn_prefill_tc(const AttnArgs& a, int grid, cudaStream_t st);
cudaError_t launch_attn_prefill5(const CUtensorMap& mk, const CUtensorMap& mv, const CUtensorMap& mq,
                                 const AttnArgs& a, int grid, cudaStream_t st);
int attn_prefill5_ctas_per_sm(int H, int Hkv);   // grid = n_sms * this (2 query tiles per CTA for even GQA groups)
cudaError_t launch_attn_decode_tc(const CUtensorMap& mk, const CUtensorMap& mv, const AttnArgs& a, int grid, int ng,
                                  cudaStream_t st);   // mk / mv as for launch_attn_prefill5 (a.kv_tma)
size_t attn_decode_smem_bytes();
// tcgen05 decode attention (attn_decode5.cu): grid = n_sms, GQA group <= 8, head_dim 128, block 16;
// mk / mv as for launch_attn_prefill5
cudaError_t launch_attn_decode5(const CUtensorMap& mk, const CUtensorMap& mv, const AttnArgs& a, int grid,
                                cudaStream_t st);
cudaError_t preload_attn_decode5();
int attn_decode_max_blocks();
cudaError_t launch_plan(const PlanArgs& a, cudaStream_t st);   // grid sized to n_tok
cudaError_t launch_stream(const StreamArgs& a, int grid, cudaStream_t st);
cudaError_t launch_stream_mc(const uint8_t* src, size_t bytes, int mc, int grid, uint32_t* sink, cudaStream_t st);
cudaError_t launch_probe(int* out_smid, int n, cudaStream_t st);
cudaError_t launch_die_probe(const void* lines, int n_lines, int stride_bytes, uint32_t* lat, int grid, cudaStream_t st);
cudaError_t launch_set_gates(Gate* d_gates, const Gate& pre, const Gate& dec, cudaStream_t st);

// Lazy module loading (CUDA default) loads a kernel at its first launch
// with a device-wide synchronisation, which can deadlock kernels that wait
// on kernels of another stream (the fused all-reduce): load every kernel at
// bullet_create instead.
cudaError_t preload_attn_decode();
cudaError_t preload_attn_prefill5();
cudaError_t preload_attn_tc();
cudaError_t preload_attn_simt();
cudaError_t preload_elementwise();
cudaError_t preload_gemm_tc();
cudaError_t preload_stream();

constexpr int ATTN_TC_BQ = 128;
constexpr int DEC_ORDER_BUCKETS = 512;   // LPT sort buckets (block counts; longer rows share the last)   // query rows per prefill attention tile (plan granularity)
constexpr int ROWS_PER_UNIT = 8;  // rows per work unit of row-wise kernels

}  // namespace bl
