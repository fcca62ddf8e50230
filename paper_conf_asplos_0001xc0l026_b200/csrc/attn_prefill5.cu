// attn_prefill5.cu — causal prefill attention on 5th-gen tensor cores
// (tcgen05 + TMEM), bf16, head_dim 128 (the paper's
// FlashAttention).
//
// Work unit = (request, 128-row query tile, NQ query heads of one KV
// group), LPT order from the plan kernel.  NQ = 2 (GQA groups of even size):
// one CTA per SM, two query tiles share every K / V tile in shared memory
// (half the gather traffic per MMA; 512 TMEM columns); NQ = 1: two CTAs per
// SM (112 KB smem, 256 TMEM columns each).  Per 64-key KV tile t and query
// tile q:
//   S_q(t) = Q_q K(t)^T  tcgen05.mma M=128 (queries) N=64 (keys) -> TMEM fp32,
//                     double-buffered so S(t+1) runs during softmax(t)
//   softmax           4 warps per query tile, thread r owns query row r = TMEM
//                     lane r: tcgen05.ld, causal mask, exp2 against a lazily
//                     moved reference max, P = hi + lo (two bf16 halves, R-4b)
//                     tcgen05.st'd over S(t) in TMEM
//   O_q += P V        tcgen05.mma with A = P from TMEM, B = V(t) used as an
//                     MN-major operand straight from its [key][dim] tile; O
//                     stays in TMEM, rescaled only when a row max grows > 2^8
// One warp issues S(t+1) and PV(t) back to back (an elected lane of the
// converged warp).  Q, K and V tiles are fed by TMA (Q: [T][H][128] boxes of
// 128 tokens x 64 dims of one head; rows past the batch read as zeros, rows
// of the next request are never stored): the pool viewed as a 2-D tensor
// [blocks * Hkv * 16 rows][128 dims] with 16 x 64-element boxes and the
// 128-byte swizzle, so a (block, head) half-chunk lands in exactly the
// swizzled layout the UMMA descriptors describe — 8 copies of 2 KB per 64-key
// operand tile, issued by one elected lane, completion counted in bytes on
// the tile's mbarrier.  The last tile of a sequence (rows past its end must
// read as zeros: P = 0 times a stale non-finite V would poison O) is gathered
// with zero-filling cp.async instead, as is every tile when a.kv_tma = 0.
// NKB K buffers (K(t) loads once S(t-NKB) is done), two V buffers.
// Measured (round 2, scripts/attn_pre_bench.py): the gathers, not the MMAs,
// bound the NQ = 1 kernel (without them it runs at 0.65 of the bf16 peak,
// with them 0.47; loading every other tile only: 0.55), hence NQ = 2.
#include "kernels.h"

namespace bl {

namespace {
constexpr int BQ = 128, BKV = 64, HD = 128, KB = 16;
template <int NQ>
struct Cfg {
  // warps [0, 4 NQ) softmax + epilogue (query tile w / 4), then the K/Q
  // loader + unit claimer, the V loader, one MMA issuer per query tile (the
  // tiles' S -> softmax -> PV chains stay independent, as with two CTAs)
  // NLW warps gather each of K (and Q) and V (the first K warp claims units)
#ifndef PF5_NLW
#define PF5_NLW 2
#endif
  static constexpr int NLW = NQ == 2 ? PF5_NLW : 1;
  static constexpr int NSW = 4 * NQ, W_LOAD = NSW, W_VLOAD = NSW + NLW, W_MMA = NSW + 2 * NLW,
                       NT = (NSW + 2 * NLW + NQ) * 32;
  static constexpr int CTAS = 2 / NQ;   // per SM
  // smem: Q [NQ][2][128][128 B] | K [NKB][2][64][128 B] | V [2][2][64][128 B] | barriers.
  // The dynamic window must start 1024-byte aligned (128-byte swizzle atoms); checked at entry.
#ifndef PF5_NKB2
#define PF5_NKB2 4
#endif
  static constexpr int NKB = NQ == 2 ? PF5_NKB2 : 3;
  static constexpr int OFF_Q = 0, OFF_K = NQ * 32768, OFF_V = OFF_K + NKB * 16384, OFF_BAR = OFF_V + 2 * 16384;
  static constexpr int SMEM_BYTES = OFF_BAR + 512;   // mbarriers, TMEM slot, unit ring
  // TMEM per query tile q (256 columns from 256 q): S/P double buffer in
  // [0,64) and [64,128) (P = bf16 hi|lo packed two per column, written over
  // the S it came from), O in [128,256)
  static constexpr uint32_t TMEM_COLS = 256 * NQ;
};

// 128-byte swizzled offset of 16-byte chunk c of `row` in a tile whose
// 64-element halves are `half` bytes apart
__device__ __forceinline__ uint32_t sw(int row, int c, int half) {
  return (c >> 3) * half + row * 128 + (((c & 7) ^ (row & 7)) << 4);
}
__device__ __forceinline__ uint64_t desc_k(uint32_t addr) {   // K-major SW128
  return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)64 << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr) {  // MN-major SW128: LBO 8 KB, SBO 1 KB
  return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)(8192 >> 4) << 16) | ((uint64_t)64 << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void tc_mma(uint32_t d, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tc_mma_ts(uint32_t d, uint32_t a_tmem, uint64_t bd, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
      "r"(a_tmem), "l"(bd), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float* v) {
  uint32_t r[32];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%"
      "15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_st32(uint32_t taddr, const float* v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%"
      "14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]),
      "f"(v[8]), "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15]),
      "f"(v[16]), "f"(v[17]), "f"(v[18]), "f"(v[19]), "f"(v[20]), "f"(v[21]), "f"(v[22]),
      "f"(v[23]), "f"(v[24]), "f"(v[25]), "f"(v[26]), "f"(v[27]), "f"(v[28]), "f"(v[29]),
      "f"(v[30]), "f"(v[31])
      : "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t* v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
      "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ void cp_async16_zfill(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(valid ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ float ex2(float x) {   // 2^x, MUFU only (ftz)
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// Blackwell packed fp32 pairs (FFMA2 / FADD2)
__device__ __forceinline__ float2 ffma2(float2 a, float b, float c) {
  unsigned long long d;
  const float2 bb = make_float2(b, b), cc = make_float2(c, c);
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d)
      : "l"(*reinterpret_cast<const unsigned long long*>(&a)), "l"(*reinterpret_cast<const unsigned long long*>(&bb)),
        "l"(*reinterpret_cast<const unsigned long long*>(&cc)));
  return *reinterpret_cast<float2*>(&d);
}
__device__ __forceinline__ float2 fadd2(float2 a, float2 b) {
  unsigned long long d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d)
      : "l"(*reinterpret_cast<const unsigned long long*>(&a)), "l"(*reinterpret_cast<const unsigned long long*>(&b)));
  return *reinterpret_cast<float2*>(&d);
}
__device__ __forceinline__ float2 fsub2(float2 a, float2 b) {
  unsigned long long d;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d)
      : "l"(*reinterpret_cast<const unsigned long long*>(&a)), "l"(*reinterpret_cast<const unsigned long long*>(&b)));
  return *reinterpret_cast<float2*>(&d);
}
__device__ __forceinline__ uint32_t pack_bf2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

struct Unit {
  int h, g, q0, tok0, q_len, ctx, kv_len, n_kt, r;   // h: first of the unit's NQ query heads
};
template <int NQ>
__device__ __forceinline__ Unit unit_of(const AttnArgs& a, int u) {
  Unit U;
  const int hq = a.H / NQ;
  const int2 rt = a.tiles[u / hq];
  U.h = (u % hq) * NQ;
  U.g = U.h / (a.H / a.Hkv);   // NQ = 2 only for even groups: both heads read KV head g
  U.r = rt.x;
  U.q0 = rt.y * BQ;
  U.tok0 = __ldg(a.cu + U.r);
  U.q_len = __ldg(a.cu + U.r + 1) - U.tok0;
  U.ctx = __ldg(a.ctx + U.r);
  U.kv_len = U.ctx + U.q_len;
  U.n_kt = (min(U.kv_len, U.ctx + U.q0 + BQ) + BKV - 1) / BKV;
  return U;
}
__device__ __forceinline__ void cp_async_arrive_noinc(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// Suspending wait (the warp sleeps until the phase completes instead of
// spinning and taking issue slots from the softmax warps).
__device__ __forceinline__ void wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, 0x989680;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// Block-table window of a loader warp: lane l holds entry 32w + l of the
// unit's block-table row for the current window w (8 KV tiles) and prefetches
// the next window, so no tile waits on a block-table load.
struct BtWin {
  int cur, nxt;
  __device__ __forceinline__ void start(const int32_t* bt, int n_blk, int lane) {
    cur = lane < n_blk ? __ldg(bt + lane) : 0;
    nxt = 32 + lane < n_blk ? __ldg(bt + 32 + lane) : 0;
  }
  // call at tile kt (kt % 8 == 0, kt > 0): window kt / 8 becomes current
  __device__ __forceinline__ void advance(const int32_t* bt, int n_blk, int kt, int lane) {
    cur = nxt;
    const int e = (kt / 8 + 1) * 32 + lane;
    nxt = e < n_blk ? __ldg(bt + e) : 0;
  }
};
// One warp gathers blocks [b0, b0 + NB) of KV tile kt (16 rows each, of head
// U.g through the block table) into a 128-byte-swizzled [2][64][128 B] tile;
// `bar` gets this warp's arrivals when they land.
template <int NB>
__device__ __forceinline__ void load_kv_tile(uint8_t* dst, const __nv_bfloat16* pool, const AttnArgs& a,
                                             const Unit& U, int kt, int lane, uint64_t* bar, const BtWin& w, int b0) {
  const int r0 = lane >> 4, c = lane & 15;   // this lane: rows r0 + 2j, 16-byte chunk c
  const int kb = kt * BKV;
  const bool full = kb + BKV <= U.kv_len;
#pragma unroll
  for (int b = b0; b < b0 + NB; ++b) {
    const int blk = __shfl_sync(0xffffffffu, w.cur, (kt % 8) * (BKV / KB) + b);
    const __nv_bfloat16* src = pool + (((size_t)blk * a.Hkv + U.g) * KB + r0) * HD + c * 8;
#pragma unroll
    for (int j = 0; j < KB / 2; ++j) {
      const int row = b * KB + r0 + 2 * j;
      const bool ok = full || kb + row < U.kv_len;
      cp_async16_zfill(dst + sw(row, c, 8192), ok ? src + j * 2 * HD : pool, ok);
    }
  }
  cp_async_arrive_noinc(bar);
}
// KV tile kt by TMA (a full tile: every row inside the sequence).  The whole
// warp calls it: the block ids come from the lanes' window, one elected lane
// arms the barrier with the tile's bytes and issues the 8 copies (4 blocks x
// 2 halves of 64 dims), the other lanes arrive plainly (the barrier counts
// 32 arrivals per loader warp whichever path fed the tile).
__device__ __forceinline__ void tma_kv_tile(uint8_t* dst, const CUtensorMap* map, const AttnArgs& a,
                                            const Unit& U, int kt, uint64_t* bar, const BtWin& w) {
  int blk[BKV / KB];
#pragma unroll
  for (int b = 0; b < BKV / KB; ++b) blk[b] = __shfl_sync(0xffffffffu, w.cur, (kt % 8) * (BKV / KB) + b);
  if (elect_one()) {
    mbar_arrive_expect_tx(bar, BKV * HD * 2);
#pragma unroll
    for (int b = 0; b < BKV / KB; ++b)
#pragma unroll
      for (int half = 0; half < 2; ++half)
        tma_load_2d(dst + half * 8192 + b * KB * 128, map, bar, half * 64, (blk[b] * a.Hkv + U.g) * KB);
  } else {
    mbar_arrive(bar);
  }
}
}  // namespace

template <int NQ>
__global__ void __launch_bounds__(Cfg<NQ>::NT, Cfg<NQ>::CTAS)
    k_attn_prefill5(const __grid_constant__ CUtensorMap mk, const __grid_constant__ CUtensorMap mv,
                    const __grid_constant__ CUtensorMap mq, AttnArgs a) {
  using C = Cfg<NQ>;
  constexpr int NKB = C::NKB, W_LOAD = C::W_LOAD, W_VLOAD = C::W_VLOAD, W_MMA = C::W_MMA, NLW = C::NLW;
  constexpr int NBW = BKV / KB / NLW;   // blocks of a KV tile per loader warp
  constexpr int OFF_Q = C::OFF_Q, OFF_K = C::OFF_K, OFF_V = C::OFF_V;
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = smem_raw;
  if (smem_u32(sm) & 1023) __trap();   // swizzle atoms need 1024-byte alignment
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + C::OFF_BAR);
  // sfull / pfull / pvdone: [query tile][S/P or V buffer]; oempty: [query tile]
  uint64_t *vfull = bars, *pvdone = bars + 2, *sfull = pvdone + 2 * NQ, *pfull = sfull + 2 * NQ;
  uint64_t *oempty = pfull + 2 * NQ, *qfull = oempty + NQ, *qempty = qfull + 1, *ufull = qfull + 2, *uempty = ufull + 2;
  uint64_t *kfull = uempty + 2, *kempty = kfull + NKB;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(kempty + NKB);
  volatile int* ring = reinterpret_cast<volatile int*>(tslot + 1);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t sbase = smem_u32(sm);
  if (tid == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(vfull + i, 32 * NLW);   // one cp.async-completion arrive per loader lane
      mbar_init(ufull + i, 1);
      mbar_init(uempty + i, 2 * NLW - 1 + NQ + C::NSW);   // loaders but the claimer, MMA warps, softmax warps
    }
    for (int i = 0; i < 2 * NQ; ++i) {
      mbar_init(sfull + i, 1);    // tcgen05.commit
      mbar_init(pfull + i, 4);    // one arrive per softmax warp of the tile
      mbar_init(pvdone + i, 1);
    }
    for (int i = 0; i < NKB; ++i) {
      mbar_init(kfull + i, 32 * NLW);
      mbar_init(kempty + i, NQ);  // each query tile's S
    }
    for (int i = 0; i < NQ; ++i) mbar_init(oempty + i, 4);
    mbar_init(qfull, 32 * NLW);
    mbar_init(qempty, NQ);
    mbar_fence_init();
  }
  if (warp == W_MMA) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)), "r"(C::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_before();
  __syncthreads();
  tc_after();
  const uint32_t tmem = *tslot;
  const __nv_bfloat16* pk = reinterpret_cast<const __nv_bfloat16*>(a.pool_k);
  const __nv_bfloat16* pv = reinterpret_cast<const __nv_bfloat16*>(a.pool_v);
  const int units = (*a.n_tiles) * (a.H / NQ);

  if (warp >= W_LOAD && warp < W_VLOAD) {
    // ---------------- K/Q loaders: warp W_LOAD claims units (the others read
    // them from the ring); each gathers its share of Q (NQ heads) and of K(g)
    // as soon as S(g-NKB) has released K buffer g % NKB
    const int lw = warp - W_LOAD;
    const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
    const int r0 = lane >> 4, c = lane & 15;   // this lane: rows r0 + 2j, 16-byte chunk c
    uint32_t g = 0;
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      int u = 0;
      if (lw == 0) {
        if (lane == 0) u = atomicAdd(a.L.ctr, 1);
        u = __shfl_sync(0xffffffffu, u, 0);
        if (n >= 2) wait(uempty + slot, ((n - 2) >> 1) & 1);
        if (lane == 0) {
          ring[slot] = u < units ? u : -1;
          mbar_arrive(ufull + slot);
        }
        if (u >= units) {   // all units claimed: the next kernel may launch (PDL)
          if (lane == 0) pdl_trigger();
          break;
        }
        if (lane == 0) log_unit(a.L, u);
      } else {
        wait(ufull + slot, (n >> 1) & 1);
        u = ring[slot];
        __syncwarp();
        if (lane == 0) mbar_arrive(uempty + slot);
        if (u < 0) break;
      }
      const Unit U = unit_of<NQ>(a, u);
      const int32_t* bt = a.bt + (size_t)U.r * a.max_blocks;
      const int n_blk = (U.kv_len + KB - 1) / KB;   // blocks this sequence owns
      BtWin w;
      w.start(bt, n_blk, lane);
      for (int kt = 0; kt < U.n_kt; ++kt, ++g) {
        const int kb = g % NKB;
        if (kt > 0 && kt % 8 == 0) w.advance(bt, n_blk, kt, lane);
        if (g >= NKB) wait(kempty + kb, (g / NKB - 1) & 1);
        if (a.kv_tma && (kt + 1) * BKV <= U.kv_len) {
          if (lw == 0) tma_kv_tile(sm + OFF_K + kb * 16384, &mk, a, U, kt, kfull + kb, w);
          else mbar_arrive(kfull + kb);
        } else {
          load_kv_tile<NBW>(sm + OFF_K + kb * 16384, pk, a, U, kt, lane, kfull + kb, w, lw * NBW);
        }
        if (kt == 0 && a.kv_tma) {   // Q tiles by TMA: [T][H][128] boxes {64 dims, 1 head, 128 tokens}
          if (n >= 1) wait(qempty, (n - 1) & 1);         // last S of the previous unit done
          if (lw == 0 && elect_one()) {
            mbar_arrive_expect_tx(qfull, NQ * BQ * HD * 2);
#pragma unroll
            for (int q = 0; q < NQ; ++q)
#pragma unroll
              for (int half = 0; half < 2; ++half)
                tma_load_3d(sm + OFF_Q + q * 32768 + half * 16384, &mq, qfull, half * 64, U.h + q, U.tok0 + U.q0);
          } else {
            mbar_arrive(qfull);
          }
        } else if (kt == 0) {
          if (n >= 1) wait(qempty, (n - 1) & 1);         // last S of the previous unit done
#pragma unroll
          for (int q = 0; q < NQ; ++q) {
#pragma unroll 8
            for (int j = lw * (BQ / 2 / NLW); j < (lw + 1) * (BQ / 2 / NLW); ++j) {
              const int row = r0 + 2 * j;
              const bool ok = U.q0 + row < U.q_len;
              cp_async16_zfill(sm + OFF_Q + q * 32768 + sw(row, c, 16384),
                               qg + (size_t)(U.tok0 + (ok ? U.q0 + row : 0)) * a.H * HD + (U.h + q) * HD + c * 8, ok);
            }
          }
          cp_async_arrive_noinc(qfull);
        }
      }
    }
  } else if (warp >= W_VLOAD && warp < W_MMA) {
    // ---------------- V loaders: their share of V(g) as soon as PV(g-2) has released buffer g & 1
    const int lw = warp - W_VLOAD;
    uint32_t g = 0;
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      wait(ufull + slot, (n >> 1) & 1);
      const int u = ring[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(uempty + slot);
      if (u < 0) break;
      const Unit U = unit_of<NQ>(a, u);
      const int32_t* bt = a.bt + (size_t)U.r * a.max_blocks;
      const int n_blk = (U.kv_len + KB - 1) / KB;   // blocks this sequence owns
      BtWin w;
      w.start(bt, n_blk, lane);
      for (int kt = 0; kt < U.n_kt; ++kt, ++g) {
        const int b = g & 1;
        if (kt > 0 && kt % 8 == 0) w.advance(bt, n_blk, kt, lane);
        if (g >= 2)
#pragma unroll
          for (int q = 0; q < NQ; ++q) wait(pvdone + q * 2 + b, ((g - 2) >> 1) & 1);
        if (a.kv_tma && (kt + 1) * BKV <= U.kv_len) {
          if (lw == 0) tma_kv_tile(sm + OFF_V + b * 16384, &mv, a, U, kt, vfull + b, w);
          else mbar_arrive(vfull + b);
        } else {
          load_kv_tile<NBW>(sm + OFF_V + b * 16384, pv, a, U, kt, lane, vfull + b, w, lw * NBW);
        }
      }
    }
  } else if (warp >= W_MMA) {
    // ---------------- MMA issuer of query tile qm: the whole warp runs the
    // loop (descriptors stay warp-uniform, in uniform registers) and one
    // elected lane issues each tcgen05 op; an issuer in a lane-0 branch made
    // the compiler wrap every MMA in a per-lane waterfall loop
    // f32 accumulate, bf16 A/B; S: N = 64, B K-major; O: N = 128, B MN-major
    const int qm = warp - W_MMA;
    const uint32_t id_s = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BKV >> 3) << 17) | ((uint32_t)(BQ >> 4) << 24);
    const uint32_t id_o = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(HD >> 3) << 17) |
                          ((uint32_t)(BQ >> 4) << 24);
    const uint32_t t_q = tmem + qm * 256, t_o = t_q + 128, qa = sbase + OFF_Q + qm * 32768;
    uint32_t g = 0;
    auto issue_pv = [&](uint32_t gp, bool first, int n) {
      const int b = gp & 1;
      wait(vfull + b, (gp >> 1) & 1);
      if (first && n >= 1) wait(oempty + qm, (n - 1) & 1);   // previous unit's O read out
      wait(pfull + qm * 2 + b, (gp >> 1) & 1);
      tc_after();
      fence_async_smem();
      const uint32_t va = sbase + OFF_V + b * 16384, pa = t_q + b * 64;
      if (elect_one()) {
        // A = P from TMEM: keys 16kk..16kk+15 hi at column 32(kk/2) + 8(kk%2), lo 16 further
#pragma unroll
        for (int kk = 0; kk < BKV / 16; ++kk)
          tc_mma_ts(t_o, pa + (kk >> 1) * 32 + (kk & 1) * 8, desc_mn(va + kk * 2048), id_o, (!first || kk > 0) ? 1u : 0u);
#pragma unroll
        for (int kk = 0; kk < BKV / 16; ++kk)
          tc_mma_ts(t_o, pa + (kk >> 1) * 32 + 16 + (kk & 1) * 8, desc_mn(va + kk * 2048), id_o, 1u);
        tc_commit(pvdone + qm * 2 + b);
      }
      __syncwarp();
    };
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      wait(ufull + slot, (n >> 1) & 1);
      const int u = ring[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(uempty + slot);
      if (u < 0) break;
      const Unit U = unit_of<NQ>(a, u);
      wait(qfull, n & 1);
      for (int kt = 0; kt < U.n_kt; ++kt, ++g) {
        const int b = g & 1, kb = g % NKB;
        wait(kfull + kb, (g / NKB) & 1);
        if (g >= 2) wait(pvdone + qm * 2 + b, ((g - 2) >> 1) & 1);   // P(g-2) consumed: S buffer b free
        tc_after();
        fence_async_smem();
        const uint32_t ka = sbase + OFF_K + kb * 16384;
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < HD / 16; ++kk)
            tc_mma(t_q + b * 64, desc_k(qa + (kk >> 2) * 16384 + (kk & 3) * 32),
                   desc_k(ka + (kk >> 2) * 8192 + (kk & 3) * 32), id_s, kk > 0 ? 1u : 0u);
          tc_commit(sfull + qm * 2 + b);
          tc_commit(kempty + kb);
          if (kt == U.n_kt - 1) tc_commit(qempty);
        }
        __syncwarp();
        if (kt > 0) issue_pv(g - 1, kt == 1, n);
      }
      issue_pv(g - 1, U.n_kt == 1, n);
    }
  } else {
    // ---------------- softmax + epilogue: warp w serves query tile w / 4;
    // thread owns query row (w % 4) * 32 + lane = its TMEM lane
    __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
    const float sl2 = a.scale * 1.4426950408889634f;
    const int qt = warp >> 2, row = tid & 127;
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    const uint32_t t_s = tmem + qt * 256, t_o = t_s + 128;
    uint32_t g = 0;
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      wait(ufull + slot, (n >> 1) & 1);
      const int u = ring[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(uempty + slot);
      if (u < 0) break;
      const Unit U = unit_of<NQ>(a, u);
      const int qpos = U.ctx + U.q0 + row;
      float m_ref = -INFINITY, l_run = 0.f;
      for (int kt = 0; kt < U.n_kt; ++kt, ++g) {
        const int b = g & 1;
        const uint32_t t_sb = t_s + b * 64 + lane_off;
        wait(sfull + qt * 2 + b, (g >> 1) & 1);
        tc_after();
        // two passes over S in TMEM (32 columns at a time) keep ~32 scores live:
        // pass 1 row max, pass 2 P.  Only tiles crossing the causal diagonal or
        // the end of the sequence need the per-element mask (warp-uniform test).
        const bool edge = (kt + 1) * BKV - 1 > U.ctx + U.q0 || (kt + 1) * BKV > U.kv_len;
        const int lim = min(qpos + 1, U.kv_len) - kt * BKV;   // keys [0, lim) of this tile are visible
        float mx = -INFINITY;
#pragma unroll
        for (int half = 0; half < 2; ++half) {
          float v[32];
          tmem_ld32(t_sb + half * 32, v);
          if (edge) {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (half * 32 + i >= lim) v[i] = -INFINITY;
          }
#pragma unroll
          for (int i = 0; i < 32; ++i) mx = fmaxf(mx, v[i]);
        }
        const float mx_s = mx * sl2;                  // scale > 0 commutes with max
        const bool move = mx_s > m_ref + 8.f;         // includes m_ref = -inf (first tile)
        const float m_new = move ? mx_s : m_ref;
        const float alpha = move ? ex2(m_ref - m_new) : 1.f;
        if (kt > 0 && __any_sync(0xffffffffu, move)) {   // lazy rescale of O: PV(g-1) must be done
          wait(pvdone + qt * 2 + ((g - 1) & 1), ((g - 1) >> 1) & 1);
          tc_after();
#pragma unroll 1
          for (int c = 0; c < 4; ++c) {
            float w[32];
            tmem_ld32(t_o + lane_off + c * 32, w);
#pragma unroll
            for (int i = 0; i < 32; ++i) w[i] *= alpha;
            tmem_st32(t_o + lane_off + c * 32, w);
          }
        }
        // P = 2^(s*scale*log2e - m) as bf16 hi + lo, written over S(g): keys
        // 32h..32h+31 go to columns [32h, 32h+16) (hi) and [32h+16, 32h+32) (lo),
        // exactly the columns their scores came from, so half 1's scores are
        // still intact when half 0's P is stored.
        float2 acc = make_float2(0.f, 0.f);
#pragma unroll
        for (int half = 0; half < 2; ++half) {
          float v[32];
          tmem_ld32(t_sb + half * 32, v);
          if (edge) {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (half * 32 + i >= lim) v[i] = -INFINITY;
          }
          uint32_t hi[16], lo[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            const float2 t = ffma2(make_float2(v[2 * j], v[2 * j + 1]), sl2, -m_new);
            const float2 pp = make_float2(ex2(t.x), ex2(t.y));
            acc = fadd2(acc, pp);
            // P = hi + lo with both parts truncated to bf16 by byte permutes
            // (ALU) instead of two cvt.rn.bf16x2 (conversion pipe, shared with
            // nothing the MMA needs but slow): x - trunc(x) is exact, so the
            // only error is lo's truncation, < 2^-15 |P| (R-4b asks for better
            // than bf16's 2^-9)
            const uint32_t ux = __float_as_uint(pp.x), uy = __float_as_uint(pp.y);
            const float2 l = fsub2(pp, make_float2(__uint_as_float(ux & 0xFFFF0000u), __uint_as_float(uy & 0xFFFF0000u)));
            hi[j] = __byte_perm(ux, uy, 0x7632);
            lo[j] = __byte_perm(__float_as_uint(l.x), __float_as_uint(l.y), 0x7632);
          }
          tmem_st16(t_sb + half * 32, hi);
          tmem_st16(t_sb + half * 32 + 16, lo);
        }
        l_run = l_run * alpha + (acc.x + acc.y);
        m_ref = m_new;
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(pfull + qt * 2 + b);
      }
      // ---- normalise and store row `row` of head U.h + qt (bf16, point R3) once the last PV is done
      wait(pvdone + qt * 2 + ((g - 1) & 1), ((g - 1) >> 1) & 1);
      tc_after();
      const float inv = 1.f / l_run;
      const bool ok = U.q0 + row < U.q_len;
      __nv_bfloat16* dst = og + (size_t)(U.tok0 + U.q0 + (ok ? row : 0)) * a.H * HD + (U.h + qt) * HD;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        float w[32];
        tmem_ld32(t_o + lane_off + c * 32, w);
        if (ok) {
#pragma unroll
          for (int q = 0; q < 4; ++q)
            *reinterpret_cast<uint4*>(dst + c * 32 + q * 8) =
                make_uint4(pack_bf2(w[8 * q] * inv, w[8 * q + 1] * inv), pack_bf2(w[8 * q + 2] * inv, w[8 * q + 3] * inv),
                           pack_bf2(w[8 * q + 4] * inv, w[8 * q + 5] * inv), pack_bf2(w[8 * q + 6] * inv, w[8 * q + 7] * inv));
        }
      }
      tc_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(oempty + qt);
    }
  }
  tc_before();
  __syncthreads();
  if (warp == W_MMA) {
    tc_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C::TMEM_COLS));
  }
}

// Query tiles per CTA: 2 when the GQA group size is even (the two heads
// share their K / V tiles), else 1; BULLET_PF5_NQ=1 forces the single-tile
// kernel (A/B).
int attn_prefill5_nq(int H, int Hkv) {
  static const int forced = getenv("BULLET_PF5_NQ") ? atoi(getenv("BULLET_PF5_NQ")) : 0;
  if (forced == 1) return 1;
  return (H / Hkv) % 2 == 0 ? 2 : 1;
}
int attn_prefill5_ctas_per_sm(int H, int Hkv) { return attn_prefill5_nq(H, Hkv) == 2 ? 1 : 2; }

template <int NQ>
static cudaError_t launch_nq(const CUtensorMap& mk, const CUtensorMap& mv, const CUtensorMap& mq, const AttnArgs& a,
                             int grid, cudaStream_t st) {
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_prefill5<NQ>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<NQ>::SMEM_BYTES);
    if (e != cudaSuccess) return e;
    set = true;
  }
  return launch_ex(k_attn_prefill5<NQ>, grid, Cfg<NQ>::NT, Cfg<NQ>::SMEM_BYTES, st, a.L.pdl, mk, mv, mq, a);
}

// `grid` must be n_sms * attn_prefill5_ctas_per_sm(H, Hkv) (persistent, gated).
// mk / mv: the layer's K / V pool as [blocks * Hkv * 16][128] bf16 tensors,
// box {64, 16}; mq: q as [T][H][128], box {64, 1, 128}; 128-byte swizzle
// (used when a.kv_tma != 0).
cudaError_t launch_attn_prefill5(const CUtensorMap& mk, const CUtensorMap& mv, const CUtensorMap& mq,
                                 const AttnArgs& a, int grid, cudaStream_t st) {
  return attn_prefill5_nq(a.H, a.Hkv) == 2 ? launch_nq<2>(mk, mv, mq, a, grid, st)
                                           : launch_nq<1>(mk, mv, mq, a, grid, st);
}

cudaError_t preload_attn_prefill5() {
  cudaFuncAttributes f;
  cudaError_t e = cudaFuncGetAttributes(&f, k_attn_prefill5<1>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_attn_prefill5<2>);
  return e;
}

}  // namespace bl
