// attn_decode.cu — paged decode attention on tensor cores, bf16, hd 128
// (the paper's PagedAttention decode: "irregular
// memory access" — here every (block, kv head) is one contiguous 4 KB chunk).
//
// Memory side: each of the 12 consumer warps streams its own blocks, DEPTH
// blocks in flight per warp: by TMA (default, a.kv_tma: the pool viewed as a
// [blocks * Hkv * 16][128] tensor, K and V of a block as two 16-row x 64-dim
// boxes each with the 128-byte swizzle, issued by one elected lane, completion
// in bytes on the stage's mbarrier) or with 16-byte cp.async (coalesced 4 KB
// chunks, XOR-swizzled; BULLET_DEC_TMA=0).  Round 2 measured the TMA stream
// 1.5-2.5 % faster on 64-70 SMs and bit-identical (round 1's TMA attempt,
// capped near 27 GB/s per SM, issued from a single thread).  A claimer warp takes units from the
// gated work counter and publishes each unit's block-table row and Q rows in
// shared memory up to 4 units ahead, so no consumer waits on a dependent
// global load; warps prefetch the next unit's first blocks before merging the
// current one.
// Math side: swap-AB so the 16 keys of a block fill the MMA M dimension and
// the GQA group (<= 8 query heads) fills N = 8:
//   S^T[16 keys x 8 heads] = K[16 x 128] . Q^T[128 x 8]   (mma.m16n8k16 bf16)
//   O^T[128 x 8]         += V^T[128 x 16] . P^T[16 x 8]  (P = hi + lo bf16)
// P^T fragments come from the S^T accumulators by movmatrix (8x8 transpose).
// Warps take blocks round-robin with private (max, sum, O^T) states, merged
// through shared memory at the end of each unit.
// Unit = (token, kv head); decode tokens are requests.
#include <stdlib.h>

#include "kernels.h"

namespace bl {

namespace {
// DEPTH stages per warp: DEPTH - 1 blocks stay in flight while one is computed
// 12 consumer warps x 2 stages (8 x 3 before): the kernel is bound by the
// per-warp latency of its block math, so more warps beat deeper per-warp
// pipelines — 68 SMs, 1k / 4k contexts: 62 -> 72-79 / 71 -> 84-86 GB/s/SM;
// 148 SMs: 6.8 TB/s (the HBM roofline); 6 x 4 and 4 x 5 were slower
// (scripts/attn_dec_bench.py)
#ifndef DEC_NCW
#define DEC_NCW 12
#define DEC_DEPTH 2
#endif
constexpr int KB = 16, HD = 128, NCW = DEC_NCW, DEPTH = DEC_DEPTH;
static_assert(DEPTH <= 5, "cp.async wait ladder covers DEPTH <= 5");
constexpr int BLK_BYTES = KB * HD * 2;       // 4 KB: one (block, kv head) of K or V
constexpr int STAGE_BYTES = 2 * BLK_BYTES;   // K + V
constexpr int CMB_FLOATS = HD * 8 + 16;      // O^T[128][8] + m[8] + l[8] per warp (in a free stage)
constexpr int THREADS = (NCW + 1) * 32;
constexpr int QSLOT_BYTES = 8 * HD * 2;      // Q rows of up to 8 heads (bf16)
constexpr int MAXNB = 512;                   // blocks per unit held in smem (8k tokens)
constexpr int NS_MAX = 8;                    // unit slots (2 per consumer group, up to 4 groups)
static_assert(CMB_FLOATS * 4 <= STAGE_BYTES, "merge record must fit in one stage");

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t* r) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t* r) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
__device__ __forceinline__ void mma_bf16(float* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t movtrans(uint32_t x) {
  uint32_t y;
  asm volatile("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;" : "=r"(y) : "r"(x));
  return y;
}
__device__ __forceinline__ uint32_t pack_bf2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}
// x -> hi = bf16(x), lo = bf16(x - hi), packed pairwise.
__device__ __forceinline__ void split_bf2(float a, float b, uint32_t& hi, uint32_t& lo) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  const float2 f = __bfloat1622float2(h);
  hi = *reinterpret_cast<uint32_t*>(&h);
  lo = pack_bf2(a - f.x, b - f.y);
}
// byte offset of 16-byte chunk c (0..15) of key row `row` in a [16][128] bf16
// tile: rows of 256 B, chunk index XOR (row & 7) -> conflict-free ldmatrix
__device__ __forceinline__ uint32_t tile_off(int row, int c) {
  return row * 256 + ((c ^ (row & 7)) << 4);
}

// byte offset of 16-byte chunk c (0..15) of key row `row` in the layout the
// TMA boxes produce: [2 halves of 64 dims][16 rows][128 B], 128-byte swizzle
__device__ __forceinline__ uint32_t tile_off_sw128(int row, int c) {
  return (c >> 3) * 2048 + row * 128 + (((c & 7) ^ (row & 7)) << 4);
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tma_load_2d_hint(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                                 uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}

// KV is streamed once per launch: evict-first keeps it from displacing the
// other phase's L2-resident activation tiles.
__device__ __forceinline__ void cp_async16_ef(void* dst, const void* src, uint64_t pol) {
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "l"(pol)
               : "memory");
}

struct Slot {  // one published unit: blocks [b0, b0 + nb) of (token t, kv head u % Hkv)
  int u, t, pos, nb, b0, c;   // c: KV chunk of a split unit (kv_chunks > 1), else 0
};
}  // namespace

// NG consumer groups of NCW / NG warps: group gw takes the units it = gw,
// gw + NG, ... (units alternate between groups), so a unit's blocks are
// split over fewer warps and the per-unit merge is paid over more blocks.
template <int NG>
__global__ void __launch_bounds__(THREADS, 1)
    k_attn_decode_tc(const __grid_constant__ CUtensorMap mk, const __grid_constant__ CUtensorMap mv, AttnArgs a) {
  constexpr int GW = NCW / NG;
  constexpr int NS = 2 * NG;   // unit slots: each group holds <= 2 units (current + next)
  if (!gate_enter(a.L)) return;
  if (threadIdx.x == 0 && a.L.trace) { trace_at(a.L, 0, smid()); trace_at(a.L, 1, gtimer()); }
  pdl_wait();      // q and the new token's k / v come from the QKV GEMM
  extern __shared__ __align__(128) uint8_t smem[];
  uint8_t* stages = smem;                                                      // [NCW][DEPTH][STAGE]
  uint8_t* qbuf = stages + NCW * DEPTH * STAGE_BYTES;                          // [NS_MAX][QSLOT_BYTES]
  int* btbuf = reinterpret_cast<int*>(qbuf + NS_MAX * QSLOT_BYTES);            // [NS_MAX][MAXNB]
  Slot* uq = reinterpret_cast<Slot*>(btbuf + NS_MAX * MAXNB);
  uint64_t* uqf = reinterpret_cast<uint64_t*>(uq + NS_MAX);
  uint64_t* uqe = uqf + NS_MAX;
  int* rec_stage = reinterpret_cast<int*>(uqe + NS_MAX);                       // [NCW] (+ NG merge flags)
  uint64_t* sfull = reinterpret_cast<uint64_t*>(rec_stage + NCW + 4);          // [NCW][DEPTH] (a.kv_tma)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int grp = a.H / a.Hkv;
  const int units = (a.n_tok - a.tok_base) * a.Hkv;   // decode rows are tokens [tok_base, n_tok)
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) { mbar_init(uqf + i, 1); mbar_init(uqe + i, GW); }
    for (int i = 0; i < NCW * DEPTH; ++i) mbar_init(sfull + i, 1);
    mbar_fence_init();
  }
  __syncthreads();

  if (warp == NCW) {  // ------------------------------------------ claimer
    const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
    int n_end = 0;
    for (int it = 0;; ++it) {
      const int slot = it % NS;
      // a group holds at most 2 units (current + next, so its warps can
      // prefetch across the boundary): unit it waits for unit it - 2 NG of
      // the same group (load balance across CTAs; 4 slots = 2 NG)
      if (lane == 0 && it >= NS) mbar_wait(uqe + ((it - NS) % NS), ((it - NS) / NS) & 1);
      __syncwarp();
      // sub-unit v = c * units + u: KV chunk c (MAXNB blocks) of unit u;
      // chunks past a row's length are empty and skipped
      Slot sl{-1, 0, 0, 0, 0, 0};
      int32_t const* bt = nullptr;
      for (;;) {
        int v = 0;
        if (lane == 0) v = n_end ? units * a.kv_chunks : atomicAdd(a.L.ctr, 1);
        v = __shfl_sync(0xffffffffu, v, 0);
        if (v >= units * a.kv_chunks) break;
        const int u = v % units, c = v / units;
        int r;
        if (a.order) {   // (row, request, position) from the plan kernel: one load
          const int4 od = __ldg(a.order + u / a.Hkv);
          sl.t = a.tok_base + od.x; r = od.y; sl.pos = od.z;
        } else {
          sl.t = a.tok_base + u / a.Hkv;
          r = find_req(a.cu, a.n_reqs, sl.t);
          sl.pos = __ldg(a.ctx + r) + (sl.t - __ldg(a.cu + r));
        }
        const int nb_all = sl.pos / KB + 1;
        if (c * MAXNB >= nb_all) continue;   // empty chunk of a short row
        sl.u = u; sl.c = c; sl.b0 = c * MAXNB; sl.nb = min(MAXNB, nb_all - sl.b0);
        bt = a.bt + (size_t)r * a.max_blocks + sl.b0;
        break;
      }
      const int u = sl.u;
      if (u >= 0)
        for (int b = lane; b < sl.nb; b += 32) btbuf[slot * MAXNB + b] = __ldg(bt + b);
      __syncwarp();
      if (lane == 0) {
        uq[slot] = sl;
        if (u >= 0) {  // Q rows of the unit ride on the slot's barrier
          const int g = u % a.Hkv;
          mbar_arrive_expect_tx(uqf + slot, grp * HD * 2);
          bulk_g2s(qbuf + slot * QSLOT_BYTES, qg + (size_t)sl.t * a.H * HD + (size_t)g * grp * HD,
                   grp * HD * 2, uqf + slot);
          log_unit(a.L, u);
        } else {
          mbar_arrive(uqf + slot);
        }
      }
      if (u < 0 && lane == 0 && n_end == 0) pdl_trigger();   // all units claimed: let the next kernel launch
      if (u < 0 && ++n_end == NG) break;   // one terminator per group
    }
    return;
  }

  // ------------------------------------------------------------ consumers
  const int gq = lane >> 2, tq = lane & 3;
  const float sl2 = a.scale * 1.4426950408889634f;
  const __nv_bfloat16* pk = reinterpret_cast<const __nv_bfloat16*>(a.pool_k);
  const __nv_bfloat16* pv = reinterpret_cast<const __nv_bfloat16*>(a.pool_v);
  __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
  uint8_t* my = stages + warp * DEPTH * STAGE_BYTES;
  uint64_t pol_kv;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_kv));
  const uint32_t my_s = smem_u32(my);
  const int gw = warp / GW, wl = warp % GW;   // group, index in the group
  auto my_count = [&](int nb) { return nb > wl ? (nb - wl + GW - 1) / GW : 0; };
  // per-lane swizzled offsets (loop invariant): cp.async destinations and
  // ldmatrix sources for the QK (K, by k-step) and PV (V^T, by m-tile) MMAs
  // (a.kv_tma: the TMA boxes land K / V as [2 halves of 64 dims][16 rows][128 B]
  // with the 128-byte swizzle — also conflict-free for ldmatrix)
  const bool tma = a.kv_tma != 0;
  auto off = [&](int row, int c) { return tma ? tile_off_sw128(row, c) : tile_off(row, c); };
  uint32_t cp_off[8], k_off[8], v_off[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    cp_off[i] = tile_off(2 * i + (lane >> 4), lane & 15);
    k_off[i] = off(lane & 15, i * 2 + (lane >> 4));
    v_off[i] = BLK_BYTES + off(((lane >> 3) >> 1) * 8 + (lane & 7), i * 2 + ((lane >> 3) & 1));
  }
  uint64_t* my_full = sfull + warp * DEPTH;

  const int pf = a.dec_pf;   // L2 prefetch distance in this warp's blocks (0 = off)
  // issue cursor over this warp's block sequence (units in claim order,
  // my blocks warp, warp + 8, ... of each), never beyond unit `limit`
  int iu = gw, ij = 0, n_issued = 0, n_cons = 0;
  int cur_nb = -1, cur_g = 0, cur_u = 0;   // cached slot of unit iu (-1: not read yet)
  auto fill = [&](int limit, int cap) {
    while (n_issued - n_cons < cap && iu <= limit) {
      const int sl = iu % NS;
      if (cur_nb < 0) {
        mbar_wait(uqf + sl, (iu / NS) & 1);
        const Slot X = uq[sl];
        cur_u = X.u; cur_nb = my_count(X.nb); cur_g = X.u >= 0 ? X.u % a.Hkv : 0;
      }
      if (cur_u < 0) return;
      if (ij >= cur_nb) { iu += NG; ij = 0; cur_nb = -1; continue; }
      const int blk = btbuf[sl * MAXNB + wl + ij * GW];
      const uint8_t* ks = reinterpret_cast<const uint8_t*>(pk + ((size_t)blk * a.Hkv + cur_g) * KB * HD) + lane * 16;
      const uint8_t* vs = reinterpret_cast<const uint8_t*>(pv + ((size_t)blk * a.Hkv + cur_g) * KB * HD) + lane * 16;
      if (pf > 0 && lane == 0 && ij + pf < cur_nb) {
        // L2 prefetch pf blocks ahead of this warp's stream: the cp.async that
        // follows hits L2, so the smem ring (the bytes a warp can keep in
        // flight) covers the L2 latency instead of the DRAM latency
        const int b2 = btbuf[sl * MAXNB + wl + (ij + pf) * GW];
        prefetch_l2(pk + ((size_t)b2 * a.Hkv + cur_g) * KB * HD, BLK_BYTES);
        prefetch_l2(pv + ((size_t)b2 * a.Hkv + cur_g) * KB * HD, BLK_BYTES);
      }
      uint8_t* dk = my + (n_issued % DEPTH) * STAGE_BYTES;
      if (tma) {   // one elected lane: K and V as 2 boxes each (16 rows x 64 dims), bytes counted on the stage barrier
        const int row = (blk * a.Hkv + cur_g) * KB;
        if (elect_one()) {
          uint64_t* bar = my_full + (n_issued % DEPTH);
          fence_proxy_async();   // this warp's generic reads / merge-record writes of the stage come first
          mbar_arrive_expect_tx(bar, STAGE_BYTES);
          tma_load_2d_hint(dk, &mk, bar, 0, row, pol_kv);
          tma_load_2d_hint(dk + BLK_BYTES / 2, &mk, bar, 64, row, pol_kv);
          tma_load_2d_hint(dk + BLK_BYTES, &mv, bar, 0, row, pol_kv);
          tma_load_2d_hint(dk + BLK_BYTES + BLK_BYTES / 2, &mv, bar, 64, row, pol_kv);
        }
        __syncwarp();
      } else {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        cp_async16_ef(dk + cp_off[i], ks + 512 * i, pol_kv);
        cp_async16_ef(dk + BLK_BYTES + cp_off[i], vs + 512 * i, pol_kv);
      }
      cp_async_commit();
      }
      ++n_issued;
      ++ij;
    }
  };

  for (int it = gw;; it += NG) {
    const int slot = it % NS;
    mbar_wait(uqf + slot, (it / NS) & 1);
    const Slot S = uq[slot];
    if (S.u < 0) break;
    const int g = S.u % a.Hkv;
    // Q^T as the B operand: n = head gq (zero beyond the group), k = dims
    uint32_t qb[8][2];
    {
      const bool ok = gq < grp;
      const uint8_t* qh = qbuf + slot * QSLOT_BYTES + (ok ? gq : 0) * HD * 2;
#pragma unroll
      for (int ks = 0; ks < 8; ++ks) {
        qb[ks][0] = ok ? *reinterpret_cast<const uint32_t*>(qh + (ks * 16 + 2 * tq) * 2) : 0u;
        qb[ks][1] = ok ? *reinterpret_cast<const uint32_t*>(qh + (ks * 16 + 8 + 2 * tq) * 2) : 0u;
      }
    }
    float m0 = -INFINITY, m1 = -INFINITY, l0 = 0.f, l1 = 0.f;   // heads 2tq, 2tq+1
    float oacc[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) oacc[i][0] = oacc[i][1] = oacc[i][2] = oacc[i][3] = 0.f;

    const int mine = my_count(S.nb);
    for (int j = 0; j < mine; ++j) {
      fill(it + NG, DEPTH);
      if (tma) {
        mbar_wait(my_full + (n_cons % DEPTH), (n_cons / DEPTH) & 1);
      } else {
      const int pend = n_issued - n_cons;   // groups in flight; the oldest is block j
      if (pend >= 5) cp_async_wait<4>(); else if (pend == 4) cp_async_wait<3>();
      else if (pend == 3) cp_async_wait<2>(); else if (pend == 2) cp_async_wait<1>(); else cp_async_wait<0>();
      }
      __syncwarp();
      const int b = wl + j * GW;
      const uint32_t kt = my_s + (n_cons % DEPTH) * STAGE_BYTES;
      if (a.dbg & 1) {   // diagnostics (BULLET_DBG): stream only, no math
        __syncwarp();
        ++n_cons;
        continue;
      }
      float s[4] = {0.f, 0.f, 0.f, 0.f}, s2[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int ks = 0; ks < 8; ks += 2) {   // two independent accumulation chains
        uint32_t af[4], ag[4];
        ldsm_x4(kt + k_off[ks], af);
        ldsm_x4(kt + k_off[ks + 1], ag);
        mma_bf16(s, af, qb[ks][0], qb[ks][1]);
        mma_bf16(s2, ag, qb[ks + 1][0], qb[ks + 1][1]);
      }
      s[0] += s2[0]; s[1] += s2[1]; s[2] += s2[2]; s[3] += s2[3];
      // s[0] (key gq, head 2tq), s[1] (gq, 2tq+1), s[2] (gq+8, 2tq), s[3] (gq+8, 2tq+1)
      const int k0 = (S.b0 + b) * KB + gq, k1 = k0 + 8;
      s[0] = k0 <= S.pos ? s[0] * sl2 : -INFINITY;
      s[1] = k0 <= S.pos ? s[1] * sl2 : -INFINITY;
      s[2] = k1 <= S.pos ? s[2] * sl2 : -INFINITY;
      s[3] = k1 <= S.pos ? s[3] * sl2 : -INFINITY;
      float bm0 = fmaxf(s[0], s[2]), bm1 = fmaxf(s[1], s[3]);
#pragma unroll
      for (int o = 4; o < 32; o <<= 1) {
        bm0 = fmaxf(bm0, __shfl_xor_sync(0xffffffffu, bm0, o));
        bm1 = fmaxf(bm1, __shfl_xor_sync(0xffffffffu, bm1, o));
      }
      const float mn0 = fmaxf(m0, bm0), mn1 = fmaxf(m1, bm1);
      const float al0 = exp2f(m0 - mn0), al1 = exp2f(m1 - mn1);
      m0 = mn0; m1 = mn1;
      const float p00 = exp2f(s[0] - mn0), p01 = exp2f(s[1] - mn1);
      const float p10 = exp2f(s[2] - mn0), p11 = exp2f(s[3] - mn1);
      l0 = l0 * al0 + p00 + p10;
      l1 = l1 * al1 + p01 + p11;
      if (__any_sync(0xffffffffu, al0 != 1.f || al1 != 1.f)) {   // max moved: rescale O
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          oacc[i][0] *= al0; oacc[i][1] *= al1; oacc[i][2] *= al0; oacc[i][3] *= al1;
        }
      }
      uint32_t h0, h1, lo0, lo1;
      split_bf2(p00, p01, h0, lo0);
      split_bf2(p10, p11, h1, lo1);
      const uint32_t bh0 = movtrans(h0), bh1 = movtrans(h1);
      const uint32_t bl0 = movtrans(lo0), bl1 = movtrans(lo1);
      uint32_t vf[8][4];
#pragma unroll
      for (int mt = 0; mt < 8; ++mt) ldsm_x4_t(kt + v_off[mt], vf[mt]);
#pragma unroll
      for (int mt = 0; mt < 8; ++mt) mma_bf16(oacc[mt], vf[mt], bh0, bh1);
#pragma unroll
      for (int mt = 0; mt < 8; ++mt) mma_bf16(oacc[mt], vf[mt], bl0, bl1);
      __syncwarp();
      ++n_cons;
    }
    // the next unit's first DEPTH-1 blocks fly during the merge; the stage
    // left free holds this warp's merge record
    fill(it + NG, DEPTH - 1);
    if (a.dbg & 2) {   // diagnostics (BULLET_DBG): skip the merge and the output
      __syncwarp();
      if (lane == 0) mbar_arrive(uqe + slot);
      continue;
    }
    // full row sums over the 8 key lanes of each head
#pragma unroll
    for (int o = 4; o < 32; o <<= 1) {
      l0 += __shfl_xor_sync(0xffffffffu, l0, o);
      l1 += __shfl_xor_sync(0xffffffffu, l1, o);
    }
    const int fs = n_issued % DEPTH;
    if (lane == 0) rec_stage[warp] = warp * DEPTH + fs;
    float* rec = reinterpret_cast<float*>(my + fs * STAGE_BYTES);   // O^T[dim][head], m[8], l[8]
#pragma unroll
    for (int mt = 0; mt < 8; ++mt) {
      rec[(mt * 16 + gq) * 8 + 2 * tq] = oacc[mt][0];
      rec[(mt * 16 + gq) * 8 + 2 * tq + 1] = oacc[mt][1];
      rec[(mt * 16 + gq + 8) * 8 + 2 * tq] = oacc[mt][2];
      rec[(mt * 16 + gq + 8) * 8 + 2 * tq + 1] = oacc[mt][3];
    }
    if (gq == 0) {
      rec[HD * 8 + 2 * tq] = m0; rec[HD * 8 + 2 * tq + 1] = m1;
      rec[HD * 8 + 8 + 2 * tq] = l0; rec[HD * 8 + 8 + 2 * tq + 1] = l1;
    }
    named_bar_sync(1 + gw, GW * 32);
    const float* recs[GW];
#pragma unroll
    for (int w = 0; w < GW; ++w) recs[w] = reinterpret_cast<const float*>(stages + rec_stage[gw * GW + w] * STAGE_BYTES);
    const int n_ch = a.kv_chunks > 1 ? (S.pos / KB + 1 + MAXNB - 1) / MAXNB : 1;   // chunks of this unit
    // split unit: [unit][chunk] records of grp x (O[128], m, l) in the scratch
    float* part = n_ch > 1 ? a.kv_part + ((size_t)S.u * a.kv_chunks + S.c) * 8 * (HD + 2) : nullptr;
    for (int e = threadIdx.x - gw * GW * 32; e < grp * HD; e += GW * 32) {
      const int h = e / HD, d = e % HD;
      float M = -INFINITY;
      for (int w = 0; w < GW; ++w) M = fmaxf(M, recs[w][HD * 8 + h]);
      float L = 0.f, O = 0.f;
      for (int w = 0; w < GW; ++w) {
        const float* rw = recs[w];
        const float mw = rw[HD * 8 + h];
        if (mw == -INFINITY) continue;
        const float f = exp2f(mw - M);
        L += rw[HD * 8 + 8 + h] * f;
        O += rw[d * 8 + h] * f;
      }
      if (part) {
        part[h * (HD + 2) + d] = O;
        if (d == 0) { part[h * (HD + 2) + HD] = M; part[h * (HD + 2) + HD + 1] = L; }
      } else {
        og[(size_t)S.t * a.H * HD + (size_t)(g * grp + h) * HD + d] = __float2bfloat16_rn(O / L);
      }
    }
    if (part) {   // the unit's last chunk to finish merges all chunks in chunk order (deterministic)
      __threadfence();
      named_bar_sync(1 + gw, GW * 32);
      int* s_flag = rec_stage + NCW + gw;
      if (threadIdx.x == gw * GW * 32) {
        const int old = atomicAdd(a.kv_tick + S.u, 1);
        *s_flag = old == n_ch - 1;
        if (old == n_ch - 1) a.kv_tick[S.u] = 0;   // self-reset for the next launch
      }
      named_bar_sync(1 + gw, GW * 32);
      if (*s_flag) {
        __threadfence();
        const float* P0 = a.kv_part + (size_t)S.u * a.kv_chunks * 8 * (HD + 2);
        for (int e = threadIdx.x - gw * GW * 32; e < grp * HD; e += GW * 32) {
          const int h = e / HD, d = e % HD;
          float M = -INFINITY;
          for (int c = 0; c < n_ch; ++c) M = fmaxf(M, __ldcg(P0 + ((size_t)c * 8 + h) * (HD + 2) + HD));
          float L = 0.f, O = 0.f;
          for (int c = 0; c < n_ch; ++c) {
            const float* pc = P0 + ((size_t)c * 8 + h) * (HD + 2);
            const float mc = __ldcg(pc + HD);
            if (mc == -INFINITY) continue;
            const float f = exp2f(mc - M);
            L += __ldcg(pc + HD + 1) * f;
            O += __ldcg(pc + d) * f;
          }
          og[(size_t)S.t * a.H * HD + (size_t)(g * grp + h) * HD + d] = __float2bfloat16_rn(O / L);
        }
      }
    }
    named_bar_sync(1 + gw, GW * 32);
    if (lane == 0) mbar_arrive(uqe + slot);
  }
  cp_async_wait<0>();
  if (threadIdx.x == 0 && a.L.trace) trace_at(a.L, 5, gtimer());
}

size_t attn_decode_smem_bytes() {
  return (size_t)NCW * DEPTH * STAGE_BYTES + NS_MAX * QSLOT_BYTES + NS_MAX * MAXNB * 4 + NS_MAX * sizeof(Slot) +
         2 * NS_MAX * 8 + (NCW + 4) * 4 + NCW * DEPTH * 8;
}
int attn_decode_max_blocks() { return MAXNB; }

// `ng` consumer groups per CTA (1, 2 or 4; BULLET_DEC_GROUPS overrides).
cudaError_t launch_attn_decode_tc(const CUtensorMap& mk, const CUtensorMap& mv, const AttnArgs& a, int grid, int ng,
                                  cudaStream_t st) {
  const size_t smem = attn_decode_smem_bytes();
  static const int forced = getenv("BULLET_DEC_GROUPS") ? atoi(getenv("BULLET_DEC_GROUPS")) : 0;
  if (forced >= 1 && forced <= 4) ng = forced;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_decode_tc<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(k_attn_decode_tc<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(k_attn_decode_tc<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(k_attn_decode_tc<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    set = true;
  }
  if (ng == 1) return launch_ex(k_attn_decode_tc<1>, grid, THREADS, smem, st, a.L.pdl, mk, mv, a);
  if (ng == 4 && NCW % 4 == 0) return launch_ex(k_attn_decode_tc<4>, grid, THREADS, smem, st, a.L.pdl, mk, mv, a);
  if (ng == 3 && NCW % 3 == 0) return launch_ex(k_attn_decode_tc<3>, grid, THREADS, smem, st, a.L.pdl, mk, mv, a);
  return launch_ex(k_attn_decode_tc<2>, grid, THREADS, smem, st, a.L.pdl, mk, mv, a);
}

cudaError_t preload_attn_decode() {
  cudaFuncAttributes f;
  cudaError_t e = cudaFuncGetAttributes(&f, k_attn_decode_tc<1>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_attn_decode_tc<2>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_attn_decode_tc<4>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_attn_decode_tc<3>);
  return e;
}

}  // namespace bl
