// attn_decode5.cu — paged decode attention on 5th-gen tensor cores (tcgen05
// + TMEM), bf16, head_dim 128, GQA group <= 8 (the paper's
// PagedAttention decode).
//
// Work unit = (decode token, kv head g): its query heads g*grp .. g*grp+grp-1
// against ctx + 1 keys read through the block table.  Per 128-key tile t
// (8 blocks of 16 keys):
//   S^T(t)[128 keys x 16] = K(t)[128 x 128] . Q^T[128 x 16]      tcgen05.mma M=128 N=16
//   softmax over the keys (thread = key = TMEM lane, 4 warps; tile max per
//   head through warp shuffles and shared memory), P^T = hi | lo bf16 halves
//   (R-4b) written to shared memory as the B operand: rows 0..7 = hi of the
//   heads, rows 8..15 = lo
//   O^T[128 dims x 16] += V(t)^T . P^T(t)                         tcgen05.mma M=128 N=16,
//                        A = V used as an MN-major operand straight from its [key][dim] tile
// so O = O^T[:, h] + O^T[:, 8 + h] (hi and lo products in separate columns,
// summed once at the end).  The lane-level MMA chains of the mma.sync kernel
// (attn_decode.cu: ~380 instructions per 16-key block, issue-latency bound)
// become 16 tcgen05 ops per 128 keys issued by one thread.
// Warps: 0 = unit claimer + TMA producer (K and V of a tile = 8 blocks x 2
// halves x 2 boxes of 16 rows x 64 dims, 128-byte swizzle, 64 KB on the
// stage's mbarrier; blocks past the sequence are out-of-bounds boxes, i.e.
// zeros), 1 = MMA issuer (allocates TMEM), 2..5 = softmax + epilogue
// (TMEM lane quadrant = warp % 4).  Stage ring of 3 x 64 KB; S double-
// buffered in TMEM; P double-buffered in shared memory; O^T in TMEM, rescaled
// lazily (only when a head's running max grows by more than 2^8).
#include <stdlib.h>

#include "kernels.h"

namespace bl {

namespace {
constexpr int HD = 128, KB = 16, TK = 128;          // head dim, block size, keys per tile
constexpr int NSTG = 3;                             // K+V stages
constexpr int KT_BYTES = TK * HD * 2;               // 32 KB: K (or V) of a tile
constexpr int ST_BYTES = 2 * KT_BYTES;              // K + V
constexpr int QB_BYTES = 16 * HD * 2;               // Q^T operand: 16 rows (heads) x 128 dims
constexpr int PB_BYTES = 16 * TK * 2;               // P^T operand: 16 rows x 128 keys
constexpr int OFF_Q = NSTG * ST_BYTES, OFF_P = OFF_Q + 2 * QB_BYTES, OFF_RED = OFF_P + 2 * PB_BYTES;
constexpr int OFF_BAR = OFF_RED + 3 * 4 * 8 * 4;    // [3][4 warps][8 heads] floats: tile max x2, l
constexpr int SMEM_BYTES = OFF_BAR + 512;
constexpr int NT = 6 * 32;
constexpr int W_PROD = 0, W_MMA = 1, W_SM0 = 2;     // softmax warps 2..5
constexpr int GMAX = 8;                             // heads per group (N = 16: hi + lo)
constexpr uint32_t TMEM_COLS = 64;                  // S x2 (16 each) + O (16)

__device__ __forceinline__ uint64_t desc_k(uint32_t addr) {   // K-major SW128, SBO 1 KB
  return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)64 << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr) {  // MN-major SW128: LBO 16 KB (dim halves), SBO 1 KB
  return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)(16384 >> 4) << 16) | ((uint64_t)64 << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void tc_mma(uint32_t d, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float* v) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const float* v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          taddr),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
      "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
      : "memory");
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void tma_kv(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}
// SW128 K-major operand of 16 rows: byte offset of 16-byte chunk c (0..15) of row r
__device__ __forceinline__ uint32_t op16_off(int r, int c) {
  return (c >> 3) * 2048 + r * 128 + (((c & 7) ^ (r & 7)) << 4);
}

struct DUnit {   // one published unit
  int u;         // unit index (-1: end)
  int t, pos;    // token row, position (ctx): keys 0..pos
};
}  // namespace

__global__ void __launch_bounds__(NT, 1)
    k_attn_decode5(const __grid_constant__ CUtensorMap mk, const __grid_constant__ CUtensorMap mv, AttnArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();   // q and the new token's k / v come from the QKV GEMM
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = smem_raw;
  if (smem_u32(sm) & 1023) __trap();
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + OFF_BAR);
  uint64_t *kvfull = bars, *kvempty = kvfull + NSTG;        // [NSTG]
  uint64_t *ufull = kvempty + NSTG, *uempty = ufull + 2;    // [2] unit ring (also Q slot)
  uint64_t *qempty = uempty + 2;                            // [2] Q slot free (S MMAs of its unit done)
  uint64_t *sfull = qempty + 2, *sempty = sfull + 2;        // [2] S buffers
  uint64_t *pfull = sempty + 2, *pvdone = pfull + 2;        // [2] P buffers / their PV done
  uint64_t *odone = pvdone + 2, *oempty = odone + 1;        // O of the unit complete / read out
  uint32_t* tslot = reinterpret_cast<uint32_t*>(oempty + 1);
  DUnit* ring = reinterpret_cast<DUnit*>(tslot + 2);        // [2]
  float* red = reinterpret_cast<float*>(sm + OFF_RED);      // [3][4][8]
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int grp = a.H / a.Hkv;
  const int units = (a.n_tok - a.tok_base) * a.Hkv;
  const uint32_t sbase = smem_u32(sm);
  if (tid == 0) {
    for (int i = 0; i < NSTG; ++i) { mbar_init(kvfull + i, 1); mbar_init(kvempty + i, 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(ufull + i, 1);
      mbar_init(uempty + i, 1 + 4);   // MMA warp + softmax warps (lane 0 each)
      mbar_init(qempty + i, 1);
      mbar_init(sfull + i, 1);
      mbar_init(sempty + i, 4);
      mbar_init(pfull + i, 4);
      mbar_init(pvdone + i, 1);
    }
    mbar_init(odone, 1);
    mbar_init(oempty, 4);
    mbar_fence_init();
  }
  // rows of heads >= grp in the Q^T and P^T operands stay zero
  for (int i = tid; i < (2 * QB_BYTES + 2 * PB_BYTES) / 16; i += NT)
    reinterpret_cast<uint4*>(sm + OFF_Q)[i] = make_uint4(0, 0, 0, 0);
  if (warp == W_MMA) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_async_smem();
  tc_before();
  __syncthreads();
  tc_after();
  const uint32_t tmem = *tslot;
  const uint32_t t_o = tmem + 32;   // S buffers at columns [0,16), [16,32); O^T at [32,48)

  if (warp == W_PROD) {
    // ---------------- claimer + producer: units in LPT order, Q^T rows into the unit's slot, K / V tiles by TMA
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
    uint32_t g_tile = 0;   // tiles issued by this CTA (stage ring position)
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      int u = 0;
      if (lane == 0) u = atomicAdd(a.L.ctr, 1);
      u = __shfl_sync(0xffffffffu, u, 0);
      if (n >= 2) mbar_wait(uempty + slot, ((n - 2) >> 1) & 1);
      DUnit U{-1, 0, 0};
      int r = 0;
      if (u < units) {
        U.u = u;
        if (a.order) {
          const int4 od = __ldg(a.order + u / a.Hkv);
          U.t = a.tok_base + od.x; r = od.y; U.pos = od.z;
        } else {
          U.t = a.tok_base + u / a.Hkv;
          r = find_req(a.cu, a.n_reqs, U.t);
          U.pos = __ldg(a.ctx + r) + (U.t - __ldg(a.cu + r));
        }
      }
      if (lane == 0) ring[slot] = U;
      if (u >= units) {
        __syncwarp();
        if (lane == 0) { mbar_arrive(ufull + slot); pdl_trigger(); }
        break;
      }
      if (lane == 0) log_unit(a.L, u);
      const int g = u % a.Hkv;
      // Q^T: rows h < grp of the unit's heads (256 B each) into slot `slot`, 128-byte swizzle
      if (n >= 2) mbar_wait(qempty + slot, ((n - 2) >> 1) & 1);
      {
        uint8_t* qs = sm + OFF_Q + slot * QB_BYTES;
        const uint4* src = reinterpret_cast<const uint4*>(qg + (size_t)U.t * a.H * HD + (size_t)g * grp * HD);
        for (int i = lane; i < grp * 16; i += 32) {
          const int h = i >> 4, c = i & 15;
          *reinterpret_cast<uint4*>(qs + op16_off(h, c)) = __ldg(src + i);
        }
        fence_async_smem();
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(ufull + slot);   // unit + Q published
      // K / V tiles
      const int nb = U.pos / KB + 1, n_t = (nb + 7) / 8;
      const int32_t* bt = a.bt + (size_t)r * a.max_blocks;
      int cur = lane < nb ? __ldg(bt + lane) : -1;                 // entries of window w (4 tiles)
      int nxt = 32 + lane < nb ? __ldg(bt + 32 + lane) : -1;
      for (int t = 0; t < n_t; ++t, ++g_tile) {
        if (t > 0 && (t & 3) == 0) {
          cur = nxt;
          const int e = (t / 4 + 1) * 32 + lane;
          nxt = e < nb ? __ldg(bt + e) : -1;
        }
        const int st = g_tile % NSTG;
        if (g_tile >= NSTG) mbar_wait(kvempty + st, ((g_tile / NSTG) - 1) & 1);
        int blk[8];
#pragma unroll
        for (int b = 0; b < 8; ++b) blk[b] = __shfl_sync(0xffffffffu, cur, (t & 3) * 8 + b);
        if (elect_one()) {
          uint64_t* bar = kvfull + st;
          mbar_arrive_expect_tx(bar, ST_BYTES);
          uint8_t* ks = sm + st * ST_BYTES;
#pragma unroll
          for (int b = 0; b < 8; ++b) {
            // past the sequence: an out-of-bounds box (rows -16..-1) reads as zeros
            const int row = blk[b] >= 0 ? (blk[b] * a.Hkv + g) * KB : -KB;
#pragma unroll
            for (int half = 0; half < 2; ++half) {
              tma_kv(ks + half * (KT_BYTES / 2) + b * KB * 128, &mk, bar, half * 64, row, pol);
              tma_kv(ks + KT_BYTES + half * (KT_BYTES / 2) + b * KB * 128, &mv, bar, half * 64, row, pol);
            }
          }
        }
        __syncwarp();
      }
    }
  } else if (warp == W_MMA) {
    // ---------------- MMA issuer (whole warp runs the loop, one elected lane issues)
    // f32 accumulate, bf16 operands, M = 128, N = 16; S: A K-major (keys x dims), B K-major (heads x dims);
    // PV: A MN-major (V [key][dim] read as dims x keys), B K-major (P^T rows x keys)
    const uint32_t id_s = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(16 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    const uint32_t id_o = id_s | (1u << 15);
    uint32_t g_tile = 0, g_pv = 0;
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      mbar_wait(ufull + slot, (n >> 1) & 1);
      const DUnit U = ring[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(uempty + slot);
      if (U.u < 0) break;
      const int n_t = (U.pos / KB + 1 + 7) / 8;
      const uint32_t qa = sbase + OFF_Q + slot * QB_BYTES;
      auto issue_pv = [&](uint32_t gt, bool first) {   // O^T += V(gt)^T . P^T(gt)
        const int pb = g_pv & 1;
        mbar_wait(pfull + pb, (g_pv >> 1) & 1);
        if (first && n >= 1) mbar_wait(oempty, (n - 1) & 1);   // previous unit's O read out
        tc_after();
        const uint32_t va = sbase + (gt % NSTG) * ST_BYTES + KT_BYTES, pa = sbase + OFF_P + pb * PB_BYTES;
        if (elect_one()) {
          if (!(a.dbg & 16))   // (diagnostics: bit 4 skips the PV MMAs)
#pragma unroll
          for (int kk = 0; kk < TK / 16; ++kk)
            tc_mma(t_o, desc_mn(va + kk * 2048), desc_k(pa + (kk >> 2) * 2048 + (kk & 3) * 32), id_o,
                   (!first || kk > 0) ? 1u : 0u);
          tc_commit(pvdone + pb);
          tc_commit(kvempty + gt % NSTG);
        }
        __syncwarp();
        ++g_pv;
      };
      for (int t = 0; t < n_t; ++t, ++g_tile) {
        const int st = g_tile % NSTG, sb = g_tile & 1;
        mbar_wait(kvfull + st, (g_tile / NSTG) & 1);
        if (g_tile >= 2) mbar_wait(sempty + sb, ((g_tile - 2) >> 1) & 1);   // softmax read S(g-2)
        tc_after();
        const uint32_t ka = sbase + st * ST_BYTES;
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < HD / 16; ++kk)
            tc_mma(tmem + sb * 16, desc_k(ka + (kk >> 2) * (KT_BYTES / 2) + (kk & 3) * 32),
                   desc_k(qa + (kk >> 2) * 2048 + (kk & 3) * 32), id_s, kk > 0 ? 1u : 0u);
          tc_commit(sfull + sb);
          if (t == n_t - 1) tc_commit(qempty + slot);
        }
        __syncwarp();
        if (t > 0) issue_pv(g_tile - 1, t == 1);
      }
      issue_pv(g_tile - 1, n_t == 1);
      if (elect_one()) tc_commit(odone);
      __syncwarp();
    }
  } else {
    // ---------------- softmax + epilogue: thread = key (S) / dim (O) = TMEM lane q * 32 + lane
    const int q4 = warp & 3, wi = warp - W_SM0, row = q4 * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q4 * 32) << 16;
    const float sl2 = a.scale * 1.4426950408889634f;
    __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
    uint32_t g_tile = 0;
    for (int n = 0;; ++n) {
      const int slot = n & 1;
      mbar_wait(ufull + slot, (n >> 1) & 1);
      const DUnit U = ring[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(uempty + slot);
      if (U.u < 0) break;
      const int g = U.u % a.Hkv, n_t = (U.pos / KB + 1 + 7) / 8;
      float m_ref[GMAX], lp[GMAX];
#pragma unroll
      for (int h = 0; h < GMAX; ++h) { m_ref[h] = -INFINITY; lp[h] = 0.f; }
      for (int t = 0; t < n_t; ++t, ++g_tile) {
        const int sb = g_tile & 1;
        mbar_wait(sfull + sb, (g_tile >> 1) & 1);
        tc_after();
        float s[16];
        tmem_ld16(tmem + sb * 16 + lane_off, s);
        tc_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(sempty + sb);
        if (a.dbg & 32) {   // diagnostics (BULLET_DBG, wrong results): hand-offs only
          const int pb = g_tile & 1;
          if (g_tile >= 2) mbar_wait(pvdone + pb, ((g_tile - 2) >> 1) & 1);
          __syncwarp();
          if (lane == 0) mbar_arrive(pfull + pb);
          continue;
        }
        const bool ok = t * TK + row <= U.pos;   // keys 0..pos are visible
        float mx[GMAX];
#pragma unroll
        for (int h = 0; h < GMAX; ++h) {
          s[h] = ok ? s[h] * sl2 : -INFINITY;
          mx[h] = s[h];
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
          for (int h = 0; h < GMAX; ++h)
            if (h < grp) mx[h] = fmaxf(mx[h], __shfl_xor_sync(0xffffffffu, mx[h], o));
        float* rb = red + (t & 1) * 32;   // [4 warps][8 heads], alternating per tile
        if (lane < GMAX) {
          float v = mx[0];
#pragma unroll
          for (int h = 1; h < GMAX; ++h) v = lane == h ? mx[h] : v;
          rb[wi * 8 + lane] = v;
        }
        if (!(a.dbg & 4)) named_bar_sync(1, 128);   // (diagnostics: bit 2 skips the exchange's barrier)
        float alpha[GMAX];
        bool any = false;
#pragma unroll
        for (int h = 0; h < GMAX; ++h) {
          const float tm = fmaxf(fmaxf(rb[h], rb[8 + h]), fmaxf(rb[16 + h], rb[24 + h]));
          const bool move = tm > m_ref[h] + 8.f;   // includes m_ref = -inf (first tile)
          alpha[h] = move ? ex2(m_ref[h] - tm) : 1.f;
          if (move) m_ref[h] = tm;
          any |= move && h < grp;
        }
        // P^T(t) into buffer pb once PV(t - 2) has read it
        const int pb = g_tile & 1;
        if (g_tile >= 2) mbar_wait(pvdone + pb, ((g_tile - 2) >> 1) & 1);
        if (t > 0 && any) {   // lazy rescale of O^T: PV(t - 1) must be complete (pvdone of the other buffer)
          mbar_wait(pvdone + (pb ^ 1), ((g_tile - 1) >> 1) & 1);
          tc_after();
          float o[16];
          tmem_ld16(t_o + lane_off, o);
#pragma unroll
          for (int h = 0; h < GMAX; ++h) { o[h] *= alpha[h]; o[8 + h] *= alpha[h]; }
          tmem_st16(t_o + lane_off, o);
          tc_before();
        }
        uint8_t* ps = sm + OFF_P + pb * PB_BYTES;
        const int c16 = row >> 3, byte = (row & 7) * 2;   // key = row: 16-byte chunk row / 8 of the 128-key row
#pragma unroll
        for (int h = 0; h < GMAX; ++h) {
          if (h < grp) {
            const float p = ex2(s[h] - m_ref[h]);
            lp[h] = lp[h] * alpha[h] + p;
            // P = hi + lo, both truncated bf16 (hi exact prefix, lo the remainder's prefix: < 2^-15 |P|)
            const uint32_t up = __float_as_uint(p);
            const float rem = p - __uint_as_float(up & 0xFFFF0000u);
            if (!(a.dbg & 8)) {   // (diagnostics: bit 3 skips the P stores)
              *reinterpret_cast<uint16_t*>(ps + op16_off(h, c16) + byte) = (uint16_t)(up >> 16);
              *reinterpret_cast<uint16_t*>(ps + op16_off(8 + h, c16) + byte) = (uint16_t)(__float_as_uint(rem) >> 16);
            }
          }
        }
        fence_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(pfull + pb);
      }
      // ---- epilogue: l per head over the 128 threads, then O = (O^T[:, h] + O^T[:, 8 + h]) / l
#pragma unroll
      for (int o = 16; o > 0; o >>= 1)
#pragma unroll
        for (int h = 0; h < GMAX; ++h)
          if (h < grp) lp[h] += __shfl_xor_sync(0xffffffffu, lp[h], o);
      float* rl = red + 64;   // [4][8] after the two max buffers
      if (lane < GMAX) {
        float v = lp[0];
#pragma unroll
        for (int h = 1; h < GMAX; ++h) v = lane == h ? lp[h] : v;
        rl[wi * 8 + lane] = v;
      }
      named_bar_sync(1, 128);
      mbar_wait(odone, n & 1);
      tc_after();
      float o[16];
      tmem_ld16(t_o + lane_off, o);
      tc_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(oempty);
      __nv_bfloat16* dst = og + (size_t)U.t * a.H * HD + (size_t)g * grp * HD + row;
#pragma unroll
      for (int h = 0; h < GMAX; ++h)
        if (h < grp) {
          const float l = (rl[h] + rl[8 + h]) + (rl[16 + h] + rl[24 + h]);
          dst[(size_t)h * HD] = __float2bfloat16_rn((o[h] + o[8 + h]) / l);
        }
      named_bar_sync(1, 128);   // rl is rewritten by the next unit
    }
  }
  tc_before();
  __syncthreads();
  if (warp == W_MMA) {
    tc_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

size_t attn_decode5_smem_bytes() { return SMEM_BYTES; }

// grid = n_sms (one CTA per SM, persistent, gated); GQA group <= 8, head_dim 128, block 16.
cudaError_t launch_attn_decode5(const CUtensorMap& mk, const CUtensorMap& mv, const AttnArgs& a, int grid,
                                cudaStream_t st) {
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_decode5, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return e;
    set = true;
  }
  return launch_ex(k_attn_decode5, grid, NT, SMEM_BYTES, st, a.L.pdl, mk, mv, a);
}

cudaError_t preload_attn_decode5() {
  cudaFuncAttributes f;
  return cudaFuncGetAttributes(&f, k_attn_decode5);
}

}  // namespace bl
