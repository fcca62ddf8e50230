// attn_prefill5.cu — causal prefill attention on 5th-gen tensor cores
// (tcgen05 + TMEM), bf16, head_dim 128 (the paper's
// FlashAttention).
//
// Work unit = (request, 128-row query tile, query head), LPT order from the
// plan kernel.  Two CTAs per SM (96 KB smem, 256 TMEM columns each).  Per
// 64-key KV tile t:
//   S(t) = Q K(t)^T   tcgen05.mma M=128 (queries) N=64 (keys) -> TMEM fp32,
//                     double-buffered so S(t+1) runs during softmax(t)
//   softmax           4 warps, thread r owns query row r = TMEM lane r:
//                     tcgen05.ld, causal mask, exp2 against a lazily moved
//                     reference max, P = hi + lo (two bf16 halves, R-4b)
//                     tcgen05.st'd over S(t) in TMEM
//   O += P V          tcgen05.mma with A = P from TMEM, B = V(t) used as an
//                     MN-major operand straight from its [key][dim] tile; O
//                     stays in TMEM, rescaled only when a row max grows > 2^8
// One __syncthreads per tile: after it one thread issues S(t+1) and PV(t)
// back to back.  K/V rows are gathered through the block table with coalesced
// cp.async into the 128-byte-swizzled layouts the UMMA descriptors describe,
// two buffers each: K(t+2) loads from tile t on, V(t+1) during tile t.
#include "kernels.h"

namespace bl {

namespace {
constexpr int BQ = 128, BKV = 64, HD = 128, KB = 16, NT = 128;
// smem: Q [2][128][128 B] | K[2 buffers] [2][64][128 B] | V[2 buffers] [2][64][128 B]
// = 96 KB + barriers: two CTAs per SM.  The dynamic window must start
// 1024-byte aligned (128-byte swizzle atoms); checked at entry.
constexpr int OFF_Q = 0, OFF_K = 32768, OFF_V = 65536;
constexpr int SMEM_BYTES = 98304 + 64;
// TMEM: S/P double buffer in columns [0,64) and [64,128) (P = bf16 hi|lo
// packed two per column, written over the S it came from), O in [128,256)
constexpr uint32_t TMEM_COLS = 256;

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
}  // namespace

__global__ void __launch_bounds__(NT, 2) k_attn_prefill5(AttnArgs a) {
  if (!gate_ok(a.L.gate)) return;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = smem_raw;
  if (smem_u32(sm) & 1023) __trap();   // swizzle atoms need 1024-byte alignment
  uint64_t* bar_s = reinterpret_cast<uint64_t*>(sm + 98304);
  uint64_t* bar_o = bar_s + 1;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bar_o + 1);
  int* s_u = reinterpret_cast<int*>(tslot + 1);
  const int tid = threadIdx.x, warp = tid >> 5;
  const uint32_t sbase = smem_u32(sm);
  if (tid == 0) { mbar_init(bar_s, 1); mbar_init(bar_o, 1); mbar_fence_init(); }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)), "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_before();
  __syncthreads();
  tc_after();
  const uint32_t tmem = *tslot;
  const uint32_t t_s = tmem, t_o = tmem + 128;
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
  // f32 accumulate, bf16 A/B; S: N = 64, B K-major; O: N = 128, B MN-major
  const uint32_t id_s = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BKV >> 3) << 17) | ((uint32_t)(BQ >> 4) << 24);
  const uint32_t id_o = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(HD >> 3) << 17) |
                        ((uint32_t)(BQ >> 4) << 24);
  const int grp = a.H / a.Hkv;
  const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
  const __nv_bfloat16* pk = reinterpret_cast<const __nv_bfloat16*>(a.pool_k);
  const __nv_bfloat16* pv = reinterpret_cast<const __nv_bfloat16*>(a.pool_v);
  __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
  const float sl2 = a.scale * 1.4426950408889634f;
  const int units = (*a.n_tiles) * a.H;
  uint32_t ph_s = 0, ph_o = 0;

  for (;;) {
    if (tid == 0) *s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int u = *s_u;
    __syncthreads();
    if (u >= units) break;
    if (tid == 0) log_unit(a.L, u);
    const int2 rt = a.tiles[u / a.H];
    const int h = u % a.H, g = h / grp, r = rt.x, q0 = rt.y * BQ;
    const int tok0 = __ldg(a.cu + r);
    const int q_len = __ldg(a.cu + r + 1) - tok0;
    const int ctx = __ldg(a.ctx + r);
    const int kv_len = ctx + q_len;
    const int kmax = min(kv_len, ctx + q0 + BQ);
    const int n_kt = (kmax + BKV - 1) / BKV;
    const int32_t* bt = a.bt + (size_t)r * a.max_blocks;

    // coalesced gathers: 16 lanes per 256-byte row
    {
#pragma unroll
      for (int i = 0; i < 16; ++i) {   // Q: 128 rows x 16 chunks
        const int e = tid + NT * i, row = e >> 4, c = e & 15;
        const bool ok = q0 + row < q_len;
        cp_async16_zfill(sm + OFF_Q + sw(row, c, 16384),
                         qg + (size_t)(tok0 + (ok ? q0 + row : 0)) * a.H * HD + h * HD + c * 8, ok);
      }
    }
    auto load_kv = [&](int kt, int off, const __nv_bfloat16* pool) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {    // 64 rows x 16 chunks
        const int e = tid + NT * i, row = e >> 4, c = e & 15;
        const int kp = kt * BKV + row;
        const bool ok = kp < kv_len;
        const int blk = ok ? __ldg(bt + kp / KB) : 0;
        cp_async16_zfill(sm + off + sw(row, c, 8192),
                         pool + (((size_t)blk * a.Hkv + g) * KB + (ok ? kp % KB : 0)) * HD + c * 8, ok);
      }
    };
    auto issue_s = [&](int kt) {       // S(kt) = Q K(kt)^T -> TMEM buffer kt&1
      const uint32_t qa = sbase + OFF_Q, ka = sbase + OFF_K + (kt & 1) * 16384;
#pragma unroll
      for (int kk = 0; kk < HD / 16; ++kk)
        tc_mma(t_s + (kt & 1) * 64, desc_k(qa + (kk >> 2) * 16384 + (kk & 3) * 32),
               desc_k(ka + (kk >> 2) * 8192 + (kk & 3) * 32), id_s, kk > 0 ? 1u : 0u);
      tc_commit(bar_s);
    };
    // cp.async groups, oldest first: {Q, K0, V0}, {K1}, then per tile t
    // {K(t+2)}, {V(t+1)}; waiting for all but the newest two before tile
    // t's MMAs leaves exactly K(t+2), V(t+1) in flight.
    load_kv(0, OFF_K, pk);
    load_kv(0, OFF_V, pv);
    cp_async_commit();
    if (n_kt > 1) load_kv(1, OFF_K + 16384, pk);
    cp_async_commit();
    cp_async_wait<1>();
    fence_async_smem();
    tc_before();
    __syncthreads();
    tc_after();
    if (tid == 0) issue_s(0);

    float m_ref = -INFINITY, l_run = 0.f;
    const int qpos = ctx + q0 + tid;

    for (int kt = 0; kt < n_kt; ++kt) {
      const uint32_t t_sb = t_s + (kt & 1) * 64;
      mbar_wait(bar_s, ph_s);        // S(kt) in TMEM
      ph_s ^= 1;
      tc_after();
      if (kt + 2 < n_kt) load_kv(kt + 2, OFF_K + (kt & 1) * 16384, pk);   // K buffer of S(kt) is free
      cp_async_commit();
      // ---- softmax of row tid over the 64 keys of this tile; P -> TMEM in
      //      place of S(kt) (hi in columns [0,32), lo in [32,64) of the buffer)
      float v[64];
      tmem_ld32(t_sb + lane_off, v);
      tmem_ld32(t_sb + lane_off + 32, v + 32);
      // only tiles crossing the causal diagonal or the end of the sequence
      // need the per-element mask (CTA-uniform test)
      if ((kt + 1) * BKV - 1 > ctx + q0 || (kt + 1) * BKV > kv_len) {
#pragma unroll
        for (int i = 0; i < 64; ++i) {
          const int kp = kt * BKV + i;
          if (!(kp <= qpos && kp < kv_len)) v[i] = -INFINITY;
        }
      }
      float mx = v[0];
#pragma unroll
      for (int i = 1; i < 64; ++i) mx = fmaxf(mx, v[i]);
      const float mx_s = mx * sl2;                  // scale > 0 commutes with max
      const bool move = mx_s > m_ref + 8.f;         // includes m_ref = -inf (first tile)
      const float m_new = move ? mx_s : m_ref;
      const float alpha = move ? ex2(m_ref - m_new) : 1.f;
      float ls;
      {
        uint32_t hi[32], lo[32];
        float2 acc = make_float2(0.f, 0.f);
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const float2 t = ffma2(make_float2(v[2 * j], v[2 * j + 1]), sl2, -m_new);
          const float2 pp = make_float2(ex2(t.x), ex2(t.y));
          acc = fadd2(acc, pp);
          const uint32_t h = pack_bf2(pp.x, pp.y);
          const float2 l = fsub2(pp, make_float2(__uint_as_float(h << 16), __uint_as_float(h & 0xFFFF0000u)));
          hi[j] = h;
          lo[j] = pack_bf2(l.x, l.y);
        }
        ls = acc.x + acc.y;
        tmem_st32(t_sb + lane_off, reinterpret_cast<const float*>(hi));
        tmem_st32(t_sb + lane_off + 32, reinterpret_cast<const float*>(lo));
      }
      if (kt > 0) {                  // PV(kt-1) done: O may be rescaled, its V / P buffers reused
        mbar_wait(bar_o, ph_o);
        ph_o ^= 1;
        tc_after();
        if (__any_sync(0xffffffffu, move)) {   // warp-uniform lazy rescale of O (> 2^8 growth)
          float w[32];
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            tmem_ld32(t_o + lane_off + c * 32, w);
#pragma unroll
            for (int i = 0; i < 32; ++i) w[i] *= alpha;
            tmem_st32(t_o + lane_off + c * 32, w);
          }
        }
      }
      l_run = l_run * alpha + ls;
      m_ref = m_new;
      if (kt + 1 < n_kt) load_kv(kt + 1, OFF_V + ((kt + 1) & 1) * 16384, pv);
      cp_async_commit();
      cp_async_wait<2>();            // K(kt+1), V(kt) landed
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      fence_async_smem();
      tc_before();
      __syncthreads();
      tc_after();
      if (tid == 0) {
        if (kt + 1 < n_kt) issue_s(kt + 1);   // overwrites P(kt-1): PV(kt-1) is done
        // ---- O += P V   (A = P from TMEM, B = V(kt) MN-major from smem)
        const uint32_t va = sbase + OFF_V + (kt & 1) * 16384;
#pragma unroll
        for (int kk = 0; kk < BKV / 16; ++kk)
          tc_mma_ts(t_o, t_sb + kk * 8, desc_mn(va + kk * 2048), id_o, (kt > 0 || kk > 0) ? 1u : 0u);
#pragma unroll
        for (int kk = 0; kk < BKV / 16; ++kk)
          tc_mma_ts(t_o, t_sb + 32 + kk * 8, desc_mn(va + kk * 2048), id_o, 1u);
        tc_commit(bar_o);
      }
    }
    mbar_wait(bar_o, ph_o);          // last PV
    ph_o ^= 1;
    tc_after();
    // ---- normalise and store row tid (bf16, point R3)
    {
      const float inv = 1.f / l_run;
      const bool ok = q0 + tid < q_len;
      __nv_bfloat16* dst = og + (size_t)(tok0 + q0 + (ok ? tid : 0)) * a.H * HD + h * HD;
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
    }
    tc_before();
    __syncthreads();
    tc_after();
  }
  if (warp == 0) {
    tc_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

cudaError_t launch_attn_prefill5(const AttnArgs& a, int grid, cudaStream_t st) {
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_prefill5, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return e;
    set = true;
  }
  k_attn_prefill5<<<grid, NT, SMEM_BYTES, st>>>(a);
  return cudaGetLastError();
}

}  // namespace bl
