// attn_tc.cu — causal prefill attention on tensor cores (the
// paper's FlashAttention), bf16, head_dim 128.
//
// Work unit = (request, 64-row query tile, query head); tiles are listed
// longest key range first by the plan kernel.  K/V tiles of 64 keys are
// gathered through the block table from the paged pool with 16-byte
// cp.async into XOR-swizzled shared memory (double-buffered).  Each of the
// 4 warps owns 16 query rows: S = Q K^T with mma.m16n8k16 bf16 -> fp32,
// online softmax in fp32 (exp2), then O += P V with V in fp16 and P as an
// fp16 hi + lo pair (DESIGN R-4b: a single bf16 or fp16 P adds measurable
// error at the 1e-3 bar; bf16 -> fp16 is exact for |v| in [2^-14, 65504]).  Round-1 kernel: mma.sync; the tcgen05 version is the
// next step.
#include "kernels.h"

namespace bl {

namespace {
constexpr int BQ = 64, BKV = 64, HDIM = 128, KB = 16;
constexpr int TILE_BYTES = 64 * HDIM * 2;  // 16 KB

__device__ __forceinline__ uint32_t swz(int row, int chunk) {  // byte offset in a [64][128] bf16 tile
  return row * 256 + ((chunk ^ (row & 7)) << 4);
}
__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(addr));
}
__device__ __forceinline__ void mma_bf16(float* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void mma_f16(float* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t bf2_to_h2(uint32_t x) {
  __nv_bfloat162 b = *reinterpret_cast<__nv_bfloat162*>(&x);
  __half2 h = __float22half2_rn(__bfloat1622float2(b));
  return *reinterpret_cast<uint32_t*>(&h);
}
__device__ __forceinline__ uint32_t pack_h2(float lo, float hi) {
  __half2 h = __floats2half2_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}
// x -> (hi, lo) fp16 pairs with hi = fp16(x), lo = fp16(x - hi).
__device__ __forceinline__ void split_h2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
  __half2 h = __floats2half2_rn(x0, x1);
  const float2 hf = __half22float2(h);
  __half2 l = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
  hi = *reinterpret_cast<uint32_t*>(&h);
  lo = *reinterpret_cast<uint32_t*>(&l);
}
__device__ __forceinline__ void cp_async16_zfill(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(valid ? 16 : 0)
               : "memory");
}
}  // namespace

__global__ void __launch_bounds__(128) k_attn_prefill_tc(AttnArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  extern __shared__ __align__(128) uint8_t sm[];
  uint8_t* Qs = sm;
  uint8_t* Ks = sm + TILE_BYTES;          // [2][64][128]
  uint8_t* Vs = sm + 3 * TILE_BYTES;      // [2][64][128]
  __shared__ int s_u;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int gq = lane >> 2, tq = lane & 3;
  const int grp = a.H / a.Hkv;
  const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
  const __nv_bfloat16* pk = reinterpret_cast<const __nv_bfloat16*>(a.pool_k);
  const __nv_bfloat16* pv = reinterpret_cast<const __nv_bfloat16*>(a.pool_v);
  __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
  const float sl2 = a.scale * 1.4426950408889634f;
  const int units = (*a.n_tiles) * a.H;

  for (;;) {
    if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int u = s_u;
    __syncthreads();
    if (u >= units) break;
    if (tid == 0) log_unit(a.L, u);
    const int2 rt = a.tiles[u / a.H];
    const int h = u % a.H, g = h / grp, r = rt.x;
    const int tok0 = __ldg(a.cu + r);
    const int q_len = __ldg(a.cu + r + 1) - tok0;
    for (int q0 = rt.y * ATTN_TC_BQ; q0 < min(q_len, (rt.y + 1) * ATTN_TC_BQ); q0 += BQ) {  // 64-row halves
    const int ctx = __ldg(a.ctx + r);
    const int kv_len = ctx + q_len;
    const int kmax = min(kv_len, ctx + q0 + BQ);
    const int n_kt = (kmax + BKV - 1) / BKV;
    const int32_t* bt = a.bt + (size_t)r * a.max_blocks;

    // Q tile (rows beyond q_len zero-filled)
    for (int e = tid; e < BQ * 16; e += 128) {
      const int row = e >> 4, c = e & 15;
      const bool ok = (q0 + row) < q_len;
      const __nv_bfloat16* src = qg + (size_t)(tok0 + (ok ? q0 + row : 0)) * a.H * HDIM + h * HDIM + c * 8;
      cp_async16_zfill(Qs + swz(row, c), src, ok);
    }
    auto load_kv = [&](int kt, int st) {
      for (int e = tid; e < BKV * 16; e += 128) {
        const int row = e >> 4, c = e & 15;
        const int kp = kt * BKV + row;
        const bool ok = kp < kv_len;
        const int blk = ok ? __ldg(bt + kp / KB) : 0;
        const size_t off = (((size_t)blk * a.Hkv + g) * KB + (ok ? kp % KB : 0)) * HDIM + c * 8;
        cp_async16_zfill(Ks + st * TILE_BYTES + swz(row, c), pk + off, ok);
        cp_async16_zfill(Vs + st * TILE_BYTES + swz(row, c), pv + off, ok);
      }
    };
    load_kv(0, 0);
    cp_async_commit();

    uint32_t qf[8][4];
    float oacc[16][4];
#pragma unroll
    for (int i = 0; i < 16; ++i) oacc[i][0] = oacc[i][1] = oacc[i][2] = oacc[i][3] = 0.f;
    float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
    const int qpos0 = ctx + q0 + warp * 16 + gq;  // positions of rows gq and gq+8

    for (int kt = 0; kt < n_kt; ++kt) {
      if (kt + 1 < n_kt) load_kv(kt + 1, (kt + 1) & 1);
      cp_async_commit();
      cp_async_wait<1>();
      __syncthreads();
      if (kt == 0) {
#pragma unroll
        for (int ks = 0; ks < 8; ++ks)
          ldsm_x4(smem_u32(Qs) + swz(warp * 16 + (lane & 15), ks * 2 + (lane >> 4)), qf[ks][0],
                  qf[ks][1], qf[ks][2], qf[ks][3]);
      }
      const uint32_t kbase = smem_u32(Ks + (kt & 1) * TILE_BYTES);
      const uint32_t vbase = smem_u32(Vs + (kt & 1) * TILE_BYTES);
      float s[8][4];
#pragma unroll
      for (int i = 0; i < 8; ++i) s[i][0] = s[i][1] = s[i][2] = s[i][3] = 0.f;
#pragma unroll
      for (int ks = 0; ks < 8; ++ks)
#pragma unroll
        for (int np = 0; np < 4; ++np) {
          uint32_t b0, b1, b2, b3;
          const int mi = lane >> 3;
          ldsm_x4(kbase + swz((2 * np + (mi >> 1)) * 8 + (lane & 7), ks * 2 + (mi & 1)), b0, b1, b2, b3);
          mma_bf16(s[2 * np], qf[ks], b0, b1);
          mma_bf16(s[2 * np + 1], qf[ks], b2, b3);
        }
      // causal + length mask, online softmax (rows gq, gq+8)
      float mx[2] = {-INFINITY, -INFINITY};
#pragma unroll
      for (int nt = 0; nt < 8; ++nt)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int kj = kt * BKV + nt * 8 + 2 * tq + (e & 1);
          const int qp = qpos0 + (e >> 1) * 8;
          const float v = (kj <= qp && kj < kv_len) ? s[nt][e] * sl2 : -INFINITY;
          s[nt][e] = v;
          mx[e >> 1] = fmaxf(mx[e >> 1], v);
        }
      float alpha[2];
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        mx[i] = fmaxf(mx[i], __shfl_xor_sync(0xffffffffu, mx[i], 1));
        mx[i] = fmaxf(mx[i], __shfl_xor_sync(0xffffffffu, mx[i], 2));
        const float mn = fmaxf(mrow[i], mx[i]);
        alpha[i] = (mn == -INFINITY) ? 1.f : exp2f(mrow[i] - mn);
        mrow[i] = mn;
      }
      float ps[2] = {0.f, 0.f};
#pragma unroll
      for (int nt = 0; nt < 8; ++nt)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float mn = mrow[e >> 1];
          const float p = (mn == -INFINITY) ? 0.f : exp2f(s[nt][e] - mn);
          s[nt][e] = p;
          ps[e >> 1] += p;
        }
      lrow[0] = lrow[0] * alpha[0] + ps[0];
      lrow[1] = lrow[1] * alpha[1] + ps[1];
#pragma unroll
      for (int nd = 0; nd < 16; ++nd) {
        oacc[nd][0] *= alpha[0]; oacc[nd][1] *= alpha[0];
        oacc[nd][2] *= alpha[1]; oacc[nd][3] *= alpha[1];
      }
      // O += P V with V in fp16 (exact) and P split into two fp16 halves
      // P = P_hi + P_lo (22 significant bits): the P rounding stays far below
      // the bf16 rounding of o (DESIGN R-4b).
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t pa[4], pl[4];
        split_h2(s[2 * kk][0], s[2 * kk][1], pa[0], pl[0]);
        split_h2(s[2 * kk][2], s[2 * kk][3], pa[1], pl[1]);
        split_h2(s[2 * kk + 1][0], s[2 * kk + 1][1], pa[2], pl[2]);
        split_h2(s[2 * kk + 1][2], s[2 * kk + 1][3], pa[3], pl[3]);
#pragma unroll
        for (int ndp = 0; ndp < 8; ++ndp) {
          uint32_t b0, b1, b2, b3;
          const int mi = lane >> 3;
          ldsm_x4_t(vbase + swz(kk * 16 + (mi & 1) * 8 + (lane & 7), ndp * 2 + (mi >> 1)), b0, b1, b2, b3);
          b0 = bf2_to_h2(b0); b1 = bf2_to_h2(b1); b2 = bf2_to_h2(b2); b3 = bf2_to_h2(b3);
          mma_f16(oacc[2 * ndp], pa, b0, b1);
          mma_f16(oacc[2 * ndp + 1], pa, b2, b3);
          mma_f16(oacc[2 * ndp], pl, b0, b1);
          mma_f16(oacc[2 * ndp + 1], pl, b2, b3);
        }
      }
      __syncthreads();
    }
    cp_async_wait<0>();
    // finalize: full row sums across the quad, normalise, store bf16 (point R3)
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      lrow[i] += __shfl_xor_sync(0xffffffffu, lrow[i], 1);
      lrow[i] += __shfl_xor_sync(0xffffffffu, lrow[i], 2);
    }
#pragma unroll
    for (int half = 0; half < 2; ++half) {
      const int row = q0 + warp * 16 + gq + half * 8;
      if (row < q_len) {
        const float inv = 1.f / lrow[half];
        __nv_bfloat16* dst = og + (size_t)(tok0 + row) * a.H * HDIM + h * HDIM + 2 * tq;
#pragma unroll
        for (int nd = 0; nd < 16; ++nd)
          *reinterpret_cast<__nv_bfloat162*>(dst + nd * 8) =
              __floats2bfloat162_rn(oacc[nd][2 * half] * inv, oacc[nd][2 * half + 1] * inv);
      }
    }
    __syncthreads();
    }
  }
}

cudaError_t launch_attn_prefill_tc(const AttnArgs& a, int grid, cudaStream_t st) {
  const int smem = 5 * TILE_BYTES;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_prefill_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    set = true;
  }
  cudaError_t e = launch_ex(k_attn_prefill_tc, grid, 128, smem, st, a.L.pdl, a);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

cudaError_t preload_attn_tc() {
  cudaFuncAttributes f;
  return cudaFuncGetAttributes(&f, k_attn_prefill_tc);
}

}  // namespace bl
