// attn_decode2.cu — paged decode attention, register-direct, bf16, hd 128
// (one query token per request over its ctx + 1 keys,
// gathered through the block table; P:L42 decode, P:L69 paged attention).
//
// Why register-direct: KI2 (profiles/r01_ki2_producer.jsonl) measured the
// per-SM HBM read rate by load path: async copies into shared memory
// (cp.async, cp.async.bulk) stop at ~80-88 GB/s per SM, LDG.128 into
// registers reaches ~140-155 GB/s per SM below HBM saturation.  A decode
// partition of m SMs saturates HBM only with the register path, so this
// kernel feeds mma.sync straight from LDG'd registers (no shared memory).
//
// Work unit = (decode token t, kv head, chunk of `cb` KV blocks), one warp
// per unit, 16 warps per SM claiming units from the gated counter; units
// of one (t, head) write (m, l, O) partials and the last of them (atomic
// ticket) merges them in chunk order (deterministic).  Single-chunk units
// write O directly.  The chunk list is built per step by the plan kernel.
//
// Per 16-key block (swap-AB so keys fill M = 16 and the GQA group fills N):
//   S^T[16 keys x 8] = K[16 x 128] . Q^T[128 x 8]     (8 x mma.m16n8k16)
//   O^T[128 x 8]    += V^T[128 x 16] . P^T[16 x 8]    (8 or 16 mma)
// Operand fragments come straight from 16-byte loads: the MMA contraction
// index may be permuted freely, so each lane loads whole 8-dim chunks of K
// rows (K: dims 32s + 8t.., Q loaded with the same permutation) and of V
// rows (V^T rows = dims are permuted the same way on output; key pairs are
// packed with PRMT).  P is never a single bf16: P = hi + lo (R-4b).  For
// GQA groups <= 4 the lo half rides in the unused columns 4..7 of N, so PV
// costs 8 MMAs per block instead of 16.
// Pipelining per warp: K(j+1) is issued right after S(j), V(j+1) right
// after PV(j), so about one 8 KB block is always in flight per warp.
#include <stdlib.h>

#include "kernels.h"

namespace bl {

namespace {
constexpr int KB = 16, HD = 128;
constexpr int NW_MAX = 16;                   // warps per CTA (template NW), one CTA per SM
constexpr int QROW = HD * 2 + 16;            // padded Q row in shared memory (bytes)

__device__ __forceinline__ void mma16816(float* c, uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t movtrans(uint32_t x) {
  uint32_t y;
  asm volatile("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;" : "=r"(y) : "r"(x));
  return y;
}
__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
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
__device__ __forceinline__ uint32_t w_of(const uint4& v, int i) {
  return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w;
}
}  // namespace

// Record of one chunk's partial result: m[8], l[8] (log2 domain), O[grp][128].
__host__ __device__ constexpr int dec_rec_floats(int grp) { return 16 + grp * HD; }

template <bool PK, int NW, int MODE>
__global__ void __launch_bounds__(NW * 32, 1) k_attn_decode2(AttnArgs a) {
  if (!gate_ok(a.L.gate)) return;
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int grp = a.H / a.Hkv;
  const int units = (*a.n_tiles) * a.Hkv;
  const __nv_bfloat16* pk = reinterpret_cast<const __nv_bfloat16*>(a.pool_k);
  const __nv_bfloat16* pv = reinterpret_cast<const __nv_bfloat16*>(a.pool_v);
  const __nv_bfloat16* qg = reinterpret_cast<const __nv_bfloat16*>(a.q);
  __nv_bfloat16* og = reinterpret_cast<__nv_bfloat16*>(a.o);
  const float sl2 = a.scale * 1.4426950408889634f;
  const int rec_f = dec_rec_floats(grp);
  // Q rows of the warp's current unit (8 heads, rows >= grp stay zero)
  __shared__ __align__(16) uint8_t qs_all[NW][8 * QROW];
  uint8_t* qs = qs_all[threadIdx.x >> 5];
  for (int i = lane; i < 8 * QROW / 16; i += 32) reinterpret_cast<uint4*>(qs)[i] = make_uint4(0, 0, 0, 0);
  const uint32_t q_lane = smem_u32(qs) + g * QROW + 16 * t;   // + 64 sx + 4 h: dims 32sx + 8t + 2h

  for (;;) {
    int u = 0;
    if (lane == 0) u = atomicAdd(a.L.ctr, 1);
    u = __shfl_sync(0xffffffffu, u, 0);
    if (u >= units) break;
    if (lane == 0) log_unit(a.L, u);
    const int2 e = a.tiles[u / a.Hkv];           // (token, chunk)
    const int hk = u % a.Hkv, tok = e.x, ch = e.y;
    const int pos = __ldg(a.ctx + tok);          // decode: one token per request
    const int nb = pos / KB + 1, nch = (nb + a.cb - 1) / a.cb;
    const int b0 = ch * a.cb, b1 = min(nb, b0 + a.cb);
    const int32_t* bt = a.bt + (size_t)tok * a.max_blocks;
    const size_t kv_stride = (size_t)a.Hkv * KB * HD;   // elements per block
    // block ids of the chunk, 32 at a time in a lane-distributed register
    int idr = (b0 + lane < b1) ? __ldg(bt + b0 + lane) : 0;
    auto blk_id = [&](int j) { return __shfl_sync(0xffffffffu, idr, (j - b0) & 31); };

    // Q rows of the group into this warp's shared slot (B operand source)
    {
      const uint4* qp = reinterpret_cast<const uint4*>(qg + ((size_t)tok * a.H + hk * grp) * HD);
      __syncwarp();
      for (int i = lane; i < grp * 16; i += 32)
        *reinterpret_cast<uint4*>(qs + (i >> 4) * QROW + (i & 15) * 16) = __ldg(qp + i);
      __syncwarp();
    }
    uint4 kr[2][4];   // keys g, g + 8; dims 32s + 8t .. + 8
    uint4 vr[4][2];   // keys 2t, 2t+1, 2t+8, 2t+9; dims 8(g + 8 sig) .. + 8
    auto load_k = [&](int blk) {
      const uint4* base = reinterpret_cast<const uint4*>(pk + (size_t)blk * kv_stride + (size_t)hk * KB * HD);
#pragma unroll
      for (int kk = 0; kk < 2; ++kk)
#pragma unroll
        for (int s = 0; s < 4; ++s) kr[kk][s] = ldg_stream(base + (g + 8 * kk) * 16 + 4 * s + t);
    };
    auto load_v = [&](int blk) {
      const uint4* base = reinterpret_cast<const uint4*>(pv + (size_t)blk * kv_stride + (size_t)hk * KB * HD);
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const int key = 2 * t + (r & 1) + 8 * (r >> 1);
#pragma unroll
        for (int sg = 0; sg < 2; ++sg) vr[r][sg] = ldg_stream(base + key * 16 + g + 8 * sg);
      }
    };
    float m0 = -INFINITY, m1 = -INFINITY, l0 = 0.f, l1 = 0.f;   // heads 2t, 2t + 1
    float o[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;

    if (MODE != 2) {
      const int id0 = blk_id(b0);
      load_k(id0);
      load_v(id0);
    }
    uint32_t sink = 0;
    for (int j = b0; j < b1; ++j) {
      if (MODE == 2) {   // experiment: both loads at the top, no prefetch
        const int idj = blk_id(j);
        if (((j + 1 - b0) & 31) == 0 && j + 1 < b1) idr = (j + 1 + lane < b1) ? __ldg(bt + j + 1 + lane) : 0;
        load_k(idj);
        load_v(idj);
      }
      if (MODE == 1) {   // experiment: loads only
#pragma unroll
        for (int x = 0; x < 4; ++x) sink ^= kr[0][x].x ^ kr[1][x].y ^ vr[x][0].z ^ vr[x][1].w;
        int idn2 = 0;
        if (j + 1 < b1) {
          if (((j + 1 - b0) & 31) == 0) idr = (j + 1 + lane < b1) ? __ldg(bt + j + 1 + lane) : 0;
          idn2 = blk_id(j + 1);
          load_k(idn2);
          load_v(idn2);
        }
        continue;
      }
      // next block's id (refill the id register every 32 blocks)
      int idn = 0;
      if (MODE == 0 && j + 1 < b1) {
        if (((j + 1 - b0) & 31) == 0) idr = (j + 1 + lane < b1) ? __ldg(bt + j + 1 + lane) : 0;
        idn = blk_id(j + 1);
      }
      // ---- S^T = K . Q^T
      float s[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int ks = 0; ks < 8; ++ks) {
        const int sx = ks >> 1, h = (ks & 1) * 2;
        uint32_t q0, q1;   // Q^T: head g, dims 32sx + 8t + 2h .. + 3
        asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(q0), "=r"(q1) : "r"(q_lane + 64 * sx + 4 * h));
        mma16816(s, w_of(kr[0][sx], h), w_of(kr[1][sx], h), w_of(kr[0][sx], h + 1), w_of(kr[1][sx], h + 1),
                 q0, q1);
      }
      if (MODE == 0 && j + 1 < b1) load_k(idn);
      // ---- online softmax (log2 domain); s: (key g, head 2t), (g, 2t+1), (g+8, 2t), (g+8, 2t+1)
      const int k0 = j * KB + g, k1 = k0 + 8;
      s[0] = k0 <= pos ? s[0] * sl2 : -INFINITY;
      s[1] = k0 <= pos ? s[1] * sl2 : -INFINITY;
      s[2] = k1 <= pos ? s[2] * sl2 : -INFINITY;
      s[3] = k1 <= pos ? s[3] * sl2 : -INFINITY;
      float bm0 = fmaxf(s[0], s[2]), bm1 = fmaxf(s[1], s[3]);
#pragma unroll
      for (int x = 4; x < 32; x <<= 1) {
        bm0 = fmaxf(bm0, __shfl_xor_sync(0xffffffffu, bm0, x));
        bm1 = fmaxf(bm1, __shfl_xor_sync(0xffffffffu, bm1, x));
      }
      const float mn0 = fmaxf(m0, bm0), mn1 = fmaxf(m1, bm1);   // key 16j <= pos: finite
      float al0 = exp2f(m0 - mn0), al1 = exp2f(m1 - mn1);
      m0 = mn0; m1 = mn1;
      const float p00 = exp2f(s[0] - mn0), p01 = exp2f(s[1] - mn1);
      const float p10 = exp2f(s[2] - mn0), p11 = exp2f(s[3] - mn1);
      l0 = l0 * al0 + p00 + p10;
      l1 = l1 * al1 + p01 + p11;
      uint32_t h0, h1, lo0, lo1;
      split_bf2(p00, p01, h0, lo0);
      split_bf2(p10, p11, h1, lo1);
      const uint32_t bh0 = movtrans(h0), bh1 = movtrans(h1), bl0 = movtrans(lo0), bl1 = movtrans(lo1);
      uint32_t pb0, pb1;
      if (PK) {   // columns 4..7 carry P_lo of heads 0..3 (from lane - 16)
        const uint32_t x0 = __shfl_xor_sync(0xffffffffu, bl0, 16), x1 = __shfl_xor_sync(0xffffffffu, bl1, 16);
        pb0 = g < 4 ? bh0 : x0;
        pb1 = g < 4 ? bh1 : x1;
        // O^T columns 2t, 2t+1 hold heads (2t, 2t+1) mod 4: lanes t >= 2 rescale with t - 2's factors
        const float y0 = __shfl_xor_sync(0xffffffffu, al0, 2), y1 = __shfl_xor_sync(0xffffffffu, al1, 2);
        if (t >= 2) { al0 = y0; al1 = y1; }
      }
      if (al0 != 1.f || al1 != 1.f) {
#pragma unroll
        for (int i = 0; i < 8; ++i) { o[i][0] *= al0; o[i][1] *= al1; o[i][2] *= al0; o[i][3] *= al1; }
      }
      // ---- O^T += V^T . P^T; m-tile (sg, i): rows g -> dim 8(g+8sg)+2i, g+8 -> that dim + 1
#pragma unroll
      for (int sg = 0; sg < 2; ++sg)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const uint32_t v0 = w_of(vr[0][sg], i), v1 = w_of(vr[1][sg], i);
          const uint32_t v2 = w_of(vr[2][sg], i), v3 = w_of(vr[3][sg], i);
          const uint32_t a0 = __byte_perm(v0, v1, 0x5410), a1 = __byte_perm(v0, v1, 0x7632);
          const uint32_t a2 = __byte_perm(v2, v3, 0x5410), a3 = __byte_perm(v2, v3, 0x7632);
          if (PK) {
            mma16816(o[sg * 4 + i], a0, a1, a2, a3, pb0, pb1);
          } else {
            mma16816(o[sg * 4 + i], a0, a1, a2, a3, bh0, bh1);
            mma16816(o[sg * 4 + i], a0, a1, a2, a3, bl0, bl1);
          }
        }
      if (MODE == 0 && j + 1 < b1) load_v(idn);
    }
    if (MODE == 1 && sink == 0x9e3779b9u) o[0][0] += 1.f;
    // ---- finish: row sums over the 8 key lanes; PK: fold lo columns into hi
#pragma unroll
    for (int x = 4; x < 32; x <<= 1) {
      l0 += __shfl_xor_sync(0xffffffffu, l0, x);
      l1 += __shfl_xor_sync(0xffffffffu, l1, x);
    }
    if (PK) {
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int c = 0; c < 4; ++c) o[i][c] += __shfl_xor_sync(0xffffffffu, o[i][c], 2);
    }
    const int hA = 2 * t, hB = 2 * t + 1;   // this lane's heads (valid when < grp)
    const bool own = PK ? t < 2 : true;
    if (nch == 1) {
      const float i0 = 1.f / l0, i1 = 1.f / l1;
#pragma unroll
      for (int sg = 0; sg < 2; ++sg)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int d = 8 * (g + 8 * sg) + 2 * i;
          const float* c = o[sg * 4 + i];
          if (own && hA < grp)
            *reinterpret_cast<uint32_t*>(og + ((size_t)tok * a.H + hk * grp + hA) * HD + d) = pack_bf2(c[0] * i0, c[2] * i0);
          if (own && hB < grp)
            *reinterpret_cast<uint32_t*>(og + ((size_t)tok * a.H + hk * grp + hB) * HD + d) = pack_bf2(c[1] * i1, c[3] * i1);
        }
      continue;
    }
    // ---- partial record of this chunk, then the (t, head) ticket
    float* rec = a.part + (size_t)u * rec_f;
    if (own && g == 0) {
      if (hA < grp) { rec[hA] = m0; rec[8 + hA] = l0; }
      if (hB < grp) { rec[hB] = m1; rec[8 + hB] = l1; }
    }
#pragma unroll
    for (int sg = 0; sg < 2; ++sg)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int d = 8 * (g + 8 * sg) + 2 * i;
        const float* c = o[sg * 4 + i];
        if (own && hA < grp) __stcg(reinterpret_cast<float2*>(rec + 16 + hA * HD + d), make_float2(c[0], c[2]));
        if (own && hB < grp) __stcg(reinterpret_cast<float2*>(rec + 16 + hB * HD + d), make_float2(c[1], c[3]));
      }
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) {
      int* tk = a.tickets + (size_t)tok * a.Hkv + hk;
      last = atomicAdd(tk, 1) == nch - 1;
      if (last) *tk = 0;   // self-reset for the next launch
    }
    last = __shfl_sync(0xffffffffu, last, 0);
    if (!last) continue;
    __threadfence();
    // merge the nch records of (tok, hk) in chunk order: lane = 4 dims
    const float* r0 = a.part + (size_t)(u - ch * a.Hkv) * rec_f;   // chunk 0's record
    const size_t cstride = (size_t)a.Hkv * rec_f;                  // next chunk of the same (t, head)
    for (int h = 0; h < grp; ++h) {
      float M = -INFINITY;
      for (int c = 0; c < nch; ++c) M = fmaxf(M, __ldcg(r0 + c * cstride + h));
      float L = 0.f;
      float4 O = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int c = 0; c < nch; ++c) {
        const float* rc = r0 + c * cstride;
        const float f = exp2f(__ldcg(rc + h) - M);
        L += __ldcg(rc + 8 + h) * f;
        const float4 x = __ldcg(reinterpret_cast<const float4*>(rc + 16 + h * HD) + lane);
        O.x += x.x * f; O.y += x.y * f; O.z += x.z * f; O.w += x.w * f;
      }
      const float il = 1.f / L;
      uint2 w;
      w.x = pack_bf2(O.x * il, O.y * il);
      w.y = pack_bf2(O.z * il, O.w * il);
      *reinterpret_cast<uint2*>(og + ((size_t)tok * a.H + hk * grp + h) * HD + 4 * lane) = w;
    }
  }
}

int attn_decode2_rec_floats(int grp) { return dec_rec_floats(grp); }

// Warps per CTA: 16 (128 registers, small spills) or 12 (no spills);
// BULLET_DEC2_WARPS selects for experiments.
int attn_decode2_warps() {
  static const int nw = getenv("BULLET_DEC2_WARPS") && atoi(getenv("BULLET_DEC2_WARPS")) == 12 ? 12 : NW_MAX;
  return nw;
}

template <int NW, int MODE>
static void launch_nw(const AttnArgs& a, int grid, cudaStream_t st) {
  if (a.H / a.Hkv <= 4) k_attn_decode2<true, NW, MODE><<<grid, NW * 32, 0, st>>>(a);
  else k_attn_decode2<false, NW, MODE><<<grid, NW * 32, 0, st>>>(a);
}

// a.dbg (BULLET_DBG, experiments): 1 = loads only, 2 = no prefetch (loads at the top of each block)
cudaError_t launch_attn_decode2(const AttnArgs& a, int grid, cudaStream_t st) {
  const int mode = a.dbg & 3;
  if (attn_decode2_warps() == 12) {
    if (mode == 1) launch_nw<12, 1>(a, grid, st);
    else if (mode == 2) launch_nw<12, 2>(a, grid, st);
    else launch_nw<12, 0>(a, grid, st);
  } else {
    if (mode == 1) launch_nw<16, 1>(a, grid, st);
    else if (mode == 2) launch_nw<16, 2>(a, grid, st);
    else launch_nw<16, 0>(a, grid, st);
  }
  return cudaGetLastError();
}

}  // namespace bl
