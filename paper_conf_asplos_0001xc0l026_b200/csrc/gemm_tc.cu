// gemm_tc.cu — persistent, smid-gated tcgen05 GEMM for sm_100a.
//
// C[M x N] = A[M x K] . B[N x K]^T, bf16 operands (both K-major), fp32
// accumulation in TMEM, fused epilogues (QKV store + bias, residual add,
// SiLU(gate) * up).  Serves the QKV / O-proj / gate_up / down projections of
// both phases (the paper's cuBLAS GEMMs P:L40).
//
// Structure (one CTA per SM, 256 threads):
//   warp 0 lane 0  tile scheduler (atomic claim, gated) + TMA producer
//   warp 1 lane 0  MMA issuer: tcgen05.mma.cta_group::1.kind::f16, M=128
//   warp 2         TMEM allocator (512 columns = 2 accumulator stages)
//   warps 4..7     epilogue: tcgen05.ld 32x32b -> registers -> global (whole
//                  tiles of EPI_RESID / EPI_SILU / EPI_QKV: rows transposed
//                  through a 4 x [32][33]-word smem buffer so each warp access
//                  covers whole row segments; residual loads issued ahead)
// Pipelines: smem stage ring (full/empty mbarriers, TMA complete_tx and
// tcgen05.commit), accumulator ring (2 stages), work-unit queue (4 slots).
// Operand tiles: A mh x (128 x 64), B bn x 64 (bf16, 128-byte swizzle, TMA).
// mh = 2 (decode-sized M <= 512): a unit covers 256 rows with two M=128
// accumulators that share every B stage, so weights stream through an SM
// once per 256 rows instead of once per 128.
// Work: units [0, n_full) are whole tiles; the remaining tiles (the ragged
// last wave, or all tiles of a decode-sized GEMM) are streamed over K in
// equal ranges (stream-K, see Seg below) so every SM of the partition
// streams the same number of k-blocks.  Partial segments write fp32
// partials; after its own queue every CTA runs the fixup phase (fix_phase):
// claims items of streamed tiles, sums their partials in k order
// (deterministic) and runs the epilogue.
#include "kernels.h"

namespace bl {

namespace {

constexpr int BM = 128, BK = 64, NT = 256;
constexpr uint32_t A_BYTES = BM * BK * 2;  // 16 KB per 128-row half

// Tile order: bands of `band` M tiles; inside a band the M tile varies
// fastest, then N.  A band's activations (<= ~32 MB) stay L2-resident while
// every weight tile streams past them once per band, instead of the whole
// activation block being re-read from DRAM for every N tile.
__device__ __forceinline__ void tile_coords(int tile, int m_tiles, int n_tiles, int band, int& m_blk,
                                            int& n_blk) {
  const int per_band = band * n_tiles;            // tiles in a full band
  const int b = tile / per_band, r = tile % per_band;
  const int rows = min(band, m_tiles - b * band);  // the last band may be short
  m_blk = b * band + r % rows;
  n_blk = r / rows;
}
// ---------------------------------------------------------------- work decomposition
// Units [0, n_full) are whole tiles (rasterised by tile_coords).  The other
// sk_tiles tiles (the ragged remainder, or every tile of a decode-sized
// GEMM) are streamed: their sk_tiles * k_blocks k-block iterations are cut
// into sk_chunks equal ranges ("stream-K"), unit n_full + c = range c.  A
// range covers the pieces ("segments") of the tiles it overlaps; a segment
// covering a whole tile runs the epilogue itself, the others store an fp32
// partial in slot 2c (the range's first segment) or 2c + 1 (its last) and
// the tile's last-arriving segment sums the partials in k order
// (deterministic) and runs the epilogue.  So a GEMM with fewer tiles than
// SMs still keeps every SM streaming the same number of k-blocks.
struct Seg {   // one entry of the CTA's work queue
  int tile, kb0, kb1, slot;   // slot: partial slot, -1 = whole tile (direct epilogue); tile -1 = end
};
// (the host keeps sk_chunks * sk_tiles * k_blocks < 2^31: int arithmetic)
__device__ __forceinline__ int sk_bound(const GemmArgs& a, int k_blocks, int c) {
  return c * (a.sk_tiles * k_blocks) / a.sk_chunks;
}
// chunk holding stream iteration x (the largest c with sk_bound(c) <= x)
__device__ __forceinline__ int sk_chunk_of(const GemmArgs& a, int k_blocks, int x) {
  return ((x + 1) * a.sk_chunks - 1) / (a.sk_tiles * k_blocks);
}
constexpr int SK_MAX_SEG = 16;   // segments per streamed tile (host: chunks <= 15 x stream tiles)
constexpr int N_TILE_SEMS_DEV = 2048;   // tile_sems: [0, 2048) segments stored, [2048, 4096) items done (api.cu)

__device__ __forceinline__ uint64_t sw128_desc(uint32_t addr) {
  // UMMA shared-memory descriptor, K-major, SWIZZLE_128B: start>>4 [0,14),
  // LBO (unused for swizzled K-major) = 1 [16,30), SBO = 1024 B >> 4 [32,46),
  // version 1 [46,48), layout SWIZZLE_128B = 2 [61,64).
  return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t ad, uint64_t bd, uint32_t idesc,
                                       uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
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

// Two 32-column TMEM loads in flight under one wait (the KC merge: chunk and
// running sum together)
__device__ __forceinline__ void tmem_ld32x2(uint32_t ta, uint32_t tb, float* va, float* vb) {
  uint32_t r[64];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%64];\n\t"
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%65];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]), "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]), "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]), "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]), "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]), "=r"(r[61]), "=r"(r[62]), "=r"(r[63])
      : "r"(ta), "r"(tb));
#pragma unroll
  for (int i = 0; i < 32; ++i) { va[i] = __uint_as_float(r[i]); vb[i] = __uint_as_float(r[32 + i]); }
}

// 32 fp32 columns of this warp's 32 TMEM lanes (the KC running sum); the
// caller waits (tcgen05.wait::st) before reading them back
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

// silu(z) = z / (1 + e^-z) with the MUFU exponential and reciprocal (~1e-7
// relative error, far below the bf16 rounding R5 that follows; the IEEE
// division's slow path made the SiLU epilogue of a decode gate_up tile cost
// ~6 us, scripts/trace_step.py with BULLET_GEMM_EPI_DBG=1).  e^-z = inf for
// z < -88 gives z * 0 = -0, as the exact expression does.
__device__ __forceinline__ float silu_f(float z) { return __fdividef(z, 1.0f + __expf(-z)); }

// L2 cache policies: activation tiles are re-read by every N tile (evict
// last); decode-sized GEMMs (one M tile) stream each weight tile once (evict
// first), prefill GEMMs re-read it for every M tile of the band (normal).
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// 1-D bulk copy global -> shared, completion on an mbarrier, L2 cache hint.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
// TMA 2D tile load with an L2 cache hint.
__device__ __forceinline__ void tma_load_2d_hint(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                                 uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}

// Epilogue for 32 consecutive output columns [col, col+32) of row m.
__device__ __forceinline__ void epi_store(const GemmArgs& a, int m, int col, const float* v,
                                          const float* u) {
  const size_t o = (size_t)m * a.ldo + col;
  if (a.epi == EPI_F32) {
    float4* dst = reinterpret_cast<float4*>(a.out_f32 + o);
    const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(a.bias);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      float4 w = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
      if (b) {
        w.x += __bfloat162float(b[col + 4 * i]); w.y += __bfloat162float(b[col + 4 * i + 1]);
        w.z += __bfloat162float(b[col + 4 * i + 2]); w.w += __bfloat162float(b[col + 4 * i + 3]);
      }
      dst[i] = w;
    }
  } else if (a.epi == EPI_RESID) {
    const float4* r = reinterpret_cast<const float4*>(a.resid + o);
    float4* dst = reinterpret_cast<float4*>(a.out_f32 + o);
    const bool ld = !(a.epi_dbg & 4), st = !(a.epi_dbg & 2);
    // all loads before the first store: resid may alias out, so a load after
    // a store could not be hoisted and each would pay its own L2 round trip
    float4 rr[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) rr[i] = ld ? r[i] : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      float4 w = rr[i];
      w.x += v[4 * i]; w.y += v[4 * i + 1]; w.z += v[4 * i + 2]; w.w += v[4 * i + 3];
      if (st) dst[i] = w;
    }
  } else {  // EPI_SILU: out = silu(gate) * up, bf16
    uint32_t p[16];
    const bool math = !(a.epi_dbg & 1);
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      __nv_bfloat162 h = math ? __floats2bfloat162_rn(silu_f(v[2 * i]) * u[2 * i], silu_f(v[2 * i + 1]) * u[2 * i + 1])
                              : __floats2bfloat162_rn(v[2 * i], u[2 * i + 1]);
      p[i] = *reinterpret_cast<uint32_t*>(&h);
    }
    uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(a.out_t) + o);
    if (!(a.epi_dbg & 2))
#pragma unroll
      for (int i = 0; i < 4; ++i) dst[i] = make_uint4(p[4 * i], p[4 * i + 1], p[4 * i + 2], p[4 * i + 3]);
  }
}

// EPI_QKV for 32 columns [col, col+32) of head col/128 (col % 128 in {0, 32})
// of token m: v holds those columns, w the partner columns col+64.. of the
// rotate-half pairs.  Bias, RoPE (q and k heads), bf16 rounding (R2), then
// q -> q_out, k / v -> pool slot (same arithmetic as k_rope_kv).
__device__ __forceinline__ void epi_qkv(const GemmArgs& a, int m, int col, float* v, float* w) {
  const int head = col >> 7, i0 = col & 127;
  if (a.bias) {
    const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(a.bias);
#pragma unroll
    for (int j = 0; j < 32; ++j) { v[j] += __bfloat162float(b[col + j]); w[j] += __bfloat162float(b[col + 64 + j]); }
  }
  const TokInfo ti = a.tok[m];
  __nv_bfloat16* dst;
  if (head < a.H + a.Hkv) {
    const float4* cs = reinterpret_cast<const float4*>(a.cs + (size_t)ti.x * 64 + i0);
    const bool ld = !(a.epi_dbg & 8);
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      const float4 c = ld ? cs[j] : make_float4(1.f, 0.f, 1.f, 0.f);   // (cos, sin) of frequencies i0 + 2j, i0 + 2j + 1
      const float x0 = v[2 * j], x1 = w[2 * j], y0 = v[2 * j + 1], y1 = w[2 * j + 1];
      v[2 * j] = x0 * c.x - x1 * c.y;
      w[2 * j] = x1 * c.x + x0 * c.y;
      v[2 * j + 1] = y0 * c.z - y1 * c.w;
      w[2 * j + 1] = y1 * c.z + y0 * c.w;
    }
    dst = head < a.H ? reinterpret_cast<__nv_bfloat16*>(a.q_out) + ((size_t)m * a.H + head) * 128
                     : reinterpret_cast<__nv_bfloat16*>(a.pool_k) +
                           (((size_t)(ti.y / a.kvB) * a.Hkv + (head - a.H)) * a.kvB + ti.y % a.kvB) * 128;
  } else {
    dst = reinterpret_cast<__nv_bfloat16*>(a.pool_v) +
          (((size_t)(ti.y / a.kvB) * a.Hkv + (head - a.H - a.Hkv)) * a.kvB + ti.y % a.kvB) * 128;
  }
  uint32_t p[16], q[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    __nv_bfloat162 h = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
    __nv_bfloat162 g = __floats2bfloat162_rn(w[2 * i], w[2 * i + 1]);
    p[i] = *reinterpret_cast<uint32_t*>(&h);
    q[i] = *reinterpret_cast<uint32_t*>(&g);
  }
  uint4* d0 = reinterpret_cast<uint4*>(dst + i0);
  uint4* d1 = reinterpret_cast<uint4*>(dst + 64 + i0);
  if (a.epi_dbg & 2) return;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    d0[i] = make_uint4(p[4 * i], p[4 * i + 1], p[4 * i + 2], p[4 * i + 3]);
    d1[i] = make_uint4(q[4 * i], q[4 * i + 1], q[4 * i + 2], q[4 * i + 3]);
  }
}

// EPI_QKV, coalesced: the same arithmetic as epi_qkv (bias, rotation with the
// (cos, sin) rows `cs` loaded ahead by the caller, one bf16 rounding) for
// the warp's 32 rows, then the rows' two 64-byte segments are written through
// the warp's shared-memory buffer so each store instruction covers 4 rows x
// 2 segments x 64 B instead of 32 rows x 16 B.
__device__ __forceinline__ const float4* qkv_cs_row(const GemmArgs& a, const TokInfo& ti, int i0) {
  return reinterpret_cast<const float4*>(a.cs + (size_t)ti.x * 64 + i0);
}
__device__ __forceinline__ void epi_qkv_coal(const GemmArgs& a, uint32_t* wu, int m, int col, int lane, float* v,
                                             float* w, const TokInfo& ti, const float4* csv) {
  const int head = col >> 7, i0 = col & 127;
  if (a.bias) {
    const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(a.bias);
#pragma unroll
    for (int j = 0; j < 32; ++j) { v[j] += __bfloat162float(b[col + j]); w[j] += __bfloat162float(b[col + 64 + j]); }
  }
  __nv_bfloat16* dst;
  if (head < a.H + a.Hkv) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      const float4 c = csv[j];   // (cos, sin) of frequencies i0 + 2j, i0 + 2j + 1
      const float x0 = v[2 * j], x1 = w[2 * j], y0 = v[2 * j + 1], y1 = w[2 * j + 1];
      v[2 * j] = x0 * c.x - x1 * c.y;
      w[2 * j] = x1 * c.x + x0 * c.y;
      v[2 * j + 1] = y0 * c.z - y1 * c.w;
      w[2 * j + 1] = y1 * c.z + y0 * c.w;
    }
    dst = head < a.H ? reinterpret_cast<__nv_bfloat16*>(a.q_out) + ((size_t)m * a.H + head) * 128
                     : reinterpret_cast<__nv_bfloat16*>(a.pool_k) +
                           (((size_t)(ti.y / a.kvB) * a.Hkv + (head - a.H)) * a.kvB + ti.y % a.kvB) * 128;
  } else {
    dst = reinterpret_cast<__nv_bfloat16*>(a.pool_v) +
          (((size_t)(ti.y / a.kvB) * a.Hkv + (head - a.H - a.Hkv)) * a.kvB + ti.y % a.kvB) * 128;
  }
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    __nv_bfloat162 h = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
    __nv_bfloat162 g = __floats2bfloat162_rn(w[2 * i], w[2 * i + 1]);
    wu[lane * 33 + i] = *reinterpret_cast<uint32_t*>(&h);
    wu[lane * 33 + 16 + i] = *reinterpret_cast<uint32_t*>(&g);
  }
  __syncwarp();
  const unsigned long long dp = m < a.M ? reinterpret_cast<unsigned long long>(dst + i0) : 0ull;
  const int k = lane & 7, seg = k >> 2, qd = k & 3;
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const int r = it * 4 + (lane >> 3);
    const unsigned long long d = __shfl_sync(0xffffffffu, dp, r);
    if (d && !(a.epi_dbg & 2))
      *reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(d) + seg * 64 + qd * 8) =
          make_uint4(wu[r * 33 + seg * 16 + qd * 4], wu[r * 33 + seg * 16 + qd * 4 + 1],
                     wu[r * 33 + seg * 16 + qd * 4 + 2], wu[r * 33 + seg * 16 + qd * 4 + 3]);
  }
  __syncwarp();
}

// Epilogue inputs of row m of a tile at output column col0 (w columns), pulled
// into L2 by the epilogue thread that owns the row as soon as it learns the
// unit — the mainloop then hides their DRAM latency (the decode attention
// that precedes the O-proj / QKV GEMMs streams GBs of KV past them, so the
// residual rows and the RoPE rows are usually gone from L2 by then; measured:
// 4-13 us epilogues on decode-sized GEMMs, scripts/trace_step.py).
__device__ __forceinline__ void epi_prefetch(const GemmArgs& a, int m, int col0, int w) {
  if (m >= a.M) return;
  if (a.epi == EPI_RESID) {
    prefetch_l2(a.resid + (size_t)m * a.ldo + col0, (uint32_t)w * 4);
  } else if (a.epi == EPI_QKV) {
    const TokInfo ti = a.tok[m];
    prefetch_l2(a.cs + (size_t)ti.x * 64, 64 * sizeof(float2));
  }
}

// Coalesced epilogue of one 32-column chunk for EPI_RESID / EPI_SILU: the
// warp's 32 rows (one per lane, as they come out of TMEM) are transposed
// through a 32 x 33-word shared-memory buffer so every global access of the
// warp covers whole row segments — the residual loads and fp32 stores as
// 4 rows x 128 B per instruction, the bf16 SiLU stores as 8 rows x 64 B —
// instead of 32 rows x 16 B (per-row vectors: 8x the L2 transactions,
// measured 5-11 us per decode-sized O-proj / down tile, BULLET_GEMM_EPI_DBG).
// Same arithmetic per element as epi_store (out = resid + acc; silu(g) * u
// rounded once to bf16): bit-identical.
// residual of the warp's rows [m0, m0 + 32) at columns [col, col + 32) in the
// transposed layout (lane: column quad lane & 7 of rows it * 4 + lane / 8)
__device__ __forceinline__ void epi_resid_load(const GemmArgs& a, int m0, int col, int lane, float4* rr) {
  const int cq = lane & 7;
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const int m = m0 + it * 4 + (lane >> 3);
    rr[it] = (m < a.M && !(a.epi_dbg & 4)) ? *reinterpret_cast<const float4*>(a.resid + (size_t)m * a.ldo + col + 4 * cq)
                                           : make_float4(0.f, 0.f, 0.f, 0.f);
  }
}
// rr: the chunk's residual from epi_resid_load (loaded ahead: resid may alias
// out_f32, so loads issued after a store could not be hoisted)
__device__ __forceinline__ void epi_chunk_coalesced(const GemmArgs& a, float* wb, int m0, int col, int lane,
                                                    const float* v, const float* u, const float4* rr) {
  if (a.epi == EPI_RESID) {
#pragma unroll
    for (int j = 0; j < 32; ++j) wb[lane * 33 + j] = v[j];
    __syncwarp();
    const int cq = lane & 7;
#pragma unroll
    for (int it = 0; it < 8; ++it) {
      const int r = it * 4 + (lane >> 3), m = m0 + r;
      if (m < a.M) {
        float4 w = rr[it];
        w.x += wb[r * 33 + 4 * cq]; w.y += wb[r * 33 + 4 * cq + 1];
        w.z += wb[r * 33 + 4 * cq + 2]; w.w += wb[r * 33 + 4 * cq + 3];
        if (!(a.epi_dbg & 2)) *reinterpret_cast<float4*>(a.out_f32 + (size_t)m * a.ldo + col + 4 * cq) = w;
      }
    }
  } else {   // EPI_SILU: 32 bf16 outputs per row, 16 words
    uint32_t* wu = reinterpret_cast<uint32_t*>(wb);
    const bool math = !(a.epi_dbg & 1);
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      __nv_bfloat162 h = math ? __floats2bfloat162_rn(silu_f(v[2 * i]) * u[2 * i], silu_f(v[2 * i + 1]) * u[2 * i + 1])
                              : __floats2bfloat162_rn(v[2 * i], u[2 * i + 1]);
      wu[lane * 17 + i] = *reinterpret_cast<uint32_t*>(&h);
    }
    __syncwarp();
    const int q = lane & 3;
#pragma unroll
    for (int it = 0; it < 4; ++it) {
      const int r = it * 8 + (lane >> 2), m = m0 + r;
      if (m < a.M && !(a.epi_dbg & 2))
        *reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(a.out_t) + (size_t)m * a.ldo + col + 8 * q) =
            make_uint4(wu[r * 17 + 4 * q], wu[r * 17 + 4 * q + 1], wu[r * 17 + 4 * q + 2], wu[r * 17 + 4 * q + 3]);
    }
  }
  __syncwarp();   // the buffer is reused by the next chunk
}

// ---------------------------------------------------------------- fused all-reduce (kernels.h ArArgs)
__device__ __forceinline__ void red_release_sys_add(unsigned long long* p, unsigned long long v) {
  asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Spin until *p >= target.  Bounded: after 20 s (a dead or absent peer) the
// error word is set and the wait gives up, so a broken peer set cannot hang
// the GPU; bullet_sync reports it.
__device__ __forceinline__ void wait_ge(const unsigned long long* p, unsigned long long target, int* err) {
  if (ld_acquire_sys(p) >= target) return;
  const uint64_t t0 = globaltimer_ns();
  while (ld_acquire_sys(p) < target) {
    __nanosleep(100);
    if (*reinterpret_cast<volatile int*>(err)) return;
    if (globaltimer_ns() - t0 > 20000000000ull) { atomicExch(err, 1); return; }
  }
}
// Called by the 128 epilogue threads once the tile's rows are stored: count
// the tile's columns in ready[rank][rb] of every rank for each 128-row block.
__device__ __forceinline__ void ar_signal(const GemmArgs& a, int m_blk, int mh, int et) {
  fence_sys();               // this thread's partial stores, before the counts
  named_bar_sync(1, 128);
  if (et < a.ar.n) {
    for (int hh = 0; hh < mh; ++hh) {
      const int rb = m_blk * mh + hh;
      if (rb * BM >= a.M) break;
      red_release_sys_add(a.ar.ready[et] + (size_t)a.ar.rank * a.ar.max_rb + rb, (unsigned long long)a.bn);
    }
  }
}
// The same for `cols` columns of row block rb finished by a 128-thread group
// (named barrier `bar`) of the stream-K fixup phase.
__device__ __forceinline__ void ar_signal_cols(const GemmArgs& a, int rb, int cols, int et, int bar) {
  fence_sys();
  named_bar_sync(bar, 128);
  if (et < a.ar.n && rb * BM < a.M)
    red_release_sys_add(a.ar.ready[et] + (size_t)a.ar.rank * a.ar.max_rb + rb, (unsigned long long)cols);
}
// After the CTA's GEMM units: reduce units, then wait units (kernels.h).
__device__ __forceinline__ void ar_phase(const GemmArgs& a, int* s_u) {
  const ArArgs& r = a.ar;
  const int n = r.n, M = a.M, N4 = a.N / 4, slab4 = N4 / n, c4 = r.rank * slab4;
  constexpr int CPB = BM / AR_ROWS;   // chunks per 128-row block
  const int n_chunks = (M + AR_ROWS - 1) / AR_ROWS, n_rb = (M + BM - 1) / BM;
  for (;;) {
    if (threadIdx.x == 0) *s_u = atomicAdd(r.ctr, 1);
    __syncthreads();
    const int u = *s_u;
    __syncthreads();
    if (u >= n_chunks + n_rb) break;
    if (u < n_chunks) {
      const int rb = u / CPB;
      if ((int)threadIdx.x < n)   // every rank's partial of block rb is complete
        wait_ge(r.ready[r.rank] + (size_t)threadIdx.x * r.max_rb + rb, __ldcg(r.base + rb) + (unsigned long long)a.N,
                r.err);
      __syncthreads();
      const int row0 = u * AR_ROWS, items = min(AR_ROWS, M - row0) * slab4;
      for (int i = threadIdx.x; i < items; i += NT) {
        const size_t off = (size_t)(row0 + i / slab4) * N4 + c4 + i % slab4;
        float4 p[AR_MAX_RANKS];
#pragma unroll
        for (int s = 0; s < AR_MAX_RANKS; ++s)
          if (s < n) p[s] = __ldcg(reinterpret_cast<const float4*>(r.part[s]) + off);
        float4 acc = __ldcg(reinterpret_cast<const float4*>(r.hid[r.rank]) + off);   // x
#pragma unroll
        for (int s = 0; s < AR_MAX_RANKS; ++s)   // x + partial_0 + ... in rank order
          if (s < n) { acc.x += p[s].x; acc.y += p[s].y; acc.z += p[s].z; acc.w += p[s].w; }
#pragma unroll
        for (int s = 0; s < AR_MAX_RANKS; ++s)
          if (s < n) __stcg(reinterpret_cast<float4*>(r.hid[s]) + off, acc);
      }
      fence_sys();
      __syncthreads();
      if ((int)threadIdx.x < n) red_release_sys_add(r.done[threadIdx.x] + rb, 1ull);
    } else if (threadIdx.x == 0) {   // wait unit: all n slabs of block rb are here
      const int rb = u - n_chunks, chunks = min(CPB, n_chunks - rb * CPB);
      const unsigned long long t = __ldcg(r.base + r.max_rb + rb) + (unsigned long long)n * chunks;
      wait_ge(r.done[r.rank] + rb, t, r.err);
      __stcg(r.base + r.max_rb + rb, t);
      __stcg(r.base + rb, __ldcg(r.base + rb) + (unsigned long long)a.N);
    }
  }
}

// ---------------------------------------------------------------- fused RMSNorm (kernels.h NormFuse)
// Called by the 128 epilogue threads once the tile's rows are stored.
__device__ __forceinline__ void norm_signal(const GemmArgs& a, int m_blk, int mh, int et) {
  __threadfence();
  named_bar_sync(1, 128);
  if (et == 0)
    for (int hh = 0; hh < mh; ++hh) {
      const int rb = m_blk * mh + hh;
      if (rb * BM >= a.M) break;
      asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(a.nf.rb_ctr + rb), "r"(a.bn) : "memory");
    }
}
__device__ __forceinline__ void norm_signal_cols(const GemmArgs& a, int rb, int cols, int et, int bar) {
  __threadfence();
  named_bar_sync(bar, 128);
  if (et == 0 && rb * BM < a.M)
    asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(a.nf.rb_ctr + rb), "r"(cols) : "memory");
}
__device__ __forceinline__ int ld_acquire_gpu(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// After the CTA's GEMM units (all 256 threads): R rows per claim (their
// loads in flight together), each row with the arithmetic of
// k_rmsnorm<bf16, VPT> (elementwise.cu) in the same order: bit-identical.
template <int VPT, int R>
__device__ __forceinline__ void norm_phase(const GemmArgs& a, int* s_u, float* s_red) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, d = a.N, d4 = d / 4;
  const __nv_bfloat16* g = reinterpret_cast<const __nv_bfloat16*>(a.nf.g);
  __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(a.nf.out);
  const int units = (a.M + R - 1) / R;
  for (;;) {
    if (tid == 0) {
      const int u = atomicAdd(a.nf.unit_ctr, 1);
      if (u < units) {   // the row blocks of rows [u R, u R + R) are complete
        const int r0 = u * R, r1 = min(a.M, r0 + R) - 1;
        for (int rb = r0 / BM; rb <= r1 / BM; ++rb)
          while (ld_acquire_gpu(a.nf.rb_ctr + rb) < d) __nanosleep(64);
      }
      *s_u = u;
    }
    __syncthreads();
    const int u = *s_u;
    if (u >= units) break;
    float4 v[R][VPT];
    float ss[R];
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const int r = min(u * R + j, a.M - 1);   // rows past M: recomputed, not stored
      const float4* x = reinterpret_cast<const float4*>(a.out_f32 + (size_t)r * a.ldo);
#pragma unroll
      for (int i = 0; i < VPT; ++i) {
        const int idx = tid + i * 256;
        v[j][i] = idx < d4 ? __ldcg(x + idx) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
#pragma unroll
    for (int j = 0; j < R; ++j) {
      ss[j] = 0.f;
#pragma unroll
      for (int i = 0; i < VPT; ++i)
        ss[j] += v[j][i].x * v[j][i].x + v[j][i].y * v[j][i].y + v[j][i].z * v[j][i].z + v[j][i].w * v[j][i].w;
      ss[j] = warp_sum(ss[j]);
      if (lane == 0) s_red[j * 8 + warp] = ss[j];
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const int r = u * R + j;
      if (r >= a.M) break;
      float tot = 0.f;
#pragma unroll
      for (int w = 0; w < 8; ++w) tot += s_red[j * 8 + w];
      const float inv = rsqrtf(tot / (float)d + a.nf.eps);
      __nv_bfloat16* o = out + (size_t)r * d;
#pragma unroll
      for (int i = 0; i < VPT; ++i) {
        const int idx = tid + i * 256;
        if (idx < d4) {
          const uint2 gu = *reinterpret_cast<const uint2*>(g + 4 * idx);
          const float2 g0 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&gu.x));
          const float2 g1 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&gu.y));
          __nv_bfloat162 p0 = __floats2bfloat162_rn(v[j][i].x * inv * g0.x, v[j][i].y * inv * g0.y);
          __nv_bfloat162 p1 = __floats2bfloat162_rn(v[j][i].z * inv * g1.x, v[j][i].w * inv * g1.y);
          uint2 w2;
          w2.x = *reinterpret_cast<uint32_t*>(&p0);
          w2.y = *reinterpret_cast<uint32_t*>(&p1);
          *reinterpret_cast<uint2*>(o + 4 * idx) = w2;
        }
      }
    }
    __syncthreads();   // s_u / s_red reuse
  }
}

// ---------------------------------------------------------------- stream-K fixup phase
// After its own queue, every CTA of the launch (all 256 threads, two groups
// of 128) claims fixup items — (streamed tile, 128-row half, epilogue group
// of 32 output columns; QKV / SiLU groups pair the rotate-half / gate-up
// partner columns) — waits until all segments of the item's tile have
// stored their partials, sums them in k order (deterministic) and runs the
// epilogue for those columns.  Waiting only after the CTA's own segments are
// done keeps it deadlock-free (every segment belongs to a unit some CTA runs
// to completion first), and the reduction is spread over the whole
// partition instead of one SM per tile.  The tile's last item re-zeroes its
// counters for the next launch.
template <int mh>
__device__ __forceinline__ void fix_phase(const GemmArgs& a, int* s_u, int k_blocks, int m_tiles, int n_tiles,
                                          uint8_t* ring, uint32_t ring_bytes, uint64_t* fixb) {
  const int bn = a.bn;
  const bool pair = a.epi == EPI_QKV || a.epi == EPI_SILU;
  const int G = pair ? bn / 64 : bn / 32;   // epilogue groups per 128-row half
  const int nch = pair ? 2 : 1;             // 32-column chunks per group
  const int per_tile = mh * G, items = a.sk_tiles * per_tile;
  const int tid = threadIdx.x, et = tid & 127;
  const size_t tile_f4 = (size_t)mh * BM * bn / 4;
  constexpr uint32_t CHUNK = BM * 32 * 4;   // one 32-column chunk of one segment's partial: 16 KB
  const int* sems = a.tile_sems + (a.sk_parity ? N_TILE_SEMS_DEV : 0);
  float4* buf = reinterpret_cast<float4*>(ring);
  const int t0n = a.L.trace && tid == 0;
  if (t0n) trace_at(a.L, 8, gtimer());
  int n_items = 0;
  uint32_t fph = 0;
  const uint64_t pol = policy_evict_first();
  if (tid == 0) s_u[0] = atomicAdd(a.fix_ctr, 1);
  __syncthreads();
  int u = s_u[0];
  for (;;) {
    __syncthreads();   // (s_u, ring reuse)
    if (u >= items) break;
    ++n_items;
    int u_next = 0;
    if (tid == 0) u_next = atomicAdd(a.fix_ctr, 1);   // claim ahead: its round trip overlaps this item
    const int st_idx = u / per_tile, r = u % per_tile, hh = r / G, gi = r % G;
    const int x0 = st_idx * k_blocks, x1 = x0 + k_blocks - 1;
    const int c_lo = sk_chunk_of(a, k_blocks, x0), c_hi = sk_chunk_of(a, k_blocks, x1);
    int seg_slot[SK_MAX_SEG];
    int nseg = 0;
    {
      int b0 = sk_bound(a, k_blocks, c_lo);
      for (int c = c_lo; c <= c_hi && nseg < SK_MAX_SEG; ++c) {
        const int b1 = sk_bound(a, k_blocks, c + 1);
        if (b1 > b0) seg_slot[nseg++] = b0 < x0 ? 2 * c + 1 : 2 * c;
        b0 = b1;
      }
    }
    int m_blk, n_blk;
    tile_coords(a.n_full + st_idx, m_tiles, n_tiles, a.band, m_blk, n_blk);
    const int m = (m_blk * mh + hh) * BM + et;
    const int c = a.epi == EPI_QKV ? (gi >> 1) * 128 + (gi & 1) * 32 : gi * 32;
    const int c2 = a.epi == EPI_QKV ? c + 64 : bn / 2 + c;   // pair partner chunk
    // epilogue inputs that do not depend on the partials, loaded while waiting
    float4 r4[8];
    if (tid < 128 && a.epi == EPI_RESID && m < a.M) {
      const float4* rp = reinterpret_cast<const float4*>(a.resid + (size_t)m * a.ldo + n_blk * bn + c);
#pragma unroll
      for (int i = 0; i < 8; ++i) r4[i] = rp[i];
    }
    const bool tr = t0n && n_items == 1;
    if (tr) trace_at(a.L, 11, gtimer());
    const bool bulk = (uint32_t)(nseg * nch) * CHUNK <= ring_bytes;
    if (tid < 32) {   // every segment of the tile has stored its partial
      if (tid == 0)
        while (ld_acquire_gpu(sems + st_idx) < nseg) __nanosleep(32);
      __syncwarp();
      // all (chunk, segment) blocks in one bulk-copy round, issued by one
      // elected lane of the converged warp (uniform operands, no waterfall)
      if (bulk && elect_one()) {
        mbar_arrive_expect_tx(fixb, (uint32_t)(nseg * nch) * CHUNK);
        for (int ch = 0; ch < nch; ++ch)
          for (int sg = 0; sg < nseg; ++sg)
            bulk_g2s(ring + (size_t)(ch * nseg + sg) * CHUNK,
                     reinterpret_cast<const float4*>(a.partials) + (size_t)seg_slot[sg] * tile_f4 +
                         (size_t)hh * BM * bn / 4 + (size_t)((ch ? c2 : c) / 4) * BM,
                     CHUNK, fixb, pol);
      }
      __syncwarp();
    }
    __syncthreads();
    if (tr) trace_at(a.L, 12, gtimer());
    float v[32], w[32];
    if (bulk) {
      mbar_wait(fixb, fph);
      fph ^= 1;
      // sum the segments in k order, element-wise over the chunks (256 threads),
      // into each chunk's first block
      for (int ch = 0; ch < nch; ++ch)
        for (int f = tid; f < BM * 8; f += NT) {
          float4 acc = buf[(size_t)(ch * nseg) * BM * 8 + f];
          for (int sg = 1; sg < nseg; ++sg) {
            const float4 x = buf[(size_t)(ch * nseg + sg) * BM * 8 + f];
            acc.x += x.x; acc.y += x.y; acc.z += x.z; acc.w += x.w;
          }
          buf[(size_t)(ch * nseg) * BM * 8 + f] = acc;
        }
      __syncthreads();
      if (tid < 128) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float4 x = buf[(size_t)i * BM + et];
          v[4 * i] = x.x; v[4 * i + 1] = x.y; v[4 * i + 2] = x.z; v[4 * i + 3] = x.w;
        }
        if (pair)
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const float4 x = buf[(size_t)nseg * BM * 8 + (size_t)i * BM + et];
            w[4 * i] = x.x; w[4 * i + 1] = x.y; w[4 * i + 2] = x.z; w[4 * i + 3] = x.w;
          }
      }
    } else if (tid < 128) {   // too many segments for the ring: register batches
      const float4* T0 = reinterpret_cast<const float4*>(a.partials) + (size_t)hh * BM * bn / 4 + et;
      auto sum32 = [&](int col, float* acc) {
        const size_t off = (size_t)(col / 4) * BM;
#pragma unroll
        for (int i = 0; i < 32; ++i) acc[i] = 0.f;
        for (int j = 0; j < nseg; j += 4) {
          float4 x[4][8];
#pragma unroll
          for (int q = 0; q < 4; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i)
              x[q][i] = j + q < nseg ? __ldcg(T0 + (size_t)seg_slot[j + q] * tile_f4 + off + (size_t)i * BM)
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
          for (int q = 0; q < 4; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              acc[4 * i] += x[q][i].x; acc[4 * i + 1] += x[q][i].y;
              acc[4 * i + 2] += x[q][i].z; acc[4 * i + 3] += x[q][i].w;
            }
        }
      };
      sum32(c, v);
      if (pair) sum32(c2, w);
    }
    if (tid < 128) {
      if (a.epi == EPI_QKV) {   // group gi: head gi / 2, columns c and its rotate-half partner c + 64
        if (m < a.M) epi_qkv(a, m, n_blk * bn + c, v, w);
      } else if (a.epi == EPI_SILU) {   // gate columns c, up columns bn / 2 + c -> output n_blk bn / 2 + c
        if (m < a.M) epi_store(a, m, n_blk * (bn / 2) + c, v, w);
      } else if (a.epi == EPI_RESID) {
        if (m < a.M) {
          float4* dst = reinterpret_cast<float4*>(a.out_f32 + (size_t)m * a.ldo + n_blk * bn + c);
#pragma unroll
          for (int i = 0; i < 8; ++i)
            dst[i] = make_float4(r4[i].x + v[4 * i], r4[i].y + v[4 * i + 1], r4[i].z + v[4 * i + 2],
                                 r4[i].w + v[4 * i + 3]);
        }
      } else {
        if (m < a.M) epi_store(a, m, n_blk * bn + c, v, nullptr);
      }
      if (tr) trace_at(a.L, 13, gtimer());
      if (a.ar.n) ar_signal_cols(a, m_blk * mh + hh, 32, et, 2);
      if (a.nf.out) norm_signal_cols(a, m_blk * mh + hh, 32, et, 2);
      if (tr) trace_at(a.L, 14, gtimer());
    }
    if (tid == 0) s_u[0] = u_next;
    __syncthreads();
    u = s_u[0];
  }
  if (t0n) { trace_at(a.L, 9, gtimer()); trace_at(a.L, 10, n_items); }
}

}  // namespace

int gemm_tc_stages(int bn, int mh) {
  const int st = mh * A_BYTES + bn * BK * 2;
  int s = (192 * 1024) / st;
  return s > 8 ? 8 : s;
}
size_t gemm_tc_smem_bytes(int bn, int mh) {
  const int st = mh * A_BYTES + bn * BK * 2;
  return (size_t)gemm_tc_stages(bn, mh) * st + 1024 /*align*/ + 512 /*barriers etc.*/ + 4 * 32 * 33 * 4 /*epilogue*/;
}

template <int mh, bool KC = false>
__global__ void __launch_bounds__(NT, 1)
    k_gemm_tc(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
              GemmArgs a, int n_stages) {
  if (!gate_enter(a.L)) return;  // not this phase's SM: touch nothing
  if (threadIdx.x == 0 && a.L.trace) { trace_at(a.L, 0, smid()); trace_at(a.L, 1, gtimer()); }
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  const int bn = a.bn;
  const uint32_t a_bytes = mh * A_BYTES, b_bytes = bn * BK * 2, st_bytes = a_bytes + b_bytes;
  // accumulator ring: mh * bn TMEM columns per stage, two stages when they fit
  const uint32_t acc_cols = mh * bn;
  // two-level accumulation (KC): three 128-column chunk stages and the running
  // fp32 sum in TMEM columns [384, 512) (not in registers: 128 live floats per
  // thread spilled, and with two stages the per-chunk merge paced the MMA —
  // QKV at 8k tokens was 1.68x a plain 128-wide tile)
  const int n_acc = KC ? 3 : 2 * acc_cols <= 512 ? 2 : 1;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + n_stages * st_bytes);
  const uint32_t epi_off = n_stages * st_bytes + 512;   // 4 x [32][33] words: coalesced epilogue
  uint64_t* empty = full + n_stages;
  uint64_t* accf = empty + n_stages;
  uint64_t* acce = accf + 4;
  uint64_t* tqf = acce + 4;
  uint64_t* tqe = tqf + 4;
  uint64_t* fixb = tqe + 4;   // stream-K fixup: bulk loads of partials into the (then idle) stage ring
  Seg* tile_q = reinterpret_cast<Seg*>(fixb + 2);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tile_q + 4);
  int* s_last = reinterpret_cast<int*>(tmem_slot + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m_tiles = (a.M + BM * mh - 1) / (BM * mh);
  const int n_tiles = a.N / bn;
  const int units = a.n_full + (a.sk_tiles ? a.sk_chunks : 0);
  const int k_blocks = a.K / BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < n_stages; ++s) { mbar_init(full + s, a.split_b ? 2 : 1); mbar_init(empty + s, 1); }
    for (int i = 0; i < 4; ++i) { mbar_init(accf + i, 1); mbar_init(acce + i, 4); }
    for (int i = 0; i < 4; ++i) { mbar_init(tqf + i, 1); mbar_init(tqe + i, a.split_b ? 6 : 5); }
    mbar_init(fixb, 1);
    mbar_fence_init();
  }
  if (warp == 0 && lane == 0) { tma_prefetch_desc(&mapA); tma_prefetch_desc(&mapB); }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  // B rows of tile column n_blk (SiLU tiles take bn/2 gate rows and the
  // matching bn/2 up rows)
  auto b_rows_of = [&](int n_blk, int& r0, int& r1) {
    if (a.epi == EPI_SILU) { r0 = n_blk * (bn / 2); r1 = a.silu_half + r0; }
    else { r0 = n_blk * bn; r1 = r0 + bn / 2; }
  };

  if (warp == 0) {
    {  // ---------------- scheduler + TMA producer (whole warp; one elected lane
       // issues, so the copy operands stay in uniform registers: see the MMA issuer)
      const uint64_t pol_a = policy_evict_last(), pol_b = a.b_evict_first ? policy_evict_first() : policy_evict_normal();
      int it = 0, s = 0;
      uint32_t ph = 0;
      bool waited = false;
      // publish one queue entry and stream its operands
      auto issue = [&](const Seg& g) {
        const int slot = it & 3;
        mbar_wait(tqe + slot, ((it >> 2) & 1) ^ 1);
        if (lane == 0) {
          tile_q[slot] = g;
          mbar_arrive(tqf + slot);
        }
        __syncwarp();
        ++it;
        if (g.tile < 0) return;
        int m_blk, n_blk, r0, r1;
        tile_coords(g.tile, m_tiles, n_tiles, a.band, m_blk, n_blk);
        b_rows_of(n_blk, r0, r1);
        if (!waited) {   // activations are the predecessor's output (warp 3 streams weights meanwhile)
          pdl_wait();
          waited = true;
        }
        for (int kb = g.kb0; kb < g.kb1; ++kb) {
          mbar_wait(empty + s, ph ^ 1);
          uint8_t* sa = smem + s * st_bytes;
          if (elect_one()) {
            mbar_arrive_expect_tx(full + s, a.split_b ? a_bytes : st_bytes);
#pragma unroll
            for (int hh = 0; hh < mh; ++hh)   // rows past M are zero-filled by TMA
              tma_load_2d_hint(sa + hh * A_BYTES, &mapA, full + s, kb * BK, (m_blk * mh + hh) * BM, pol_a);
            uint8_t* sb = sa + a_bytes;
            if (!a.split_b) {   // (else B comes from warp 3's issuer)
              if (a.b_packed) {
                const uint8_t* kbase = a.b_packed + (size_t)kb * (a.b_rows / 64) * 8192;
                if (r1 == r0 + bn / 2) {
                  bulk_g2s(sb, kbase + (size_t)(r0 / 64) * 8192, b_bytes, full + s, pol_b);
                } else {
                  bulk_g2s(sb, kbase + (size_t)(r0 / 64) * 8192, b_bytes / 2, full + s, pol_b);
                  bulk_g2s(sb + b_bytes / 2, kbase + (size_t)(r1 / 64) * 8192, b_bytes / 2, full + s, pol_b);
                }
              } else {
                tma_load_2d_hint(sb, &mapB, full + s, kb * BK, r0, pol_b);
                tma_load_2d_hint(sb + b_bytes / 2, &mapB, full + s, kb * BK, r1, pol_b);
              }
            }
          }
          __syncwarp();
          if (++s == n_stages) { s = 0; ph ^= 1; }
        }
      };
      for (;;) {
        // claim just in time: only once a smem stage is free to load into, so
        // early CTAs cannot hoard units while others idle (load balance)
        mbar_wait(empty + s, ph ^ 1);
        int u = 0;
        if (lane == 0) u = atomicAdd(a.L.ctr, 1);
        u = __shfl_sync(0xffffffffu, u, 0);
        if (u >= units) {   // all units claimed: the tail; the next kernel may launch
          if (lane == 0) pdl_trigger();
          issue(Seg{-1, 0, 0, -1});
          break;
        }
        if (lane == 0) log_unit(a.L, u);
        if (u < a.n_full) {
          issue(Seg{u, 0, k_blocks, -1});
        } else {
          const int c = u - a.n_full;   // stream range c: its segments in k order
          const int xb = sk_bound(a, k_blocks, c), xe = sk_bound(a, k_blocks, c + 1);
          for (int x = xb; x < xe;) {
            const int t = x / k_blocks, k0 = x - t * k_blocks, se = min(xe, (t + 1) * k_blocks);
            const int k1 = se - t * k_blocks;
            const bool whole = k0 == 0 && k1 == k_blocks;
            issue(Seg{a.n_full + t, k0, k1, whole ? -1 : (x == xb ? 2 * c : 2 * c + 1)});
            x = se;
          }
        }
        {   // zero the stream-K counters of the next launch (the other parity slice;
            // the launch that used it last has completed): unit u takes indices u mod units
          int* nxt = a.tile_sems + (a.sk_parity ? 0 : N_TILE_SEMS_DEV);
          for (int i = u + lane * units; i < N_TILE_SEMS_DEV; i += 32 * units) nxt[i] = 0;
        }
      }
    }
  } else if (warp == 3) {
    if (a.split_b) {  // ---------------- second issuer: B (weight) tiles (whole warp, elected issue)
      // one thread's issue loop (wait for a free stage, arm, issue) caps the
      // copy stream it can keep in flight; a second issuing thread for the
      // weight operand lifts the per-SM ceiling (KI2: 99 -> 123 GB/s/SM,
      // profiles/r01c_ki2_issuers.jsonl).  Same entry / k-block / stage
      // sequence as warp 0, its own arrival on each full barrier (count 2).
      // Weights are static: no dependency on the predecessor kernel.
      const uint64_t pol_b = a.b_evict_first ? policy_evict_first() : policy_evict_normal();
      int it = 0, s = 0;
      uint32_t ph = 0;
      for (;;) {
        const int slot = it & 3;
        mbar_wait(tqf + slot, (it >> 2) & 1);
        const Seg g = tile_q[slot];
        __syncwarp();
        if (lane == 0) mbar_arrive(tqe + slot);
        ++it;
        if (g.tile < 0) break;
        int m_blk, n_blk, r0, r1;
        tile_coords(g.tile, m_tiles, n_tiles, a.band, m_blk, n_blk);
        b_rows_of(n_blk, r0, r1);
        for (int kb = g.kb0; kb < g.kb1; ++kb) {
          if (a.b_pf && a.b_packed && kb + a.b_pf < g.kb1 && lane == 0) {
            // L2 prefetch b_pf k-blocks ahead of the ring (BULLET_GEMM_PF)
            const uint8_t* kp = a.b_packed + (size_t)(kb + a.b_pf) * (a.b_rows / 64) * 8192;
            if (r1 == r0 + bn / 2) {
              prefetch_l2(kp + (size_t)(r0 / 64) * 8192, b_bytes);
            } else {
              prefetch_l2(kp + (size_t)(r0 / 64) * 8192, b_bytes / 2);
              prefetch_l2(kp + (size_t)(r1 / 64) * 8192, b_bytes / 2);
            }
          }
          mbar_wait(empty + s, ph ^ 1);
          uint8_t* sb = smem + s * st_bytes + a_bytes;
          if (elect_one()) {
            mbar_arrive_expect_tx(full + s, b_bytes);
            if (a.b_packed) {
              const uint8_t* kbase = a.b_packed + (size_t)kb * (a.b_rows / 64) * 8192;
              if (r1 == r0 + bn / 2) {
                bulk_g2s(sb, kbase + (size_t)(r0 / 64) * 8192, b_bytes, full + s, pol_b);
              } else {
                bulk_g2s(sb, kbase + (size_t)(r0 / 64) * 8192, b_bytes / 2, full + s, pol_b);
                bulk_g2s(sb + b_bytes / 2, kbase + (size_t)(r1 / 64) * 8192, b_bytes / 2, full + s, pol_b);
              }
            } else {
              tma_load_2d_hint(sb, &mapB, full + s, kb * BK, r0, pol_b);
              tma_load_2d_hint(sb + b_bytes / 2, &mapB, full + s, kb * BK, r1, pol_b);
            }
          }
          __syncwarp();
          if (++s == n_stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    {  // ---------------- MMA issuer: the whole warp runs the loop (descriptors
       // warp-uniform, in uniform registers) and one elected lane issues the
       // tcgen05 ops; a lane-0 branch made the compiler wrap every MMA in a
       // per-lane waterfall loop (R2UR + ELECT + BRA.U.ANY, ~20 instructions)
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(bn >> 3) << 17) |
                             ((uint32_t)(BM >> 4) << 24);
      int it = 0, s = 0, as = 0;
      uint32_t ph = 0, aph = 0;
      bool first = true;
      for (;;) {
        const int slot = it & 3;
        mbar_wait(tqf + slot, (it >> 2) & 1);
        const Seg g = tile_q[slot];
        __syncwarp();
        if (lane == 0) mbar_arrive(tqe + slot);
        if (g.tile < 0) break;
        const int kb0 = g.kb0, kb1 = g.kb1;
        if (first && a.L.trace) {
          mbar_wait(full + s, ph);
          if (lane == 0) trace_at(a.L, 2, gtimer());
          first = false;
        }
        mbar_wait(acce + as, aph ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem + as * acc_cols;
        uint32_t d_tmem_c = d_tmem;
        int kc0 = kb0;   // first k-block of the current accumulation chunk
        // k-blocks left in the current chunk (a countdown: no integer division
        // on the MMA issuer's path)
        int kc_left = (KC && !(a.epi_dbg & 32)) ? a.kcb : 1 << 30;   // (bit 5: one chunk, diagnostics)
        for (int kb = kb0; kb < kb1; ++kb) {
          if (KC && kc_left == 0) {
            // two-level accumulation: hand the finished chunk to the epilogue
            // (it adds it to the running sum) and start the next chunk in the
            // next accumulator stage
            kc_left = a.kcb;
            if (elect_one()) tc_commit(accf + as);
            __syncwarp();
            if (++as == n_acc) { as = 0; aph ^= 1; }
            mbar_wait(acce + as, aph ^ 1);
            tc_fence_after();
            d_tmem_c = tmem + as * acc_cols;
            kc0 = kb;
          }
          if (KC) --kc_left;
          mbar_wait(full + s, ph);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(smem + s * st_bytes), b_addr = a_addr + a_bytes;
          // two descriptors per stage; the k steps / row halves only move the
          // start-address field (addr >> 4 < 2^14: no carry out of it)
          const uint64_t da = sw128_desc(a_addr), db = sw128_desc(b_addr);
          if (elect_one()) {
#pragma unroll
            for (int k = 0; k < BK / 16; ++k)
#pragma unroll
              for (int hh = 0; hh < mh; ++hh)
                tc_mma(d_tmem_c + hh * bn, da + (uint64_t)((hh * A_BYTES + k * 32) >> 4), db + (uint64_t)(k * 2),
                       idesc, (kb > kc0 || k > 0) ? 1u : 0u);
            tc_commit(empty + s);
          }
          __syncwarp();
          if (++s == n_stages) { s = 0; ph ^= 1; }
        }
        if (elect_one()) tc_commit(accf + as);
        __syncwarp();
        if (++as == n_acc) { as = 0; aph ^= 1; }
        ++it;
      }
      if (a.L.trace && lane == 0) { trace_at(a.L, 3, gtimer()); trace_at(a.L, 6, it); }
    }
  } else if (warp >= 4) {  // ---------------- epilogue (warps 4..7 = TMEM lane quadrants 0..3)
    pdl_wait();   // reads residual / bias / token table, writes outputs and partials
    const int et = threadIdx.x - 128, eq = warp & 3;
    int it = 0, as = 0;
    uint32_t aph = 0;
    float v[32], w[32];
    for (;;) {
      const int slot = it & 3;
      mbar_wait(tqf + slot, (it >> 2) & 1);
      const Seg g = tile_q[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(tqe + slot);
      if (g.tile < 0) break;
      int m_blk, n_blk;
      tile_coords(g.tile, m_tiles, n_tiles, a.band, m_blk, n_blk);
      const int col0 = (a.epi == EPI_SILU) ? n_blk * (bn / 2) : n_blk * bn;
      const int out_chunks = (a.epi == EPI_SILU) ? bn / 64 : bn / 32;
      if (a.epi_pf && (g.slot < 0 || KC))   // this unit's epilogue runs here: warm its inputs in L2
        for (int hh = 0; hh < (KC ? 1 : mh); ++hh) epi_prefetch(a, (m_blk * mh + hh) * BM + et, col0, bn);
      // coalesced residual epilogue: the first chunk's residual is loaded
      // before the accumulator wait (it does not depend on it), each next
      // chunk's while the current one is stored
      const bool coal_resid = !KC && g.slot < 0 && a.epi == EPI_RESID && a.epi_coal;
      float4 rr[8];

      // coalesced QKV epilogue: the first head's token info and (cos, sin)
      // rows are loaded before the accumulator wait
      const bool coal_qkv = !KC && g.slot < 0 && a.epi == EPI_QKV && a.epi_coal;
      TokInfo qti{0, 0};
      if (coal_qkv) qti = m_blk * mh * BM + et < a.M ? a.tok[m_blk * mh * BM + et] : TokInfo{0, 0};
      if constexpr (KC) {   // mh == 1, bn == 128, whole tiles (plan guarantees)
        // chunk sums in IEEE fp32 in chunk order: R = R + chunk, R in TMEM
        // columns [384, 512) of this warp's lane quadrant; the last chunk's
        // sums go straight to the epilogue (column pairs c / c + 64: the QKV
        // rotate-half partners, the SiLU gate / up halves)
        const int n_ch = (a.epi_dbg & 32) ? 1 : (k_blocks + a.kcb - 1) / a.kcb;
        const uint32_t t_r = tmem + ((uint32_t)(eq * 32) << 16) + 3 * acc_cols;
        const int m = m_blk * BM + et;
        for (int ch = 0; ch < n_ch; ++ch) {
          mbar_wait(accf + as, aph);
          tc_fence_after();
          const uint32_t tb = tmem + ((uint32_t)(eq * 32) << 16) + as * acc_cols;
#pragma unroll 1
          for (int c = 0; c < ((a.epi_dbg & 16) ? 0 : 4); ++c) {   // (diagnostics: bit 4 skips the merge)
            if (ch) {
              tmem_ld32x2(tb + c * 32, t_r + c * 32, v, w);
#pragma unroll
              for (int i = 0; i < 32; ++i) v[i] = w[i] + v[i];   // chunk order: fixed
            } else {
              tmem_ld32(tb + c * 32, v);
            }
            tmem_st32(t_r + c * 32, v);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          // the stage goes back to the MMA at once — also after the last
          // chunk, so the next tile's chunks run during this tile's stores
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(acce + as);
          if (++as == n_acc) { as = 0; aph ^= 1; }
        }
        tc_fence_after();
        // the tile's stores: the coalesced (shared-memory transposed) forms of
        // the whole-tile epilogues where they exist — per-row stores here made
        // the 128-wide KC tile 27 % slower than a plain one even with a single chunk
        float* wb = reinterpret_cast<float*>(smem + epi_off) + eq * (32 * 33);
        const TokInfo ti = (a.epi == EPI_QKV && a.epi_coal && m < a.M) ? a.tok[m] : TokInfo{0, 0};
#pragma unroll 1
        for (int c = 0; c < 64; c += 32) {
          tmem_ld32x2(t_r + c, t_r + c + 64, v, w);
          if (a.epi_coal && a.epi == EPI_QKV) {
            float4 csv[16];
            if (((col0 + c) >> 7) < a.H + a.Hkv) {
              const float4* cs = qkv_cs_row(a, ti, c);
#pragma unroll
              for (int j = 0; j < 16; ++j) csv[j] = cs[j];
            }
            epi_qkv_coal(a, reinterpret_cast<uint32_t*>(wb), m, col0 + c, lane, v, w, ti, csv);
          } else if (a.epi_coal && a.epi == EPI_SILU) {
            epi_chunk_coalesced(a, wb, m - lane, col0 + c, lane, v, w, nullptr);
          } else if (a.epi_coal && a.epi == EPI_RESID) {
            float4 rr[8];
            epi_resid_load(a, m - lane, col0 + c, lane, rr);
            epi_chunk_coalesced(a, wb, m - lane, col0 + c, lane, v, nullptr, rr);
            epi_resid_load(a, m - lane, col0 + c + 64, lane, rr);
            epi_chunk_coalesced(a, wb, m - lane, col0 + c + 64, lane, w, nullptr, rr);
          } else if (m < a.M) {
            if (a.epi == EPI_QKV) {
              epi_qkv(a, m, col0 + c, v, w);
            } else if (a.epi == EPI_SILU) {
              epi_store(a, m, col0 + c, v, w);
            } else {
              epi_store(a, m, col0 + c, v, nullptr);
              epi_store(a, m, col0 + c + 64, w, nullptr);
            }
          }
        }
        tc_fence_before();
        if (a.ar.n) ar_signal(a, m_blk, mh, et);
        if (a.nf.out) norm_signal(a, m_blk, mh, et);
        ++it;
        continue;
      }
      mbar_wait(accf + as, aph);
      tc_fence_after();
      if (et == 0 && a.L.trace) trace_at(a.L, 15, gtimer());   // (last) accumulator ready
      const uint32_t tb = tmem + ((uint32_t)(eq * 32) << 16) + as * acc_cols;
      if (g.slot < 0) {   // whole tile: epilogue straight from TMEM
        // one hh loop per epilogue kind: the residual carried from one 128-row
        // half to the next (rr) must not stay live through the QKV path
        // (register pressure: spills)
        if (coal_qkv) {   // per head: column chunks (c, c + 2) are rotate-half partners
          uint32_t* wu = reinterpret_cast<uint32_t*>(smem + epi_off) + eq * (32 * 33);
          for (int hh = 0; hh < mh; ++hh) {
            const int m = (m_blk * mh + hh) * BM + et;
            for (int c0 = 0; c0 < bn; c0 += 128)
              for (int c = 0; c < 64; c += 32) {
                if (hh && !c0 && !c) qti = m < a.M ? a.tok[m] : TokInfo{0, 0};
                float4 csv[16];
                if (((col0 + c0 + c) >> 7) < a.H + a.Hkv) {
                  const float4* cs = qkv_cs_row(a, qti, c);
                  const bool ld = !(a.epi_dbg & 8);
#pragma unroll
                  for (int j = 0; j < 16; ++j) csv[j] = ld ? cs[j] : make_float4(1.f, 0.f, 1.f, 0.f);
                }
                tmem_ld32(tb + hh * bn + c0 + c, v);
                tmem_ld32(tb + hh * bn + c0 + 64 + c, w);
                epi_qkv_coal(a, wu, m, col0 + c0 + c, lane, v, w, qti, csv);
              }
          }
        } else if (coal_resid) {
          epi_resid_load(a, m_blk * mh * BM + eq * 32, col0, lane, rr);
          float* wb = reinterpret_cast<float*>(smem + epi_off) + eq * (32 * 33);
          for (int hh = 0; hh < mh; ++hh) {
            const int m = (m_blk * mh + hh) * BM + et;
            for (int c = 0; c < out_chunks; ++c) {
              float4 rn[8];
              const bool more = c + 1 < out_chunks || hh + 1 < mh;
              if (more)   // next chunk (or the next 128-row half's first) in flight now
                epi_resid_load(a, (c + 1 < out_chunks ? m : m + BM) - lane, col0 + (c + 1 < out_chunks ? (c + 1) * 32 : 0),
                               lane, rn);
              tmem_ld32(tb + hh * bn + c * 32, v);
              epi_chunk_coalesced(a, wb, m - lane, col0 + c * 32, lane, v, nullptr, rr);
              if (more)
#pragma unroll
                for (int i = 0; i < 8; ++i) rr[i] = rn[i];
            }
          }
        } else if (a.epi == EPI_SILU && a.epi_coal) {
          float* wb = reinterpret_cast<float*>(smem + epi_off) + eq * (32 * 33);
          for (int hh = 0; hh < mh; ++hh) {
            const int m = (m_blk * mh + hh) * BM + et;
            for (int c = 0; c < out_chunks; ++c) {
              tmem_ld32(tb + hh * bn + c * 32, v);
              tmem_ld32(tb + hh * bn + bn / 2 + c * 32, w);
              epi_chunk_coalesced(a, wb, m - lane, col0 + c * 32, lane, v, w, nullptr);
            }
          }
        } else {
          for (int hh = 0; hh < mh; ++hh) {
            const int m = (m_blk * mh + hh) * BM + et;
            if (a.epi == EPI_QKV) {   // per head: column chunks (c, c + 2) are rotate-half partners
              for (int c0 = 0; c0 < bn; c0 += 128)
                for (int c = 0; c < 64; c += 32) {
                  tmem_ld32(tb + hh * bn + c0 + c, v);
                  tmem_ld32(tb + hh * bn + c0 + 64 + c, w);
                  if (m < a.M) epi_qkv(a, m, col0 + c0 + c, v, w);
                }
              continue;
            }
            for (int c = 0; c < out_chunks; ++c) {
              tmem_ld32(tb + hh * bn + c * 32, v);
              if (a.epi == EPI_SILU) tmem_ld32(tb + hh * bn + bn / 2 + c * 32, w);
              if (m < a.M) epi_store(a, m, col0 + c * 32, v, w);
            }
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(acce + as);
        if (a.ar.n) ar_signal(a, m_blk, mh, et);
        if (a.nf.out) norm_signal(a, m_blk, mh, et);
      } else {
        // partial tile stored as float4 groups interleaved by row per half
        // ([hh][col/4][row][4]): a thread's 4 consecutive columns are one
        // float4 and a warp's 32 rows are 512 contiguous bytes, so stores
        // and the fixup's loads are vectorised and coalesced
        const size_t tile_f4 = (size_t)mh * BM * bn / 4;
        float4* P = reinterpret_cast<float4*>(a.partials) + (size_t)g.slot * tile_f4 + et;
        for (int hh = 0; hh < mh; ++hh)
          for (int c = 0; c < bn / 32; ++c) {
            tmem_ld32(tb + hh * bn + c * 32, v);
#pragma unroll
            for (int i = 0; i < 8; ++i)
              __stcg(P + (size_t)hh * BM * bn / 4 + (size_t)(c * 8 + i) * BM,
                     make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]));
          }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(acce + as);
        // count the segment in its tile; the tile is reduced in the fixup
        // phase (fix_phase) once all its segments are stored
        __threadfence();
        named_bar_sync(1, 128);
        if (et == 0) {
          asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(a.tile_sems + (a.sk_parity ? N_TILE_SEMS_DEV : 0) +
                                                                      (g.tile - a.n_full))
                       : "memory");
          if (a.L.trace) trace_at(a.L, 7, gtimer());
        }
      }
      if (++as == n_acc) { as = 0; aph ^= 1; }
      ++it;
    }
    if (et == 0 && a.L.trace) trace_at(a.L, 4, gtimer());
  }
  pdl_wait();   // (no-op once passed) the tails below read and write predecessor-visible memory
  if (a.sk_tiles) {   // stream-K: reduce the streamed tiles (all CTAs, after their own segments)
    __syncthreads();
    fix_phase<mh>(a, s_last + 2, k_blocks, m_tiles, n_tiles, smem, (uint32_t)n_stages * st_bytes, fixb);
  }
  if (a.ar.n) {   // fused all-reduce: this CTA's GEMM units are done
    __syncthreads();
    ar_phase(a, s_last + 1);
  }
  if (a.nf.out) {   // fused RMSNorm of the rows this GEMM finished
    __syncthreads();
    float* s_red = reinterpret_cast<float*>(smem);   // the stage ring is idle now
    const int vpt = (a.N / 4 + 255) / 256;
    if (vpt <= 4) {
      if (a.nf.rows >= 4) norm_phase<4, 4>(a, s_last + 1, s_red);
      else if (a.nf.rows == 2) norm_phase<4, 2>(a, s_last + 1, s_red);
      else norm_phase<4, 1>(a, s_last + 1, s_red);
    } else {
      if (a.nf.rows >= 2) norm_phase<8, 2>(a, s_last + 1, s_red);
      else norm_phase<8, 1>(a, s_last + 1, s_red);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0 && a.L.trace) trace_at(a.L, 5, gtimer());
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
  }
}

// One thread per 16-byte chunk of the packed image (see kernels.h).
__global__ void k_pack_weight(const __nv_bfloat16* __restrict__ W, int R, int K, uint8_t* __restrict__ out) {
  const size_t n_chunks = (size_t)R * K / 8;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n_chunks; i += (size_t)gridDim.x * blockDim.x) {
    const int p = i & 7;                       // chunk position within the 128-byte row
    const size_t row_lin = i >> 3;             // (kb, rb, r) linearised
    const int r = row_lin & 63;
    const size_t tile = row_lin >> 6;          // kb * (R/64) + rb
    const int rb = tile % (R / 64);
    const int kb = tile / (R / 64);
    const int c = p ^ (r & 7);                 // logical k-chunk held at position p
    const uint4 v = *reinterpret_cast<const uint4*>(W + (size_t)(rb * 64 + r) * K + kb * 64 + c * 8);
    *reinterpret_cast<uint4*>(out + i * 16) = v;
  }
}

cudaError_t launch_pack_weight(const __nv_bfloat16* W, int R, int K, uint8_t* out, cudaStream_t st) {
  if (R % 64 || K % 64) return cudaErrorInvalidValue;
  k_pack_weight<<<1184, 256, 0, st>>>(W, R, K, out);
  return cudaGetLastError();
}

cudaError_t launch_gemm_tc(const CUtensorMap& mapA, const CUtensorMap& mapB, const GemmArgs& a,
                           int grid, cudaStream_t st) {
  const size_t smem = gemm_tc_smem_bytes(a.bn, a.mh);
  static bool attr_set = false;
  if (!attr_set) {
    size_t mx = 0;
    for (int mh = 1; mh <= 2; ++mh)
      for (int bn = 64; bn <= 256; bn *= 2) mx = std::max(mx, gemm_tc_smem_bytes(bn, mh));
    cudaError_t e = cudaFuncSetAttribute(k_gemm_tc<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)mx);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(k_gemm_tc<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)mx);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(k_gemm_tc<1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)mx);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  if (a.mh < 1 || a.mh > 2 || (a.sk_tiles && a.sk_chunks < 1)) return cudaErrorInvalidValue;
  if (a.kcb) {
    if (a.mh != 1 || a.bn != 128 || a.sk_tiles || a.n_full != (a.M + BM - 1) / BM * (a.N / 128))
      return cudaErrorInvalidValue;
    return launch_ex(k_gemm_tc<1, true>, grid, NT, smem, st, a.L.pdl, mapA, mapB, a, gemm_tc_stages(a.bn, 1));
  }
  if (a.mh == 2) return launch_ex(k_gemm_tc<2>, grid, NT, smem, st, a.L.pdl, mapA, mapB, a, gemm_tc_stages(a.bn, 2));
  return launch_ex(k_gemm_tc<1>, grid, NT, smem, st, a.L.pdl, mapA, mapB, a, gemm_tc_stages(a.bn, 1));
}

cudaError_t preload_gemm_tc() {
  cudaFuncAttributes f;
  cudaError_t e = cudaFuncGetAttributes(&f, k_gemm_tc<1>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_gemm_tc<2>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_gemm_tc<1, true>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_pack_weight);
  return e;
}

}  // namespace bl
