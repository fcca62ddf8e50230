// attn_simt.cu — paged attention on CUDA cores (the
// paper's PagedAttention decode).  One work unit = (token, kv head):
// the GQA group of query heads sharing that kv head reads every K/V byte
// once.  Keys 0..pos of the token's request are gathered block by block
// through the block table; each (block, kv head) is a contiguous
// 16 x hd chunk of the pool, staged into shared memory with 16-byte
// cp.async (double-buffered per warp), scored with fp32 FMAs, and folded
// into an online softmax (fp32, exp2).  The 4 warps of a CTA take
// interleaved blocks and merge their (max, sum, o) states at the end.
// Also serves fp32 prefill (tiny config), where every token is a unit.
#include "kernels.h"

namespace bl {

namespace {
constexpr int KB = 16;      // tokens per pool block (bullet_create enforces)
constexpr int WARPS = 4;
}

template <typename T, int HD, int HH>
__global__ void __launch_bounds__(128) k_attn_simt(AttnArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  constexpr int EPC = 16 / sizeof(T);           // elements per 16-byte chunk
  constexpr int CPR = HD / EPC;                 // chunks per key row
  constexpr int SWZ = (CPR < 16 ? CPR : 16) - 1;
  constexpr int DPL = HD / 32;                  // output dims per lane
  constexpr int GRPMAX = 2 * HH;
  constexpr int BLK_BYTES = KB * HD * sizeof(T);
  extern __shared__ __align__(16) uint8_t sm[];
  uint8_t* stage = sm;                                            // [WARPS][2][K|V]
  float* qs = reinterpret_cast<float*>(sm + WARPS * 4 * BLK_BYTES);   // [GRPMAX][HD]
  float* cmb = reinterpret_cast<float*>(sm);                       // reuses staging after the loop
  __shared__ int s_u;

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int grp = a.H / a.Hkv;
  const int units = a.n_tok * a.Hkv;
  const T* pk = reinterpret_cast<const T*>(a.pool_k);
  const T* pv = reinterpret_cast<const T*>(a.pool_v);
  const T* qg = reinterpret_cast<const T*>(a.q);
  T* og = reinterpret_cast<T*>(a.o);
  const float sl2 = a.scale * 1.4426950408889634f;
  const int j = lane & 15, hs = lane >> 4;     // token within block, head half

  for (;;) {
    if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int u = s_u;
    __syncthreads();
    if (u >= units) break;
    if (tid == 0) log_unit(a.L, u);
    const int t = u / a.Hkv, g = u % a.Hkv;
    const int r = find_req(a.cu, a.n_reqs, t);
    const int pos = __ldg(a.ctx + r) + (t - __ldg(a.cu + r));
    const int nb = pos / KB + 1;
    const int32_t* bt = a.bt + (size_t)r * a.max_blocks;
    for (int e = tid; e < grp * HD; e += 128)
      qs[e] = Elt<T>::to_f(qg[(size_t)t * a.H * HD + (size_t)g * grp * HD + e]);
    __syncthreads();

    float m[GRPMAX], l[GRPMAX], o[GRPMAX][DPL];
#pragma unroll
    for (int h = 0; h < GRPMAX; ++h) {
      m[h] = -INFINITY; l[h] = 0.f;
#pragma unroll
      for (int d = 0; d < DPL; ++d) o[h][d] = 0.f;
    }
    uint8_t* wst = stage + warp * 4 * BLK_BYTES;
    auto issue = [&](int b, int st) {
      const int blk = __ldg(bt + b);
      const uint8_t* ksrc = reinterpret_cast<const uint8_t*>(pk + ((size_t)blk * a.Hkv + g) * KB * HD);
      const uint8_t* vsrc = reinterpret_cast<const uint8_t*>(pv + ((size_t)blk * a.Hkv + g) * KB * HD);
      uint8_t* kd = wst + st * 2 * BLK_BYTES;
      uint8_t* vd = kd + BLK_BYTES;
      for (int e = lane; e < KB * CPR; e += 32) {
        const int row = e / CPR, c = e % CPR;
        cp_async16(kd + row * CPR * 16 + ((c ^ (row & SWZ)) * 16), ksrc + e * 16);
        cp_async16(vd + e * 16, vsrc + e * 16);
      }
    };
    int it = 0;
    if (warp < nb) issue(warp, 0);
    cp_async_commit();
    for (int b = warp; b < nb; b += WARPS, ++it) {
      if (b + WARPS < nb) issue(b + WARPS, (it + 1) & 1);
      cp_async_commit();
      cp_async_wait<1>();
      __syncwarp();
      const uint8_t* ks = wst + (it & 1) * 2 * BLK_BYTES;
      const T* vs = reinterpret_cast<const T*>(ks + BLK_BYTES);
      // scores: lane (j, hs) scores token j against heads hs*HH + hl
      float s[HH];
#pragma unroll
      for (int hl = 0; hl < HH; ++hl) s[hl] = 0.f;
#pragma unroll 4
      for (int c = 0; c < CPR; ++c) {
        const uint4 raw = *reinterpret_cast<const uint4*>(ks + j * CPR * 16 + ((c ^ (j & SWZ)) * 16));
        const T* kv = reinterpret_cast<const T*>(&raw);
        float kf[EPC];
#pragma unroll
        for (int e = 0; e < EPC; ++e) kf[e] = Elt<T>::to_f(kv[e]);
#pragma unroll
        for (int hl = 0; hl < HH; ++hl) {
          const int h = hs * HH + hl;
          if (h < grp) {
            const float* qh = qs + h * HD + c * EPC;
#pragma unroll
            for (int e = 0; e < EPC; ++e) s[hl] = fmaf(kf[e], qh[e], s[hl]);
          }
        }
      }
      const bool valid = (b * KB + j) <= pos;
      float mine_max[HH], p[HH];
#pragma unroll
      for (int hl = 0; hl < HH; ++hl) {
        s[hl] = valid ? s[hl] * sl2 : -INFINITY;
        float v = s[hl];
#pragma unroll
        for (int o2 = 8; o2 > 0; o2 >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o2));
        mine_max[hl] = v;
      }
      float mnew[GRPMAX], alpha[GRPMAX];
#pragma unroll
      for (int hl = 0; hl < HH; ++hl) {
        const float other = __shfl_xor_sync(0xffffffffu, mine_max[hl], 16);
        const float b0 = hs == 0 ? mine_max[hl] : other;   // head hl
        const float b1 = hs == 0 ? other : mine_max[hl];   // head HH + hl
        mnew[hl] = fmaxf(m[hl], b0);
        mnew[HH + hl] = fmaxf(m[HH + hl], b1);
      }
#pragma unroll
      for (int h = 0; h < GRPMAX; ++h) alpha[h] = exp2f(m[h] - mnew[h]);
      float psum[HH];
#pragma unroll
      for (int hl = 0; hl < HH; ++hl) {
        p[hl] = exp2f(s[hl] - mnew[hs * HH + hl]);
        float v = p[hl];
#pragma unroll
        for (int o2 = 8; o2 > 0; o2 >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o2);
        psum[hl] = v;
      }
#pragma unroll
      for (int hl = 0; hl < HH; ++hl) {
        const float other = __shfl_xor_sync(0xffffffffu, psum[hl], 16);
        const float s0 = hs == 0 ? psum[hl] : other, s1 = hs == 0 ? other : psum[hl];
        l[hl] = l[hl] * alpha[hl] + s0;
        l[HH + hl] = l[HH + hl] * alpha[HH + hl] + s1;
      }
#pragma unroll
      for (int h = 0; h < GRPMAX; ++h) {
        m[h] = mnew[h];
#pragma unroll
        for (int d = 0; d < DPL; ++d) o[h][d] *= alpha[h];
      }
      // o[h][:] += sum_j p(j, h) v_j
#pragma unroll 4
      for (int jj = 0; jj < KB; ++jj) {
        float vf[DPL];
#pragma unroll
        for (int d = 0; d < DPL; ++d) vf[d] = Elt<T>::to_f(vs[jj * HD + lane * DPL + d]);
#pragma unroll
        for (int hs2 = 0; hs2 < 2; ++hs2)
#pragma unroll
          for (int hl = 0; hl < HH; ++hl) {
            const float pj = __shfl_sync(0xffffffffu, p[hl], jj + 16 * hs2);
#pragma unroll
            for (int d = 0; d < DPL; ++d) o[hs2 * HH + hl][d] = fmaf(pj, vf[d], o[hs2 * HH + hl][d]);
          }
      }
      __syncwarp();
    }
    cp_async_wait<0>();
    __syncthreads();
    // merge the 4 warps' states: cmb[w][h] = {m, l, o[HD]}
    constexpr int REC = HD + 2;
#pragma unroll
    for (int h = 0; h < GRPMAX; ++h) {
      if (h < grp) {
        float* rec = cmb + (warp * GRPMAX + h) * REC;
        if (lane == 0) { rec[0] = m[h]; rec[1] = l[h]; }
#pragma unroll
        for (int d = 0; d < DPL; ++d) rec[2 + lane * DPL + d] = o[h][d];
      }
    }
    __syncthreads();
    for (int e = tid; e < grp * HD; e += 128) {
      const int h = e / HD, d = e % HD;
      float M = -INFINITY;
      for (int w = 0; w < WARPS; ++w) M = fmaxf(M, cmb[(w * GRPMAX + h) * REC]);
      float L = 0.f, O = 0.f;
      for (int w = 0; w < WARPS; ++w) {
        const float* rec = cmb + (w * GRPMAX + h) * REC;
        if (rec[0] == -INFINITY) continue;
        const float f = exp2f(rec[0] - M);
        L += rec[1] * f;
        O += rec[2 + d] * f;
      }
      og[(size_t)t * a.H * HD + (size_t)(g * grp + h) * HD + d] = Elt<T>::from_f(O / L);
    }
    __syncthreads();
  }
}

template <typename T, int HD, int HH>
static cudaError_t launch_one(const AttnArgs& a, int grid, cudaStream_t st) {
  constexpr int BLK_BYTES = KB * HD * sizeof(T);
  const size_t smem_stage = WARPS * 4 * BLK_BYTES + 2 * HH * HD * sizeof(float);
  const size_t smem_cmb = WARPS * 2 * HH * (HD + 2) * sizeof(float);
  const size_t smem = smem_stage > smem_cmb ? smem_stage : smem_cmb;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k_attn_simt<T, HD, HH>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    set = true;
  }
  cudaError_t e = launch_ex(k_attn_simt<T, HD, HH>, grid, 128, smem, st, a.L.pdl, a);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_attn_simt(const AttnArgs& a, int grid, cudaStream_t st) {
  const int grp = a.H / a.Hkv;
  const int hh = (grp + 1) / 2;
  if (a.hd == 128) {
    if (hh <= 1) return launch_one<T, 128, 1>(a, grid, st);
    if (hh == 2) return launch_one<T, 128, 2>(a, grid, st);
    if (hh == 3) return launch_one<T, 128, 3>(a, grid, st);
    if (hh == 4) return launch_one<T, 128, 4>(a, grid, st);
  } else if (a.hd == 64) {
    if (hh <= 1) return launch_one<T, 64, 1>(a, grid, st);
    if (hh == 2) return launch_one<T, 64, 2>(a, grid, st);
    if (hh == 3) return launch_one<T, 64, 3>(a, grid, st);
    if (hh == 4) return launch_one<T, 64, 4>(a, grid, st);
  }
  return cudaErrorInvalidValue;
}

template <typename T>
static cudaError_t preload_simt_t() {
  cudaFuncAttributes f;
  const void* k[] = {(const void*)k_attn_simt<T, 128, 1>, (const void*)k_attn_simt<T, 128, 2>,
                     (const void*)k_attn_simt<T, 128, 3>, (const void*)k_attn_simt<T, 128, 4>,
                     (const void*)k_attn_simt<T, 64, 1>, (const void*)k_attn_simt<T, 64, 2>,
                     (const void*)k_attn_simt<T, 64, 3>, (const void*)k_attn_simt<T, 64, 4>};
  for (const void* p : k) {
    cudaError_t e = cudaFuncGetAttributes(&f, p);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}
cudaError_t preload_attn_simt() {
  cudaError_t e = preload_simt_t<float>();
  return e == cudaSuccess ? preload_simt_t<__nv_bfloat16>() : e;
}

template cudaError_t launch_attn_simt<float>(const AttnArgs&, int, cudaStream_t);
template cudaError_t launch_attn_simt<__nv_bfloat16>(const AttnArgs&, int, cudaStream_t);

}  // namespace bl
