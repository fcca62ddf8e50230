// elementwise.cu — row-wise gated persistent kernels: RMSNorm (SURVEY §8a
// S1/S6), RoPE + paged KV append (S3), the SIMT GEMM used for the fp32 model
// (KI3), the per-step plan kernel and the SM probe.
#include "kernels.h"

namespace bl {

// Warp-granular work claiming: lane 0 takes a unit, the warp shares it.
__device__ __forceinline__ int warp_claim(const Launch& L) {
  int u = 0;
  if ((threadIdx.x & 31) == 0) u = atomicAdd(L.ctr, 1);
  return __shfl_sync(0xffffffffu, u, 0);
}

// 4-element vector load / store of the storage type.
__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ float4 ld4(const __nv_bfloat16* p) {
  const uint2 u = *reinterpret_cast<const uint2*>(p);
  const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&u.x));
  const float2 b = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&u.y));
  return make_float4(a.x, a.y, b.x, b.y);
}
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }
__device__ __forceinline__ void st4(__nv_bfloat16* p, float4 v) {
  __nv_bfloat162 a = __floats2bfloat162_rn(v.x, v.y), b = __floats2bfloat162_rn(v.z, v.w);
  uint2 u;
  u.x = *reinterpret_cast<uint32_t*>(&a);
  u.y = *reinterpret_cast<uint32_t*>(&b);
  *reinterpret_cast<uint2*>(p) = u;
}
__device__ __forceinline__ void st2(float* p, float a, float b) { *reinterpret_cast<float2*>(p) = make_float2(a, b); }
__device__ __forceinline__ void st2(__nv_bfloat16* p, float a, float b) {
  *reinterpret_cast<__nv_bfloat162*>(p) = __floats2bfloat162_rn(a, b);
}

// ------------------------------------------------------------------ RMSNorm
// h = x / sqrt(mean(x^2) + eps) * g, one CTA (256 threads) per row with the
// row held in registers (VPT float4 per thread), fp32 math, rounded once to
// the output type (oracle rounding point R1 / R4).
template <typename T, int VPT>
__global__ void __launch_bounds__(256) k_rmsnorm(NormArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  __shared__ int s_u;
  __shared__ float s_red[8];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const T* g = reinterpret_cast<const T*>(a.g);
  T* out = reinterpret_cast<T*>(a.out);
  const int d4 = a.d / 4;
  for (;;) {
    if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int r = s_u;
    if (r >= a.n) break;
    if (tid == 0) log_unit(a.L, r);
    const float* x = a.x + (size_t)r * a.d;
    float4 v[VPT];
    float ss = 0.f;
#pragma unroll
    for (int i = 0; i < VPT; ++i) {
      const int idx = tid + i * 256;
      v[i] = idx < d4 ? ld4(x + 4 * idx) : make_float4(0.f, 0.f, 0.f, 0.f);
      ss += v[i].x * v[i].x + v[i].y * v[i].y + v[i].z * v[i].z + v[i].w * v[i].w;
    }
    ss = warp_sum(ss);
    if (lane == 0) s_red[warp] = ss;
    __syncthreads();
    float tot = 0.f;
#pragma unroll
    for (int w = 0; w < 8; ++w) tot += s_red[w];
    const float inv = rsqrtf(tot / (float)a.d + a.eps);
    T* o = out + (size_t)r * a.d;
#pragma unroll
    for (int i = 0; i < VPT; ++i) {
      const int idx = tid + i * 256;
      if (idx < d4) {
        const float4 gg = ld4(g + 4 * idx);
        st4(o + 4 * idx, make_float4(v[i].x * inv * gg.x, v[i].y * inv * gg.y, v[i].z * inv * gg.z,
                                     v[i].w * inv * gg.w));
      }
    }
    __syncthreads();  // s_u / s_red reuse
  }
}

// Warp-per-row RMSNorm (same contract as k_rmsnorm): each warp claims a row,
// sums x^2 over the row with shuffles only (no CTA barrier), then re-reads the
// row (L1 hit) and writes x * inv * g.  Decode batches have few rows: one
// claim round per warp instead of per-row CTA barriers.
template <typename T>
__global__ void __launch_bounds__(256) k_rmsnorm_warp(NormArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  const int lane = threadIdx.x & 31;
  const T* g = reinterpret_cast<const T*>(a.g);
  T* out = reinterpret_cast<T*>(a.out);
  const int d4 = a.d / 4;
  for (;;) {
    int r = 0;
    if (lane == 0) r = atomicAdd(a.L.ctr, 1);
    r = __shfl_sync(0xffffffffu, r, 0);
    if (r >= a.n) break;
    if (lane == 0) log_unit(a.L, r);
    const float4* x = reinterpret_cast<const float4*>(a.x + (size_t)r * a.d);
    float s0 = 0.f, s1 = 0.f;
    int i = lane;
#pragma unroll 4
    for (; i + 32 < d4; i += 64) {
      const float4 u = x[i], v = x[i + 32];
      s0 += u.x * u.x + u.y * u.y + u.z * u.z + u.w * u.w;
      s1 += v.x * v.x + v.y * v.y + v.z * v.z + v.w * v.w;
    }
    if (i < d4) { const float4 u = x[i]; s0 += u.x * u.x + u.y * u.y + u.z * u.z + u.w * u.w; }
    const float inv = rsqrtf(warp_sum(s0 + s1) / (float)a.d + a.eps);
    T* o = out + (size_t)r * a.d;
#pragma unroll 4
    for (int j = lane; j < d4; j += 32) {
      const float4 u = x[j], gg = ld4(g + 4 * j);
      st4(o + 4 * j, make_float4(u.x * inv * gg.x, u.y * inv * gg.y, u.z * inv * gg.z, u.w * inv * gg.w));
    }
  }
}

// ------------------------------------------------------- RoPE + KV append
// Token t of request r at position p = ctx[r] + (t - cu[r]).  Rotate-half
// RoPE of q and k heads with the (cos, sin) table, round to the storage type
// (point R2), q -> q_out[t], k / v -> pool slot bt[r][p / B] * B + p % B.
// One CTA (256 threads) per token; each thread rotates two adjacent pairs
// (float2 loads, 2-element stores) and copies four v elements.
template <typename T>
__global__ void __launch_bounds__(256) k_rope_kv(RopeArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  __shared__ int s_u;
  const int tid = threadIdx.x;
  const int half = a.hd / 2, hp = half / 2;  // pair-of-pairs per head
  T* q_out = reinterpret_cast<T*>(a.q_out);
  T* pk = reinterpret_cast<T*>(a.pool_k);
  T* pv = reinterpret_cast<T*>(a.pool_v);
  const int nq = (a.H + 2 * a.Hkv) * a.hd;
  for (;;) {
    if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int t = s_u;
    __syncthreads();
    if (t >= a.n_tok) break;
    if (tid == 0) log_unit(a.L, t);
    const int r = find_req(a.cu, a.n_reqs, t);
    const int pos = __ldg(a.ctx + r) + (t - __ldg(a.cu + r));
    const int blk = __ldg(a.bt + (size_t)r * a.max_blocks + pos / a.B);
    const int off = pos % a.B;
    const float* src = a.qkv + (size_t)t * nq;
    const float2* cs = a.cs + (size_t)pos * half;
    for (int idx = tid; idx < (a.H + a.Hkv) * hp; idx += 256) {
      const int h = idx / hp, i = 2 * (idx % hp);
      const float2 x0 = *reinterpret_cast<const float2*>(src + h * a.hd + i);
      const float2 x1 = *reinterpret_cast<const float2*>(src + h * a.hd + i + half);
      const float4 c = *reinterpret_cast<const float4*>(cs + i);   // (cos_i, sin_i, cos_i+1, sin_i+1)
      T* dst = h < a.H ? q_out + (size_t)t * a.H * a.hd + h * a.hd
                       : pk + (((size_t)blk * a.Hkv + (h - a.H)) * a.B + off) * a.hd;
      st2(dst + i, x0.x * c.x - x1.x * c.y, x0.y * c.z - x1.y * c.w);
      st2(dst + i + half, x1.x * c.x + x0.x * c.y, x1.y * c.z + x0.y * c.w);
    }
    const float* vs = src + (a.H + a.Hkv) * a.hd;
    for (int idx = tid; idx < a.Hkv * a.hd / 4; idx += 256) {
      const int g = (4 * idx) / a.hd, e = (4 * idx) % a.hd;
      st4(pv + (((size_t)blk * a.Hkv + g) * a.B + off) * a.hd + e, ld4(vs + 4 * idx));
    }
  }
}

// ------------------------------------------------------------ SIMT GEMM
// Same contract and epilogues as the tcgen05 GEMM; used for the fp32 model
// (tiny config, KI3).  64 x 64 output tiles, 4 x 4 per thread, fp32 FMA.
template <typename T>
__global__ void __launch_bounds__(256) k_gemm_simt(const T* __restrict__ A, const T* __restrict__ B,
                                                   GemmArgs a) {
  if (!gate_enter(a.L)) return;
  pdl_wait();      // inputs are the predecessor's outputs (common.cuh, PDL)
  __shared__ float As[16][68], Bs[16][68], Us[16][68];
  __shared__ int s_u;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int NO = (a.epi == EPI_SILU) ? a.N / 2 : a.N;
  const int mt = (a.M + 63) / 64, nt = (NO + 63) / 64, units = mt * nt;
  for (;;) {
    if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
    __syncthreads();
    const int u = s_u;
    __syncthreads();
    if (u >= units) break;
    if (tid == 0) log_unit(a.L, u);
    const int m0 = (u % mt) * 64, n0 = (u / mt) * 64;
    float acc[4][4] = {}, acu[4][4] = {};
    for (int k0 = 0; k0 < a.K; k0 += 16) {
      for (int e = tid; e < 64 * 16; e += 256) {
        const int rr = e / 16, kk = e % 16;
        const int m = m0 + rr, n = n0 + rr;
        As[kk][rr] = (m < a.M) ? Elt<T>::to_f(A[(size_t)m * a.K + k0 + kk]) : 0.f;
        Bs[kk][rr] = (n < NO) ? Elt<T>::to_f(B[(size_t)n * a.K + k0 + kk]) : 0.f;
        if (a.epi == EPI_SILU)
          Us[kk][rr] = (n < NO) ? Elt<T>::to_f(B[(size_t)(a.silu_half + n) * a.K + k0 + kk]) : 0.f;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < 16; ++kk) {
        float av[4], bv[4], uv[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) { av[i] = As[kk][ty * 4 + i]; bv[i] = Bs[kk][tx * 4 + i]; uv[i] = Us[kk][tx * 4 + i]; }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
            if (a.epi == EPI_SILU) acu[i][j] = fmaf(av[i], uv[j], acu[i][j]);
          }
      }
      __syncthreads();
    }
    for (int i = 0; i < 4; ++i) {
      const int m = m0 + ty * 4 + i;
      if (m >= a.M) continue;
      for (int j = 0; j < 4; ++j) {
        const int n = n0 + tx * 4 + j;
        if (n >= NO) continue;
        const size_t o = (size_t)m * a.ldo + n;
        if (a.epi == EPI_F32) {
          float b = a.bias ? Elt<T>::to_f(reinterpret_cast<const T*>(a.bias)[n]) : 0.f;
          a.out_f32[o] = acc[i][j] + b;
        } else if (a.epi == EPI_RESID) {
          a.out_f32[o] = a.resid[o] + acc[i][j];
        } else {
          const float z = acc[i][j];
          reinterpret_cast<T*>(a.out_t)[o] = Elt<T>::from_f(z / (1.0f + expf(-z)) * acu[i][j]);
        }
      }
    }
  }
}

// ------------------------------------------------------------------ plan
// CTA 0, thread 0: zero the phase's work counters and list the prefill
// attention tiles (request, q-tile) longest-key-range first (LPT order).
// Every thread (grid-stride over tokens): the token's position and KV slot
// (request by binary search over cu), consumed by the fused QKV epilogue.
__global__ void k_plan(PlanArgs a) {
  if (blockIdx.x == 0) {
    for (int i = threadIdx.x; i < a.n_counters; i += blockDim.x) a.counters[i] = 0;
    for (int i = threadIdx.x; i < a.n_zero2; i += blockDim.x) a.zero2[i] = 0;
    if (a.order) {   // counting sort of the decode rows by block count, descending (LPT)
      __shared__ int hist[DEC_ORDER_BUCKETS + 1];
      const int n = a.n_tok - a.order_base;
      auto nb_of = [&](int i) {
        const int t = a.order_base + i;
        const int r = find_req(a.cu, a.n_reqs, t);
        const int nb = (__ldg(a.ctx + r) + (t - __ldg(a.cu + r))) / a.B + 1;
        return nb < DEC_ORDER_BUCKETS ? nb : DEC_ORDER_BUCKETS;
      };
      for (int i = threadIdx.x; i <= DEC_ORDER_BUCKETS; i += blockDim.x) hist[i] = 0;
      __syncthreads();
      for (int i = threadIdx.x; i < n; i += blockDim.x) atomicAdd(hist + nb_of(i), 1);
      __syncthreads();
      if (threadIdx.x == 0) {   // bucket starts, longest first
        int run = 0;
        for (int b = DEC_ORDER_BUCKETS; b >= 0; --b) { const int c = hist[b]; hist[b] = run; run += c; }
      }
      __syncthreads();
      for (int i = threadIdx.x; i < n; i += blockDim.x) {
        const int t = a.order_base + i;
        const int r = find_req(a.cu, a.n_reqs, t);
        const int pos = __ldg(a.ctx + r) + (t - __ldg(a.cu + r));
        a.order[atomicAdd(hist + nb_of(i), 1)] = make_int4(i, r, pos, 0);
      }
    }
    if (threadIdx.x == 0 && a.tiles) {
      int maxt = 0;
      for (int r = 0; r < a.n_tile_reqs; ++r) {
        int len = a.cu[r + 1] - a.cu[r];
        int nt = (len + a.bq - 1) / a.bq;
        maxt = nt > maxt ? nt : maxt;
      }
      int n = 0;
      for (int t = maxt - 1; t >= 0; --t)
        for (int r = 0; r < a.n_tile_reqs; ++r) {
          int len = a.cu[r + 1] - a.cu[r];
          if (t * a.bq < len) a.tiles[n++] = make_int2(r, t);
        }
      *a.n_tiles = n;
    }
  }
  if (a.tok) {
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < a.n_tok; t += gridDim.x * blockDim.x) {
      const int r = find_req(a.cu, a.n_reqs, t);
      const int pos = __ldg(a.ctx + r) + (t - __ldg(a.cu + r));
      const int blk = __ldg(a.bt + (size_t)r * a.max_blocks + pos / a.B);
      a.tok[t] = make_int2(pos, blk * a.B + pos % a.B);
    }
  }
}

// SM probe (KI1): every CTA records its %smid; CTAs spin ~50 us so the
// first wave spreads over every SM before any CTA retires.
__global__ void k_probe(int* out, int n) {
  const long long t0 = clock64();
  while (clock64() - t0 < 100000) {
  }
  if (threadIdx.x == 0 && blockIdx.x < n) out[blockIdx.x] = (int)smid();
}

// ------------------------------------------------------------- launchers
template <typename T>
cudaError_t launch_gemm_simt(const T* A, const T* B, const GemmArgs& a, int grid, cudaStream_t st) {
  cudaError_t e = launch_ex(k_gemm_simt<T>, grid, 256, 0, st, a.L.pdl, A, B, a);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}
template <typename T>
cudaError_t launch_rmsnorm_warp(const NormArgs& a, int grid, cudaStream_t st) {
  if (a.d % 4) return cudaErrorInvalidValue;
  cudaError_t e = launch_ex(k_rmsnorm_warp<T>, grid, 256, 0, st, a.L.pdl, a);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}
template <typename T>
cudaError_t launch_rmsnorm(const NormArgs& a, int grid, cudaStream_t st) {
  const int v = (a.d / 4 + 255) / 256;
  if (v <= 1) return launch_ex(k_rmsnorm<T, 1>, grid, 256, 0, st, a.L.pdl, a);
  else if (v <= 2) return launch_ex(k_rmsnorm<T, 2>, grid, 256, 0, st, a.L.pdl, a);
  else if (v <= 4) return launch_ex(k_rmsnorm<T, 4>, grid, 256, 0, st, a.L.pdl, a);
  else if (v <= 8) return launch_ex(k_rmsnorm<T, 8>, grid, 256, 0, st, a.L.pdl, a);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}
template <typename T>
cudaError_t launch_rope_kv(const RopeArgs& a, int grid, cudaStream_t st) {
  cudaError_t e = launch_ex(k_rope_kv<T>, grid, 256, 0, st, a.L.pdl, a);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}
cudaError_t launch_plan(const PlanArgs& a, cudaStream_t st) {
  int grid = a.tok ? (a.n_tok + 255) / 256 : 1;
  grid = grid < 1 ? 1 : grid > 64 ? 64 : grid;
  k_plan<<<grid, 256, 0, st>>>(a);
  return cudaGetLastError();
}
// BULLET_DEVICE_SPLIT: write both phases' SM sets (one warp, stream-ordered).
__global__ void k_set_gates(Gate* d, Gate pre, Gate dec) {
  if (threadIdx.x < 8) { d[0].m[threadIdx.x] = pre.m[threadIdx.x]; d[1].m[threadIdx.x] = dec.m[threadIdx.x]; }
}
cudaError_t launch_set_gates(Gate* d_gates, const Gate& pre, const Gate& dec, cudaStream_t st) {
  k_set_gates<<<1, 32, 0, st>>>(d_gates, pre, dec);
  return cudaGetLastError();
}

// Die probe (KI1b): the B200 is two dies, each with half of the L2; an L2
// hit on the SM's own die is ~10 % faster than one on the other die
// (B300_MICROARCH: 234 vs 262 cycles).  Every CTA spins (so the first wave
// spreads over all SMs), touches the n lines once, then times a dependent
// ld.global.cg to each line (min of 8) and records the cycles under its smid.
__global__ void k_die_probe(const uint4* lines, int n_lines, int stride4, uint32_t* lat) {
  const long long t0 = clock64();
  while (clock64() - t0 < 100000) {
  }
  if (threadIdx.x != 0) return;
  const uint32_t s = smid();
  if (s >= 256) return;
  // the lines hold zeros: acc stays 0 at run time, but every address depends
  // on the previous load's value (no overlap), and each clock read follows
  // the add that consumes the load (volatile asm keeps the order)
  uint32_t acc = 0;
  for (int j = 0; j < n_lines; ++j) acc += __ldcg(lines + (size_t)j * stride4).x;
  for (int j = 0; j < n_lines; ++j) {
    uint32_t best = 0xffffffffu;
    for (int r = 0; r < 8; ++r) {
      const uint4* p = lines + (size_t)j * stride4 + acc;
      long long c0, c1;
      asm volatile("mov.u64 %0, %%clock64;" : "=l"(c0) :: "memory");
      const uint4 v = __ldcg(p);
      asm volatile("add.u32 %0, %0, %1;" : "+r"(acc) : "r"(v.x) : "memory");
      asm volatile("mov.u64 %0, %%clock64;" : "=l"(c1) :: "memory");
      best = min(best, (uint32_t)(c1 - c0));
    }
    lat[s * n_lines + j] = best;
  }
  if (acc == 0x12345678u) lat[0] = 0;
}
cudaError_t launch_die_probe(const void* lines, int n_lines, int stride_bytes, uint32_t* lat, int grid, cudaStream_t st) {
  k_die_probe<<<grid, 32, 0, st>>>(reinterpret_cast<const uint4*>(lines), n_lines, stride_bytes / 16, lat);
  return cudaGetLastError();
}
cudaError_t launch_probe(int* out, int n, cudaStream_t st) {
  k_probe<<<n, 32, 0, st>>>(out, n);
  return cudaGetLastError();
}

template <typename T>
static cudaError_t preload_elt_t() {
  cudaFuncAttributes f;
  const void* k[] = {(const void*)k_gemm_simt<T>, (const void*)k_rmsnorm_warp<T>, (const void*)k_rope_kv<T>,
                     (const void*)k_rmsnorm<T, 1>, (const void*)k_rmsnorm<T, 2>, (const void*)k_rmsnorm<T, 4>,
                     (const void*)k_rmsnorm<T, 8>};
  for (const void* p : k) {
    cudaError_t e = cudaFuncGetAttributes(&f, p);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}
cudaError_t preload_elementwise() {
  cudaFuncAttributes f;
  cudaError_t e = cudaFuncGetAttributes(&f, k_plan);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_set_gates);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_probe);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&f, k_die_probe);
  if (e == cudaSuccess) e = preload_elt_t<float>();
  if (e == cudaSuccess) e = preload_elt_t<__nv_bfloat16>();
  return e;
}

template cudaError_t launch_gemm_simt<float>(const float*, const float*, const GemmArgs&, int, cudaStream_t);
template cudaError_t launch_gemm_simt<__nv_bfloat16>(const __nv_bfloat16*, const __nv_bfloat16*, const GemmArgs&, int, cudaStream_t);
template cudaError_t launch_rmsnorm<float>(const NormArgs&, int, cudaStream_t);
template cudaError_t launch_rmsnorm_warp<float>(const NormArgs&, int, cudaStream_t);
template cudaError_t launch_rmsnorm_warp<__nv_bfloat16>(const NormArgs&, int, cudaStream_t);
template cudaError_t launch_rmsnorm<__nv_bfloat16>(const NormArgs&, int, cudaStream_t);
template cudaError_t launch_rope_kv<float>(const RopeArgs&, int, cudaStream_t);
template cudaError_t launch_rope_kv<__nv_bfloat16>(const RopeArgs&, int, cudaStream_t);

}  // namespace bl
