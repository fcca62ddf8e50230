// stream_bench.cu — KI2 microbenchmark: HBM read bandwidth reachable from m
// SMs (the B200 analog of the paper's Fig. 7 partial-SM scaling, P:L139-145,
// and the m_sat input of SURVEY §8d).  Gated persistent kernels stream a
// buffer and fold it into a checksum (so no load is dead):
//   mode 0  LDG.128: warps claim 8 KB units, 16 loads in flight per lane
//           (16 warps -> 128 KB in flight per SM)
//   mode 1  cp.async.bulk: one thread streams 32 KB bulk copies through a
//           6 x 32 KB smem ring (192 KB in flight per SM)
//   mode 2  cp.async 16 B (LDGSTS): 64 KB units, 3 in flight per CTA
#include "kernels.h"

namespace bl {

namespace {
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
constexpr int BULK = 32768, NB = 6;
constexpr int NB_MC = 7;   // k_stream_mc ring (7 x 32 KB)
}  // namespace

__global__ void __launch_bounds__(512, 1) k_stream(StreamArgs a) {
  if (!gate_enter(a.L)) return;
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ int s_u;
  __shared__ uint64_t bars[NB];
  const int tid = threadIdx.x, lane = tid & 31;
  uint32_t acc = 0;
  if (a.mode == 0) {
    const size_t units = a.bytes / 8192;
    if (a.param > 0 && tid >= a.param * 32) return;   // only `param` warps stream
    for (;;) {
      int u = 0;
      if (lane == 0) u = atomicAdd(a.L.ctr, 1);
      u = __shfl_sync(0xffffffffu, u, 0);
      if (u >= (int)units) break;
      const uint4* p = reinterpret_cast<const uint4*>(a.src + (((size_t)u * 8192) & a.wrap)) + lane;
      uint4 v[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) v[i] = __ldcs(p + 32 * i);
#pragma unroll
      for (int i = 0; i < 16; ++i) acc ^= v[i].x ^ v[i].y ^ v[i].z ^ v[i].w;
    }
  } else if ((a.mode == 3 || a.mode == 4) || (a.mode == 5 && tid >= 32)) {
    // mode 3: LDG.128 -> registers -> STS.128 into a per-warp smem slot (a
    // register-staged producer); mode 4: same loads, no STS.  Warps claim
    // 32 KB (4 x 8 KB) per atomic; `param` = 8 KB loads in flight per warp (1|2).
    const size_t units = a.bytes / 32768;
    const int warp = tid >> 5;
    uint4* slot = reinterpret_cast<uint4*>(sm) + (size_t)warp * 512;   // 8 KB per warp
    for (;;) {
      int u = 0;
      if (lane == 0) u = atomicAdd(a.L.ctr, 1);
      u = __shfl_sync(0xffffffffu, u, 0);
      if (u >= (int)units) break;
      const uint4* p = reinterpret_cast<const uint4*>(a.src + (((size_t)u * 32768) & a.wrap)) + lane;
      if (a.param == 2) {
#pragma unroll 1
        for (int h = 0; h < 4; h += 2) {
          uint4 v[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __ldcs(p + (h * 16 + i) * 32);
          if (a.mode == 3) {
#pragma unroll
            for (int i = 0; i < 32; ++i) slot[(i & 15) * 32 + lane] = v[i];
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i) acc ^= v[i].x ^ v[i].w;
          }
        }
      } else {
#pragma unroll 1
        for (int h = 0; h < 4; ++h) {
          uint4 v[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = __ldcs(p + (h * 16 + i) * 32);
          if (a.mode == 3) {
#pragma unroll
            for (int i = 0; i < 16; ++i) slot[i * 32 + lane] = v[i];
          } else {
#pragma unroll
            for (int i = 0; i < 16; ++i) acc ^= v[i].x ^ v[i].w;
          }
        }
      }
      __syncwarp();
      if (a.mode == 3) acc ^= reinterpret_cast<const uint32_t*>(slot)[lane];
    }
  } else if (a.mode == 1 || a.mode == 5 || a.mode == 7 || a.mode == 8) {
    // mode 5 (warp 0 only here): bulk copies concurrently with LDG warps 1..15
    // mode 7: two issuing threads (tid 0, tid 32) in ONE CTA, 3 stages each
    const size_t units = a.bytes / BULK;
    const int nb = a.mode == 7 ? NB / 2 : (a.mode == 1 && a.param > 0 && a.param < NB) ? a.param : NB;
    const int iss = (tid == 0) ? 0 : (a.mode == 7 && tid == 32) ? 1 : -1;
    if (tid == 0) {
      for (int i = 0; i < NB; ++i) mbar_init(bars + i, 1);
      mbar_fence_init();
    }
    if (a.mode != 5) __syncthreads(); else __syncwarp();
    uint64_t* bars_i = bars + (iss > 0 ? iss * nb : 0);
    uint8_t* sm_i = sm + (size_t)(iss > 0 ? iss * nb : 0) * BULK;
#define bars bars_i
#define sm sm_i
    if (iss >= 0) {
      uint32_t issued = 0, done = 0;
      int batch_u = 0, batch_left = 0;
      for (;;) {
        if (issued - done == (uint32_t)nb) {   // retire the oldest
          mbar_wait(bars + (done % nb), (done / nb) & 1);
          acc ^= *reinterpret_cast<const uint32_t*>(sm + (done % nb) * BULK);
          ++done;
        }
        // claim granularity: param2 = units per atomic (mode 1 | (depth << 8) | (batch << 16) would
        // collide with the wrap field, so mode 8 = mode 1 with 8-unit claims)
        int u;
        if (a.mode == 8) {
          if (batch_left == 0) { batch_u = atomicAdd(a.L.ctr, 8); batch_left = 8; }
          u = batch_u++; --batch_left;
        } else {
          u = atomicAdd(a.L.ctr, 1);
        }
        if (u >= (int)units) break;
        const int s = issued % nb;
        mbar_arrive_expect_tx(bars + s, BULK);
        bulk_g2s(sm + s * BULK, a.src + (((size_t)u * BULK) & a.wrap), BULK, bars + s);
        ++issued;
      }
      while (done < issued) {
        mbar_wait(bars + (done % nb), (done / nb) & 1);
        acc ^= *reinterpret_cast<const uint32_t*>(sm + (done % nb) * BULK);
        ++done;
      }
    }
#undef bars
#undef sm
  } else {
    const size_t units = a.bytes / 65536;
    int n = 0;
    for (;;) {
      if (tid == 0) s_u = atomicAdd(a.L.ctr, 1);
      __syncthreads();
      const int u = s_u;
      __syncthreads();
      if (u >= (int)units) break;
      const uint8_t* p = a.src + (((size_t)u * 65536) & a.wrap);
      uint8_t* d = sm + (n % 3) * 65536;
#pragma unroll
      for (int i = 0; i < 8; ++i) cp_async16(d + (tid + i * 512) * 16, p + (tid + i * 512) * 16);
      cp_async_commit();
      ++n;
      if (a.param == 2) {            // 2 units (128 KB) in flight
        if (n >= 2) {
          cp_async_wait<1>();
          acc ^= *reinterpret_cast<const uint32_t*>(sm + (n % 3) * 65536 + tid * 16);
        }
      } else if (n >= 3) {           // 3 units (192 KB) in flight
        cp_async_wait<2>();
        acc ^= *reinterpret_cast<const uint32_t*>(sm + (n % 3) * 65536 + tid * 16);
      }
    }
    cp_async_wait<0>();
  }
  if (acc == 0x12345678u) a.sink[0] = acc;   // keeps the loads alive
}

cudaError_t launch_stream(const StreamArgs& a, int grid, cudaStream_t st) {
  // mode 1 with param = ring depth d < NB: d x 32 KB per CTA and two CTAs per
  // SM (two bulk-copy issuers per SM: is the ~85 GB/s/SM ceiling per issuer?)
  const bool two = a.mode == 1 && a.param > 0 && a.param < NB;
  const int smem = (a.mode == 1 || a.mode == 7 || a.mode == 8) ? (two ? a.param : NB) * BULK
                               : (a.mode == 2 ? 3 * 65536 : (a.mode == 3 ? 16 * 8192 : (a.mode == 5 ? NB * BULK : 0)));
  cudaError_t e = cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, NB * BULK);
  if (e != cudaSuccess) return e;
  k_stream<<<two ? 2 * grid : grid, two ? 256 : 512, smem, st>>>(a);
  return cudaGetLastError();
}

// KI3: does TMA multicast lift the per-SM async-copy ceiling?  Clusters of
// two CTAs stream 32 KB stages; mc = 1: each CTA bulk-copies its 16 KB half
// with .multicast::cluster into both CTAs' stage (each SM requests half of
// what it receives); mc = 0: each CTA copies all 32 KB itself.  Same bytes
// delivered into every SM either way; units are assigned statically by
// cluster (no gating: a standalone microbenchmark, not a hot-path kernel).
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa_u32(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1)
    k_stream_mc(const uint8_t* src, size_t bytes, int mc, uint32_t* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ uint64_t full[NB_MC], empty[NB_MC];
  const uint32_t cr = cluster_rank();
  const int n_cl = gridDim.x / 2, cl = blockIdx.x / 2;
  const size_t units = bytes / BULK;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NB_MC; ++i) { mbar_init(full + i, 1); mbar_init(empty + i, 2); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  cluster_sync_all();
  uint32_t acc = 0;
  if (threadIdx.x == 0) {
    const int n_it = units > (size_t)cl ? (int)((units - cl + n_cl - 1) / n_cl) : 0;
    constexpr int LAG = NB_MC - 3;   // stages in flight; a stage is released 3 issues before its reuse
    for (int it = 0; it < n_it + LAG; ++it) {
      if (it < n_it) {   // issue stage `it`
        const int s = it % NB_MC;
        if (it >= NB_MC) mbar_wait(empty + s, ((it / NB_MC) & 1) ^ 1);   // both CTAs released it
        mbar_arrive_expect_tx(full + s, BULK);
        const uint8_t* g = src + ((size_t)cl + (size_t)it * n_cl) * BULK;
        if (mc) {
          const uint32_t half = BULK / 2;
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;" ::"r"(
                  smem_u32(sm + s * BULK + cr * half)),
              "l"(g + cr * half), "r"(half), "r"(smem_u32(full + s)), "h"((uint16_t)3)
              : "memory");
        } else {
          bulk_g2s(sm + s * BULK, g, BULK, full + s);
        }
      }
      const int j = it - LAG;
      if (j >= 0) {      // consume stage j, release it in both CTAs
        const int s = j % NB_MC;
        mbar_wait(full + s, (j / NB_MC) & 1);
        acc ^= *reinterpret_cast<const uint32_t*>(sm + s * BULK + (j & 1023) * 16);
        const uint32_t b = smem_u32(empty + s);
        for (uint32_t r = 0; r < 2; ++r)
          asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(mapa_u32(b, r)) : "memory");
      }
    }
  }
  cluster_sync_all();   // no multicast / arrive may target an exited CTA
  if (acc == 0x12345678u) sink[0] = acc;
}

cudaError_t launch_stream_mc(const uint8_t* src, size_t bytes, int mc, int grid, uint32_t* sink, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_stream_mc, cudaFuncAttributeMaxDynamicSharedMemorySize, NB_MC * BULK);
  if (e != cudaSuccess) return e;
  k_stream_mc<<<grid & ~1, 128, NB_MC * BULK, st>>>(src, bytes, mc, sink);
  return cudaGetLastError();
}

cudaError_t preload_stream() {
  cudaFuncAttributes f;
  return cudaFuncGetAttributes(&f, k_stream);
}

}  // namespace bl
