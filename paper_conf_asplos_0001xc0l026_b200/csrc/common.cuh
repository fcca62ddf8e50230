// common.cuh — device helpers shared by the Bullet sm_100a kernels.
//
// SM gating (replaces libsmctrl stream masks over MPS):
// every kernel is persistent; each CTA reads %smid, returns at once when the
// SM is not in its phase's set, otherwise claims work units from an atomic
// counter until they run out.  Correctness never depends on grid size or on
// where CTAs land.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace bl {

struct Gate {
  uint32_t m[8];  // bit s set <=> smid s may do work (smid < 256)
};

// Per-launch context passed by value to every kernel.
struct Launch {
  Gate gate;
  const Gate* gdev;  // non-null: the phase's SM set lives in device memory (BULLET_DEVICE_SPLIT) —
                     // a captured graph then follows bullet_set_split at replay
  int* ctr;        // work counter, zero at launch
  int* burn;       // CTAs that left out of range (zero at launch; nullable)
  int* fallback;   // handle-wide count of launches whose last CTA worked off-range (nullable)
  int32_t* log;    // smid log (nullable): [0] = count, then {launch, unit, smid, phase}
  int log_cap;
  int launch_id;
  int phase;
  unsigned long long* trace;   // nullable (bullet_trace_enable): [grid][16] per-CTA timestamps, see trace_at
  int pdl;                     // host: launched with programmatic stream serialization (launch_ex)
};

// Programmatic dependent launch (PDL).  Step kernels are launched so that
// kernel i+1 may start once every CTA of kernel i has triggered — which a
// CTA does only when kernel i's work units are all claimed (its tail) and
// after its own pdl_wait (so kernel i-1 is complete: only neighbours
// overlap).  Kernel i+1's CTAs then take SMs as kernel i's CTAs leave them,
// run their prologue and stream the static operands (weights), and only
// then pdl_wait(), which returns once kernel i has completed and its memory
// is visible.  Anything that reads a predecessor's output, or writes memory
// a predecessor may still read, comes after pdl_wait().  Out-of-range CTAs
// park in gate_enter.  Without the launch attribute both are no-ops.
// (after pdl_wait: the caller's own predecessor is complete before dependents launch)
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.wait;\n\tgriddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Per-CTA trace record (bullet_trace_enable, diagnostics only): slot 0 smid,
// 1 entry, 2 first MMA operand stage ready, 3 MMA issue done, 4 epilogue
// done, 5 exit, 6 work units (queue entries), 7 last partial stored + fenced,
// 8 first fixup start, 9 last fixup end, 10 fixups done, 15 the epilogue's
// last accumulator ready (GEMM).  Written by one
// thread per slot.
constexpr int TRACE_SLOTS = 16;
__device__ __forceinline__ void trace_at(const Launch& L, int slot, unsigned long long v) {
  if (L.trace)
    L.trace[(size_t)(blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z)) * TRACE_SLOTS + slot] = v;
}

__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

__device__ __forceinline__ bool gate_ok(const Gate& g) {
  uint32_t s = smid();
  return s < 256 && ((g.m[s >> 5] >> (s & 31)) & 1u);
}

// Kernel entry: a CTA on one of the phase's SMs works; one elsewhere leaves
// at once — unless every other CTA of the grid already left that way (they
// all landed outside the range, e.g. on SMs another phase or rank freed for
// a moment): then this last CTA works where it is, so a launch can never end
// with its units unprocessed (correctness never depends on CTA placement).
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ bool gate_enter(const Launch& L) {
  if (L.gdev ? gate_ok(*L.gdev) : gate_ok(L.gate)) return true;
  // Launched early (PDL): park until the predecessor has completed before
  // leaving, so the grid cannot drain through SMs that are free only
  // because they are not this phase's (the next CTA of the grid would land
  // on the same SM and leave again) while this phase's SMs are still busy.
  if (L.pdl) pdl_wait();
  if (!L.burn) return false;
  int last = 0;   // (no shared memory: kernels align their dynamic smem base)
  if (threadIdx.x == 0) {
    last = atomicAdd(L.burn, 1) == (int)(gridDim.x * gridDim.y * gridDim.z) - 1;
    if (last && L.fallback) atomicAdd(L.fallback, 1);   // reported by bullet_gate_fallbacks
  }
  return __syncthreads_or(last) != 0;
}

__device__ __forceinline__ void log_unit(const Launch& L, int unit) {
  if (L.log) {
    int i = atomicAdd(L.log, 1);
    if (i < L.log_cap) {
      int32_t* e = L.log + 1 + 4 * i;
      e[0] = L.launch_id; e[1] = unit; e[2] = (int32_t)smid(); e[3] = L.phase;
    }
  }
}

// ------------------------------------------------------------ element types
template <typename T> struct Elt;
template <> struct Elt<float> {
  static __device__ __forceinline__ float to_f(float v) { return v; }
  static __device__ __forceinline__ float from_f(float v) { return v; }
};
template <> struct Elt<__nv_bfloat16> {
  static __device__ __forceinline__ float to_f(__nv_bfloat16 v) { return __bfloat162float(v); }
  static __device__ __forceinline__ __nv_bfloat16 from_f(float v) { return __float2bfloat16_rn(v); }
};

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Request of token `tok` given cu_seqlens[n_reqs+1] (binary search).
__device__ __forceinline__ int find_req(const int32_t* cu, int n_reqs, int tok) {
  int lo = 0, hi = n_reqs - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (__ldg(cu + mid) <= tok) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// ------------------------------------------------------------ PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// TMA 2D tile load global -> shared, completion on an mbarrier.
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// Bulk prefetch of `bytes` (multiple of 16) into L2: hides DRAM latency for
// streams whose shared-memory ring is too shallow to cover it.
__device__ __forceinline__ void prefetch_l2(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// cp.async 16 bytes (global -> shared), L2-only caching.
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// the warp's lowest active lane (lane 0 when the warp is converged): tcgen05
// ops issued by a converged warp under this predicate keep their operands in
// uniform registers (no per-lane waterfall loop around each MMA)
__device__ __forceinline__ bool elect_one() {
  uint32_t e;
  asm volatile("{\n\t.reg .pred p;\n\telect.sync _|p, 0xffffffff;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(e));
  return e != 0;
}
__device__ __forceinline__ void named_bar_sync(int id, int n_threads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n_threads) : "memory");
}

}  // namespace bl
