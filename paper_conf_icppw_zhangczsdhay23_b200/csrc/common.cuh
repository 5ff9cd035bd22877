// common.cuh -- small device helpers shared by the sm_100a kernels of libsssp.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#define SSSP_FULL_MASK 0xFFFFFFFFu

namespace sssp {

typedef unsigned long long u64;
typedef uint32_t u32;
typedef int64_t i64;

// ---- loads / stores with explicit cache behaviour --------------------------
// Arcs are streamed (read ~once per SSSP): evict-first in L1/L2.
__device__ __forceinline__ uint2 ld_stream_u2(const uint2* p) {
  uint2 v;
  u64 pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;"
      : "=r"(v.x), "=r"(v.y)
      : "l"(p), "l"(pol));
  return v;
}
// Coherent (L2) load of mutable data (dist[], queue words).
__device__ __forceinline__ u32 ld_cg(const u32* p) { return __ldcg(p); }
__device__ __forceinline__ u64 ld_relaxed_u64(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u32 ld_relaxed_u32(const u32* p) {
  u32 v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u32 ld_acquire_u32(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(u32* p, u32 v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ u32 atom_add_acq_rel_u32(u32* p, u32 v) {
  u32 old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}

// Grid barrier arrival/departure for a cooperative (co-resident) grid, called by
// one thread per CTA after a __syncthreads (whose CTA-scope ordering the release
// extends to the GPU). `count` is a monotonic ticket counter and `gen` the
// generation word, both zeroed before the launch. Every arrival is an acq_rel
// RMW, so the last arriver (return true) has acquired every CTA's phase writes
// through the RMW release sequence; it then runs its serial step and calls
// grid_release(), whose release store the waiters acquire. No sc fences
// (MEMBAR.SC.GPU), no counter reset, one RMW per CTA.
__device__ __forceinline__ bool grid_arrive(u32* count, u32* target) {
  const u32 G = gridDim.x;
  const u32 t = atom_add_acq_rel_u32(count, 1u);
  *target = t / G + 1;
  return t % G == G - 1;
}
__device__ __forceinline__ void grid_release(u32* gen, u32 target) { st_release_u32(gen, target); }
__device__ __forceinline__ void grid_wait(const u32* gen, u32 target) {
  u32 ns = 32;
  while ((int)(ld_acquire_u32(gen) - target) < 0) {
    __nanosleep(ns);
    if (ns < 128) ns <<= 1;
  }
}

__device__ __forceinline__ void st_relaxed_u64(u64* p, u64 v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_u32(u32* p, u32 v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Bulk prefetch of a contiguous global range into L2 (sm_90+; no registers,
// no completion tracking). Used to start the arc stream of every claimed
// vertex while the batch is still being staged.
__device__ __forceinline__ void prefetch_l2(const void* p, u32 bytes) {
  const uintptr_t a = (uintptr_t)p & ~(uintptr_t)15;
  const uintptr_t e = ((uintptr_t)p + bytes + 15) & ~(uintptr_t)15;
  if (e > a)
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"((u32)(e - a)) : "memory");
}

__device__ __forceinline__ u64 policy_evict_last() {
  u64 pol;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ u32 lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ u32 lanemask_lt() {
  u32 m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

template <class T>
__device__ __forceinline__ T warp_exclusive_scan(T x, T* total) {
  const u32 lane = lane_id();
  T v = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T y = __shfl_up_sync(SSSP_FULL_MASK, v, o);
    if (lane >= (u32)o) v += y;
  }
  *total = __shfl_sync(SSSP_FULL_MASK, v, 31);
  return v - x;
}

}  // namespace sssp
