// ubench_relax.cu -- ceilings of the relaxation access pattern on one B200.
//
// One "sweep" = every arc of a synthetic CSR-like arc array (8 B {dst, w},
// read coalesced, streamed) relaxed against dist[V] (u32, random access):
//   stream   : arcs only (sum)                          -> HBM read bandwidth
//   probe    : arcs + dist[dst] load                    -> + random L2 loads
//   relax    : arcs + probe + atomicMin if it improves  -> the Delta-stepping inner loop
//   atomic   : arcs + atomicMin always                  -> random L2 atomics
// dst distribution: "unif" (uniform over V) or "skew" (V * u^3: low ids hot,
// like a degree-sorted RMAT graph after PRO).
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench tools/ubench_relax.cu
// /tmp/ubench [V=16777216] [A=536870912]
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

typedef unsigned long long u64;
typedef uint32_t u32;

__device__ __forceinline__ u64 mix(u64 x) {
  x += 0x9E3779B97F4A7C15ULL;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
  return x ^ (x >> 31);
}

__global__ void k_gen(uint2* arcs, u64 A, u32 V, int skew) {
  for (u64 i = blockIdx.x * (u64)blockDim.x + threadIdx.x; i < A; i += (u64)gridDim.x * blockDim.x) {
    const u64 r = mix(i);
    const double u = (double)(r >> 11) * (1.0 / 9007199254740992.0);
    const u32 dst = skew ? (u32)(V * u * u * u) : (u32)(r % V);
    arcs[i] = make_uint2(dst < V ? dst : V - 1, 1 + (u32)((r >> 40) % 100));
  }
}

__global__ void k_init(u32* dist, u32 V, u32 base) {
  for (u32 i = blockIdx.x * blockDim.x + threadIdx.x; i < V; i += gridDim.x * blockDim.x)
    dist[i] = base + (u32)(mix(i + 77) % 64);
}

__device__ __forceinline__ uint2 ld_arc(const uint2* p) {
  uint2 v;
  asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p));
  return v;
}

template <int MODE>  // 0 stream, 1 probe, 2 relax, 3 atomic
__global__ void __launch_bounds__(256) k_sweep(const uint2* __restrict__ arcs, u64 A, u32* dist, u32 dsrc,
                                              unsigned long long* out) {
  const u64 nt = (u64)gridDim.x * blockDim.x;
  u64 acc = 0;
  u32 nat = 0;
  constexpr int U = 4;
  for (u64 i0 = blockIdx.x * (u64)blockDim.x * U + threadIdx.x; i0 < A; i0 += nt * U) {
    uint2 a[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const u64 i = i0 + (u64)k * blockDim.x;
      a[k] = i < A ? ld_arc(arcs + i) : make_uint2(0, 0xFFFFFFFFu);
    }
    u32 cur[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      if (MODE == 0) {
        acc += a[k].x + a[k].y;
      } else if (MODE == 1 || MODE == 2) {
        cur[k] = __ldca(dist + a[k].x);
      }
    }
    if (MODE == 1) {
#pragma unroll
      for (int k = 0; k < U; ++k) acc += cur[k];
    } else if (MODE == 2) {
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const u32 nd = dsrc + a[k].y;
        if (a[k].y != 0xFFFFFFFFu && nd < cur[k]) {
          acc += atomicMin(dist + a[k].x, nd);
          ++nat;
        }
      }
    } else if (MODE == 3) {
#pragma unroll
      for (int k = 0; k < U; ++k)
        if (a[k].y != 0xFFFFFFFFu) acc += atomicMin(dist + a[k].x, dsrc + a[k].y);
    }
  }
  if (acc == 0x123456789ULL) out[0] = acc;
  if (MODE == 2) atomicAdd(out + 1, (unsigned long long)nat);
}

int main(int argc, char** argv) {
  const u32 V = argc > 1 ? (u32)atoll(argv[1]) : 16777216u;
  const u64 A = argc > 2 ? (u64)atoll(argv[2]) : 536870912ull;
  int dev = 0, sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint2* arcs;
  u32* dist;
  unsigned long long* out;
  cudaMalloc(&arcs, A * sizeof(uint2));
  cudaMalloc(&dist, (size_t)V * 4);
  cudaMalloc(&out, 16);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const char* names[] = {"stream", "probe", "relax", "atomic"};
  for (int skew = 0; skew < 2; ++skew) {
    k_gen<<<sms * 8, 256>>>(arcs, A, V, skew);
    for (int mode = 0; mode < 4; ++mode) {
      // relax: dist around base so that ~"frac" of arcs improve (base 40: nd = 1 + w in [2, 101])
      for (u32 base : {0u, 40u, 200u}) {
        if (mode != 2 && base != 0) continue;
        float best = 1e30f;
        unsigned long long nat = 0;
        for (int rep = 0; rep < 3; ++rep) {
          k_init<<<sms * 8, 256>>>(dist, V, mode == 2 ? base : 0xFFFFFF00u);
          cudaMemset(out, 0, 16);
          cudaEventRecord(e0);
          switch (mode) {
            case 0: k_sweep<0><<<sms * 8, 256>>>(arcs, A, dist, 1, out); break;
            case 1: k_sweep<1><<<sms * 8, 256>>>(arcs, A, dist, 1, out); break;
            case 2: k_sweep<2><<<sms * 8, 256>>>(arcs, A, dist, 1, out); break;
            default: k_sweep<3><<<sms * 8, 256>>>(arcs, A, dist, 1, out); break;
          }
          cudaEventRecord(e1);
          cudaEventSynchronize(e1);
          float ms;
          cudaEventElapsedTime(&ms, e0, e1);
          if (ms < best) best = ms;
          cudaMemcpy(&nat, out + 1, 8, cudaMemcpyDeviceToHost);
        }
        printf("%-5s %-7s base=%3u  %8.3f ms  arcs %6.1f G/s  arc-bytes %7.1f GB/s  atomics %.3f G\n",
               skew ? "skew" : "unif", names[mode], base, best, A / best / 1e6, 8.0 * A / best / 1e6,
               mode == 3 ? A / 1e9 : nat / 1e9);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}
