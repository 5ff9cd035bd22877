// sort.cuh -- device-wide exclusive scan and stable LSD radix-sort passes
// (8-bit digits) used by the property-driven reordering (PAPER §4.1,
// "we reorder the vertices in descending order by degree" and
// "sort the adjacency list and value list in ascending order of weight").
//
// Radix pass = per-tile digit histogram (digit-major) -> exclusive scan ->
// stable scatter. Tiles are 4096 elements: each of the 8 warps ranks its own
// contiguous 512-element sub-tile in 16 rounds of 32 with __match_any_sync
// (warp-sequential counters in shared memory), then warps are combined with
// a per-digit exclusive scan, so the output order is stable.
#pragma once
#include "common.cuh"

namespace sssp {

constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ROUNDS = 8;  // tile = 2048 elements
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ROUNDS;

template <class T>
__device__ __forceinline__ T block_exclusive_scan(T x, T* total, T* warp_sums /*[8]*/) {
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  T wt;
  T ex = warp_exclusive_scan(x, &wt);
  if (l == 31) warp_sums[w] = wt;
  __syncthreads();
  T acc = 0, tot = 0;
#pragma unroll
  for (int i = 0; i < SCAN_THREADS / 32; ++i) {
    T s = warp_sums[i];
    if (i < w) acc += s;
    tot += s;
  }
  __syncthreads();
  *total = tot;
  return ex + acc;
}

template <class T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_reduce(const T* __restrict__ in, i64 n,
                                                              T* __restrict__ sums) {
  __shared__ T ws[SCAN_THREADS / 32];
  const i64 base = (i64)blockIdx.x * SCAN_TILE;
  T acc = 0;
  for (int r = 0; r < SCAN_ROUNDS; ++r) {
    i64 i = base + r * SCAN_THREADS + threadIdx.x;
    if (i < n) acc += in[i];
  }
  T tot;
  block_exclusive_scan(acc, &tot, ws);
  if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

template <class T>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_tiles(const T* __restrict__ in, i64 n,
                                                             T* __restrict__ out,
                                                             const T* __restrict__ offs) {
  __shared__ T ws[SCAN_THREADS / 32];
  const i64 base = (i64)blockIdx.x * SCAN_TILE;
  T carry = offs ? offs[blockIdx.x] : (T)0;
  for (int r = 0; r < SCAN_ROUNDS; ++r) {
    i64 i = base + r * SCAN_THREADS + threadIdx.x;
    T x = i < n ? in[i] : (T)0;
    T tot;
    T ex = block_exclusive_scan(x, &tot, ws);
    if (i < n) out[i] = carry + ex;
    carry += tot;
  }
}

// Exclusive scan of n elements (in may equal out). tmp must hold
// scan_tmp_elems(n) elements. If total != nullptr, *total (device) gets the sum.
inline i64 scan_tmp_elems(i64 n) {
  i64 t = 0;
  while (n > SCAN_TILE) {
    n = (n + SCAN_TILE - 1) / SCAN_TILE;
    t += n;
  }
  return t + 1;
}

template <class T>
__global__ void k_scan_total(const T* in, const T* ex, i64 n, T* total) {
  *total = n > 0 ? ex[n - 1] + in[n - 1] : (T)0;
}

template <class T>
void scan_exclusive_rec(const T* in, T* out, i64 n, T* tmp, cudaStream_t st) {
  if (n <= 0) return;
  i64 nt = (n + SCAN_TILE - 1) / SCAN_TILE;
  if (nt == 1) {
    k_scan_tiles<T><<<1, SCAN_THREADS, 0, st>>>(in, n, out, (const T*)nullptr);
    return;
  }
  T* sums = tmp;
  k_scan_reduce<T><<<(unsigned)nt, SCAN_THREADS, 0, st>>>(in, n, sums);
  scan_exclusive_rec<T>(sums, sums, nt, tmp + nt, st);
  k_scan_tiles<T><<<(unsigned)nt, SCAN_THREADS, 0, st>>>(in, n, out, sums);
}

// ------------------------------------------------------------ radix ------
constexpr int RS_THREADS = 256;
constexpr int RS_ROUNDS = 16;
constexpr int RS_WARP_ELEMS = 32 * RS_ROUNDS;  // 512
constexpr int RS_TILE = RS_WARP_ELEMS * (RS_THREADS / 32);  // 4096

template <int NF>
struct Fields {
  u32* f[NF];
};

__global__ void __launch_bounds__(RS_THREADS) k_rs_hist(const u32* __restrict__ key, i64 n, int sh,
                                                        u32* __restrict__ hist, u32 ntiles) {
  __shared__ u32 cnt[256];
  cnt[threadIdx.x] = 0;
  __syncthreads();
  const i64 base = (i64)blockIdx.x * RS_TILE;
  for (int r = 0; r < RS_TILE / RS_THREADS; ++r) {
    i64 i = base + r * RS_THREADS + threadIdx.x;
    if (i < n) atomicAdd(&cnt[(key[i] >> sh) & 255u], 1u);
  }
  __syncthreads();
  hist[(i64)threadIdx.x * ntiles + blockIdx.x] = cnt[threadIdx.x];
}

// Stable scatter of one 8-bit digit pass. kf = index of the key field.
template <int NF>
__global__ void __launch_bounds__(RS_THREADS) k_rs_scatter(Fields<NF> in, Fields<NF> out, int kf,
                                                           i64 n, int sh,
                                                           const u32* __restrict__ hist_scan,
                                                           u32 ntiles) {
  __shared__ u32 wcnt[RS_THREADS / 32][256];
  __shared__ u32 gbase[256];
  const u32 w = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < RS_THREADS / 32; ++i) wcnt[i][threadIdx.x] = 0;
  gbase[threadIdx.x] = hist_scan[(i64)threadIdx.x * ntiles + blockIdx.x];
  __syncthreads();
  const i64 base = (i64)blockIdx.x * RS_TILE + (i64)w * RS_WARP_ELEMS;
  u32 val[RS_ROUNDS][NF];
  u32 dig[RS_ROUNDS];
  u32 rnk[RS_ROUNDS];
#pragma unroll
  for (int r = 0; r < RS_ROUNDS; ++r) {
    const i64 i = base + r * 32 + lane;
    const bool valid = i < n;
#pragma unroll
    for (int k = 0; k < NF; ++k) val[r][k] = valid ? in.f[k][i] : 0u;
    u32 d = 0;
#pragma unroll
    for (int k = 0; k < NF; ++k)
      if (k == kf) d = (val[r][k] >> sh) & 255u;
    dig[r] = valid ? d : 256u;
    const u32 m = __ballot_sync(SSSP_FULL_MASK, valid);
    u32 b = 0, peers = 0;
    if (valid) {
      peers = __match_any_sync(m, d);
      b = wcnt[w][d];
    }
    __syncwarp();
    if (valid && lane == (u32)(__ffs(peers) - 1)) wcnt[w][d] = b + __popc(peers);
    __syncwarp();
    rnk[r] = b + __popc(peers & lanemask_lt());
  }
  __syncthreads();
  {  // per digit: exclusive scan over warps
    u32 run = 0;
#pragma unroll
    for (int i = 0; i < RS_THREADS / 32; ++i) {
      u32 c = wcnt[i][threadIdx.x];
      wcnt[i][threadIdx.x] = run;
      run += c;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RS_ROUNDS; ++r) {
    if (dig[r] < 256u) {
      const u32 pos = gbase[dig[r]] + wcnt[w][dig[r]] + rnk[r];
#pragma unroll
      for (int k = 0; k < NF; ++k) out.f[k][pos] = val[r][k];
    }
  }
}

// Stable scatter through shared memory: the tile is first reordered by digit
// in shared memory (same stable ranks as k_rs_scatter), then written out in
// digit runs so consecutive threads store consecutive global addresses.
// Dynamic shared memory: NF * RS_TILE * 4 bytes of staging.
template <int NF>
__global__ void __launch_bounds__(RS_THREADS) k_rs_scatter_smem(Fields<NF> in, Fields<NF> out, int kf,
                                                                i64 n, int sh,
                                                                const u32* __restrict__ hist_scan,
                                                                u32 ntiles) {
  extern __shared__ u32 stage[];  // [NF][RS_TILE]
  __shared__ u32 wcnt[RS_THREADS / 32][256];
  __shared__ u32 gbase[256];
  __shared__ u32 dstart[257];
  const u32 w = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < RS_THREADS / 32; ++i) wcnt[i][threadIdx.x] = 0;
  gbase[threadIdx.x] = hist_scan[(i64)threadIdx.x * ntiles + blockIdx.x];
  __syncthreads();
  const i64 tbase = (i64)blockIdx.x * RS_TILE;
  const i64 base = tbase + (i64)w * RS_WARP_ELEMS;
  u32 dig[RS_ROUNDS];
  u32 rnk[RS_ROUNDS];
#pragma unroll
  for (int r = 0; r < RS_ROUNDS; ++r) {
    const i64 i = base + r * 32 + lane;
    const bool valid = i < n;
    const u32 d = valid ? (in.f[kf][i] >> sh) & 255u : 0u;
    dig[r] = valid ? d : 256u;
    const u32 m = __ballot_sync(SSSP_FULL_MASK, valid);
    u32 b = 0, peers = 0;
    if (valid) {
      peers = __match_any_sync(m, d);
      b = wcnt[w][d];
    }
    __syncwarp();
    if (valid && lane == (u32)(__ffs(peers) - 1)) wcnt[w][d] = b + __popc(peers);
    __syncwarp();
    rnk[r] = b + __popc(peers & lanemask_lt());
  }
  __syncthreads();
  {  // per digit: exclusive scan over warps, tile total
    u32 run = 0;
#pragma unroll
    for (int i = 0; i < RS_THREADS / 32; ++i) {
      u32 c = wcnt[i][threadIdx.x];
      wcnt[i][threadIdx.x] = run;
      run += c;
    }
    dstart[threadIdx.x] = run;  // tile count of this digit (scanned below)
  }
  __syncthreads();
  if (threadIdx.x < 32) {  // exclusive scan of 256 digit counts by one warp
    u32 v[8], t = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      v[j] = dstart[threadIdx.x * 8 + j];
      t += v[j];
    }
    u32 tot;
    u32 ex = warp_exclusive_scan(t, &tot);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const u32 c = v[j];
      dstart[threadIdx.x * 8 + j] = ex;
      ex += c;
    }
    if (threadIdx.x == 31) dstart[256] = tot;
  }
  __syncthreads();
  // scatter into shared memory in digit order
#pragma unroll
  for (int r = 0; r < RS_ROUNDS; ++r) {
    if (dig[r] < 256u) {
      const i64 i = base + r * 32 + lane;
      const u32 lp = dstart[dig[r]] + wcnt[w][dig[r]] + rnk[r];
#pragma unroll
      for (int k = 0; k < NF; ++k) stage[k * RS_TILE + lp] = in.f[k][i];
    }
  }
  __syncthreads();
  // coalesced write-out of the digit runs
  const u32 cnt = dstart[256];
  for (u32 lp = threadIdx.x; lp < cnt; lp += RS_THREADS) {
    const u32 d = (stage[kf * RS_TILE + lp] >> sh) & 255u;
    const u32 gp = gbase[d] + (lp - dstart[d]);
#pragma unroll
    for (int k = 0; k < NF; ++k) out.f[k][gp] = stage[k * RS_TILE + lp];
  }
}

}  // namespace sssp
