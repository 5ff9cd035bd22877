// sssp_api.cu -- C-ABI runtime of libsssp.so (see include/sssp.h).
// Host side: validation, device memory, stream-ordered launches. Every step
// of the SSSP path runs in the kernels of pro.cuh / sort.cuh / delta_step.cuh.
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges cost nothing without a profiler

#include <algorithm>
#include <cmath>
#include <mutex>
#include <unordered_map>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/sssp.h"
#include "delta_step.cuh"
#include "multi_source.cuh"
#include "pro.cuh"
#include "sort.cuh"

using namespace sssp;

// NVTX range over one ABI call (visible in Nsight Systems / ncu --nvtx).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// ------------------------------------------------------ allocator hook ---
// sssp_set_allocator: device buffers of every handle come from the hook (e.g. torch's caching
// allocator) when one is set; each buffer remembers the hook that made it, so it is always
// returned to the same one, also after the hook changes.
struct AllocHook {
  sssp_alloc_fn alloc = nullptr;
  sssp_free_fn free = nullptr;
  void* ctx = nullptr;
};
static std::mutex g_alloc_mu;
static AllocHook g_hook;
static std::unordered_map<void*, std::pair<AllocHook, size_t>> g_hooked;

static cudaError_t dalloc(void** ptr, size_t bytes, cudaStream_t s = nullptr) {
  AllocHook h;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    h = g_hook;
  }
  if (!h.alloc) return cudaMalloc(ptr, bytes);
  int dev = 0;
  cudaGetDevice(&dev);
  void* q = h.alloc(bytes, dev, (void*)s, h.ctx);
  if (!q) return cudaErrorMemoryAllocation;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    g_hooked[q] = {h, bytes};
  }
  *ptr = q;
  return cudaSuccess;
}
template <class T>
static cudaError_t dalloc(T** ptr, size_t bytes, cudaStream_t s = nullptr) {
  return dalloc(reinterpret_cast<void**>(ptr), bytes, s);
}

static cudaError_t dfree(void* ptr, cudaStream_t s = nullptr) {
  if (!ptr) return cudaSuccess;
  AllocHook h;
  size_t bytes = 0;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    auto it = g_hooked.find(ptr);
    if (it != g_hooked.end()) {
      h = it->second.first;
      bytes = it->second.second;
      g_hooked.erase(it);
    }
  }
  if (!h.free) return cudaFree(ptr);
  int dev = 0;
  cudaGetDevice(&dev);
  h.free(ptr, bytes, dev, (void*)s, h.ctx);
  return cudaSuccess;
}

extern "C" sssp_status sssp_set_allocator(sssp_alloc_fn alloc, sssp_free_fn free_fn, void* ctx) {
  if ((alloc == nullptr) != (free_fn == nullptr)) return SSSP_ERR_INVALID_ARGUMENT;
  std::lock_guard<std::mutex> lk(g_alloc_mu);
  g_hook.alloc = alloc;
  g_hook.free = free_fn;
  g_hook.ctx = ctx;
  return SSSP_OK;
}

// --------------------------------------------------------------- errors ---
static thread_local std::string g_last_error;

static sssp_status fail(sssp_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return s;
}

struct sssp_graph_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  int num_sms = 0;
  i64 V = 0, A = 0;
  sssp_weight_type wtype = SSSP_WEIGHT_U32;
  longlong2* rowp = nullptr;  // [V+1] {start, heavy}
  uint2* rowc = nullptr;      // [V+1] compact copy for the persistent kernel
  bool rowc_valid = false;
  uint2* rowc_lv = nullptr;   // [5][V+1] adaptive Delta: heavy offsets for light levels g << l
  bool rowc_lv_valid = false;
  u32 rowc_lv_g = 0;          // fine-unit bits the levels were built for
  uint2* arcs = nullptr;      // [A]
  u32 maxw_bits = 0;
  u32* old2new = nullptr;  // null until PRO_DEGREE
  u32* new2old = nullptr;
  std::vector<u32> h_old2new;  // host copy: source mapping without a sync per run
  unsigned pro_flags = 0;
  bool heavy_valid = false;
  u32 heavy_bits = 0;
  // run state
  u32* dist = nullptr;
  u32* xd = nullptr;
  Ctl* ctl = nullptr;
  SlotCtl* sc = nullptr;
  u64* items = nullptr;
  u64* hub_items = nullptr;
  u32* p2o = nullptr;  // [cap] + uint2 [cap]: edge-balanced phase-2 scratch
  // batched multi-source kernel (NEXT-4, sssp_run_multi)
  u32* ms_D = nullptr;     // [V][32]
  u32* ms_Q = nullptr;     // [V]
  u64* ms_items = nullptr; // [ms_K * ms_cap]
  SlotCtl* ms_sc = nullptr;
  MCtl* ms_ctl = nullptr;
  unsigned long long* ms_stats = nullptr;
  u32* ms_src = nullptr;   // [32] sources, then [32] key shifts
  std::vector<u32> h_hubdist;  // distances from the max-degree vertex (lane alignment)
  u32 hubdist_bits = 0xFFFFFFFFu;
  u32 ms_K = 0, ms_cap = 0;
  u32* out_tmp = nullptr;  // [V] staging for sssp_distances into pageable host memory
  // sssp_distances_async: the output gather writes a device staging buffer (fast, on
  // the run stream), a copy engine moves it to the host on d2h while the next run computes
  u32* stage[2] = {nullptr, nullptr};
  int stage_next = 0;
  bool stage_used[2] = {false, false};
  cudaEvent_t ev_out[2] = {nullptr, nullptr};
  cudaEvent_t ev_ran = nullptr;
  cudaStream_t d2h = nullptr;
  unsigned long long* stats = nullptr;
  TraceEnt* trace = nullptr;
  u32 K_alloc = 0, cap_alloc = 0, hub_cap = 0;
  u32 K_used = 0;
  bool need_full_reset = true;
  bool have_result = false;
  bool sticky_cuda = false;
  int grid_ctas = 0;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  // per-launch timing of the persistent kernel (sssp_kernel_time)
  std::vector<cudaEvent_t> ev_pool;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> ev_pending;
  double kt_total_ms = 0.0;
  int64_t kt_launches = 0;
  bool run_timed = false, reorder_timed = false;
  // params
  i64 p_ring = 0, p_ctas = 0, p_cap = 0, p_claim = BATCH, p_l2 = 1, p_adwl = 1, p_sync = 0, p_p2eb = -1, p_adapt = 0, p_align = 1, p_hub_delay = 0, p_pull = 0, p_local = 1, p_local_lim = LOC_CAP, p_bf = -1;
  i64 hub_ids_cached = -1;
  int sym_state = -1;  // arc multiset symmetric? -1 unknown (checked on demand after a weight sort)
  i64 v_nz = -1;       // degree-sorted graphs: vertices with arcs are ids [0, v_nz); -1 unknown
  i64 l2_window_bytes = -1;  // -1: not configured yet
  float l2_hit_ratio = 1.f;
};

#define CU(call)                                                                       \
  do {                                                                                 \
    cudaError_t e_ = (call);                                                           \
    if (e_ != cudaSuccess) {                                                           \
      if (g) g->sticky_cuda = true;                                                    \
      return fail(e_ == cudaErrorMemoryAllocation ? SSSP_ERR_OUT_OF_MEMORY : SSSP_ERR_CUDA, \
                  "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));  \
    }                                                                                  \
  } while (0)

static unsigned grid_for(i64 n, int threads = 256) {
  i64 b = (n + threads - 1) / threads;
  return (unsigned)std::max<i64>(1, std::min<i64>(b, 148 * 32));
}

static sssp_status check_handle(sssp_graph_t g) {
  if (!g) return fail(SSSP_ERR_INVALID_ARGUMENT, "null graph handle");
  if (g->sticky_cuda) return fail(SSSP_ERR_CUDA, "handle is in a failed CUDA state; destroy it");
  return SSSP_OK;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    cudaGetDevice(&prev);
    if (prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// --------------------------------------------------------------- create ---
extern "C" sssp_status sssp_graph_create(sssp_graph_t* out, int device, int64_t V, int64_t A,
                                         const int64_t* row, const uint32_t* col,
                                         const void* weights, sssp_weight_type wtype,
                                         sssp_memory where, void* cuda_stream) {
  NvtxRange nvtx_("sssp_graph_create");
  sssp_graph_s* g = nullptr;
  if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
  if (V < 1 || V >= 0x7FFFFFFFLL) return fail(SSSP_ERR_INVALID_ARGUMENT, "V=%lld out of [1, 2^31-1)", (long long)V);
  if (A < 0 || A >= 0xFFFFFFFFLL) return fail(SSSP_ERR_INVALID_ARGUMENT, "A=%lld out of [0, 2^32-1)", (long long)A);
  if (!row || (A > 0 && (!col || !weights))) return fail(SSSP_ERR_INVALID_ARGUMENT, "null CSR pointer");
  if (wtype != SSSP_WEIGHT_U32 && wtype != SSSP_WEIGHT_F32) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad weight type");
  if (where != SSSP_MEM_HOST && where != SSSP_MEM_DEVICE) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad memory kind");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
    return fail(SSSP_ERR_INVALID_ARGUMENT, "CUDA device %d not available", device);
  DeviceGuard dg(device);
  g = new (std::nothrow) sssp_graph_s();
  if (!g) return fail(SSSP_ERR_OUT_OF_MEMORY, "host allocation failed");
  g->device = device;
  g->stream = (cudaStream_t)cuda_stream;
  g->V = V;
  g->A = A;
  g->wtype = wtype;
  cudaDeviceProp prop;
  sssp_status st = SSSP_OK;
  auto bail = [&](sssp_status s) {
    sssp_destroy(g);
    return s;
  };
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return bail(fail(SSSP_ERR_CUDA, "cudaGetDeviceProperties"));
  g->num_sms = prop.multiProcessorCount;
  const cudaMemcpyKind kind = where == SSSP_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  i64* d_row = nullptr;
  u32 *d_col = nullptr, *d_w = nullptr, *d_flags = nullptr;
  do {
    cudaStream_t s = g->stream;
#define CG(call)                                                                        \
    {                                                                                   \
      cudaError_t e_ = (call);                                                          \
      if (e_ != cudaSuccess) {                                                          \
        st = fail(e_ == cudaErrorMemoryAllocation ? SSSP_ERR_OUT_OF_MEMORY : SSSP_ERR_CUDA, \
                  "create: %s: %s", #call, cudaGetErrorString(e_));                     \
        break;                                                                          \
      }                                                                                 \
    }
    CG(dalloc(&g->rowp, sizeof(longlong2) * (V + 1)));
    CG(dalloc(&g->rowc, sizeof(uint2) * (V + 1)));
    CG(dalloc(&g->arcs, sizeof(uint2) * std::max<i64>(A, 1)));
    CG(dalloc(&g->dist, sizeof(u32) * V));
    CG(dalloc(&g->xd, sizeof(u32) * (5 * V + 4)));  // sweep marks, two pull candidate lists, long scans
    CG(dalloc(&g->ctl, sizeof(Ctl)));
    CG(dalloc(&g->stats, sizeof(unsigned long long) * ST_N));
    CG(dalloc(&g->trace, sizeof(TraceEnt) * (TRACE_CAP + SAMPLE_CAP)));
    CG(cudaMemsetAsync(g->ctl, 0, sizeof(Ctl), s));
    CG(cudaMemsetAsync(g->stats, 0, sizeof(unsigned long long) * ST_N, s));
    for (int i = 0; i < 4; ++i) CG(cudaEventCreate(&g->ev[i]));
    CG(dalloc(&d_row, sizeof(i64) * (V + 1), s));
    CG(dalloc(&d_flags, sizeof(u32) * 2, s));
    CG(cudaMemsetAsync(d_flags, 0, sizeof(u32) * 2, s));
    CG(cudaMemcpyAsync(d_row, row, sizeof(i64) * (V + 1), kind, s));
    if (A > 0) {
      CG(dalloc(&d_col, sizeof(u32) * A, s));
      CG(dalloc(&d_w, sizeof(u32) * A, s));
      CG(cudaMemcpyAsync(d_col, col, sizeof(u32) * A, kind, s));
      CG(cudaMemcpyAsync(d_w, weights, sizeof(u32) * A, kind, s));
    }
    k_check_rows<<<grid_for(V), 256, 0, s>>>(d_row, V, A, d_flags);
    k_rows_to_rowp<<<grid_for(V + 1), 256, 0, s>>>(d_row, V, g->rowp);
    if (A > 0)
      k_pack_arcs<<<grid_for(A), 256, 0, s>>>(d_col, d_w, A, (u32)V, wtype == SSSP_WEIGHT_F32,
                                               g->arcs, d_flags, d_flags + 1);
    CG(cudaGetLastError());
    u32 flags[2] = {0, 0};
    CG(cudaMemcpyAsync(flags, d_flags, sizeof flags, cudaMemcpyDeviceToHost, s));
    CG(cudaStreamSynchronize(s));  // the temporaries are free to go (plain or hooked frees)
    CG(dfree(d_row, s));
    d_row = nullptr;
    CG(dfree(d_flags, s));
    d_flags = nullptr;
    CG(dfree(d_col, s));
    d_col = nullptr;
    CG(dfree(d_w, s));
    d_w = nullptr;
    if (flags[0]) {
      st = fail(SSSP_ERR_INVALID_ARGUMENT, "invalid CSR:%s%s%s%s", (flags[0] & 1) ? " row[0]!=0 or row[V]!=A" : "",
                (flags[0] & 2) ? " row offsets decrease" : "", (flags[0] & 4) ? " col index >= V" : "",
                (flags[0] & 8) ? " weight negative/NaN/inf" : "");
      break;
    }
    g->maxw_bits = flags[1];
#undef CG
  } while (0);
  if (st != SSSP_OK) {
    cudaStreamSynchronize(g->stream);
    dfree(d_row);
    dfree(d_col);
    dfree(d_w);
    dfree(d_flags);
    return bail(st);
  }
  *out = g;
  return SSSP_OK;
}

extern "C" void sssp_destroy(sssp_graph_t g) {
  if (!g) return;
  DeviceGuard dg(g->device);
  if (g->stream) cudaStreamSynchronize(g->stream);
  else cudaDeviceSynchronize();
  if (g->d2h) cudaStreamSynchronize(g->d2h);
  for (auto& e : g->ev_out)
    if (e) cudaEventDestroy(e);
  if (g->ev_ran) cudaEventDestroy(g->ev_ran);
  if (g->d2h) cudaStreamDestroy(g->d2h);
  void* ptrs[] = {g->rowp, g->rowc, g->arcs, g->old2new, g->new2old, g->dist, g->stage[0], g->stage[1], g->xd, g->ctl, g->sc,
                  g->items, g->hub_items, g->p2o, g->rowc_lv, g->ms_D, g->ms_Q, g->ms_items, g->ms_sc, g->ms_ctl, g->ms_stats, g->ms_src, g->stats, g->trace, g->out_tmp};
  for (void* p : ptrs)
    if (p) dfree(p);
  for (auto& e : g->ev)
    if (e) cudaEventDestroy(e);
  for (auto& e : g->ev_pool) cudaEventDestroy(e);
  for (auto& pr : g->ev_pending) {
    cudaEventDestroy(pr.first);
    cudaEventDestroy(pr.second);
  }
  cudaGetLastError();  // do not leak a sticky error to the caller's context
  delete g;
}

extern "C" const char* sssp_status_string(sssp_status s) {
  switch (s) {
    case SSSP_OK: return "SSSP_OK";
    case SSSP_ERR_INVALID_ARGUMENT: return "SSSP_ERR_INVALID_ARGUMENT";
    case SSSP_ERR_OUT_OF_MEMORY: return "SSSP_ERR_OUT_OF_MEMORY";
    case SSSP_ERR_CUDA: return "SSSP_ERR_CUDA";
    case SSSP_ERR_INVALID_STATE: return "SSSP_ERR_INVALID_STATE";
    case SSSP_ERR_OVERFLOW: return "SSSP_ERR_OVERFLOW";
    case SSSP_ERR_INTERNAL: return "SSSP_ERR_INTERNAL";
  }
  return "SSSP_UNKNOWN_STATUS";
}

extern "C" const char* sssp_last_error(void) { return g_last_error.c_str(); }

extern "C" sssp_status sssp_set_stream(sssp_graph_t g, void* cuda_stream) {
  sssp_status s = check_handle(g);
  if (s) return s;
  g->stream = (cudaStream_t)cuda_stream;
  return SSSP_OK;
}

extern "C" int sssp_device_sm_count(sssp_graph_t g) { return g ? g->num_sms : 0; }

extern "C" sssp_status sssp_set_param(sssp_graph_t g, sssp_param p, int64_t v) {
  sssp_status s = check_handle(g);
  if (s) return s;
  switch (p) {
    case SSSP_PARAM_RING_SLOTS:
      if (v != 0 && (v < 4 || v > 64 || (v & (v - 1)))) return fail(SSSP_ERR_INVALID_ARGUMENT, "ring slots must be 0 or a power of two in [4,64]");
      g->p_ring = v;
      return SSSP_OK;
    case SSSP_PARAM_CTAS_PER_SM:
      if (v < 0 || v > 32) return fail(SSSP_ERR_INVALID_ARGUMENT, "ctas per SM in [0,32]");
      g->p_ctas = v;
      return SSSP_OK;
    case SSSP_PARAM_SLOT_CAPACITY:
      if (v < 0 || v > 0x7FFFFFFFLL || (v != 0 && v < 4096)) return fail(SSSP_ERR_INVALID_ARGUMENT, "slot capacity 0 or in [4096, 2^31)");
      g->p_cap = v;
      return SSSP_OK;
    case SSSP_PARAM_L2_PERSIST:
      if (v != 0 && v != 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "l2 persist is 0 or 1");
      g->p_l2 = v;
      g->l2_window_bytes = -1;
      return SSSP_OK;
    case SSSP_PARAM_ADWL:
      if (v != 0 && v != 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "adwl is 0 or 1");
      g->p_adwl = v;
      return SSSP_OK;
    case SSSP_PARAM_SYNC:
      if (v != 0 && v != 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "sync is 0 or 1");
      g->p_sync = v;
      return SSSP_OK;
    case SSSP_PARAM_P2_EDGE_BALANCED:
      if (v < -1 || v > 0x7FFFFF) return fail(SSSP_ERR_INVALID_ARGUMENT, "p2 edge-balanced threshold in [-1, 2^23)");
      g->p_p2eb = v;
      return SSSP_OK;
    case SSSP_PARAM_ADAPTIVE_DELTA:
      if (v < 0 || v > 2) return fail(SSSP_ERR_INVALID_ARGUMENT, "adaptive delta is 0, 1 or 2");
      g->p_adapt = v;
      return SSSP_OK;
    case SSSP_PARAM_MULTI_ALIGN:
      if (v != 0 && v != 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "multi align is 0 or 1");
      g->p_align = v;
      return SSSP_OK;
    case SSSP_PARAM_MULTI_HUB_DELAY:
      if (v < 0 || v > 16) return fail(SSSP_ERR_INVALID_ARGUMENT, "hub delay in [0,16]");
      g->p_hub_delay = v;
      return SSSP_OK;
    case SSSP_PARAM_PULL_SYMMETRIC:
      if (v != 0 && v != 1) return fail(SSSP_ERR_INVALID_ARGUMENT, "pull is 0 or 1");
      if (v && (g->pro_flags & SSSP_PRO_WEIGHT)) {  // layout ready: verify the assertion now
        int sym = 0;
        if ((s = sssp_is_symmetric(g, &sym))) return s;
        if (!sym) return fail(SSSP_ERR_INVALID_STATE, "pull phases need a symmetric graph; this one is not");
      }
      g->p_pull = v;
      return SSSP_OK;
    case SSSP_PARAM_LOCAL_CHASE:
      if (v < 0 || v > 2) return fail(SSSP_ERR_INVALID_ARGUMENT, "local chase is 0, 1 or 2");
      g->p_local = v;
      return SSSP_OK;
    case SSSP_PARAM_BF_TAIL:
      if (v < -1 || v > 0x7FFFFFFF) return fail(SSSP_ERR_INVALID_ARGUMENT, "Bellman-Ford end threshold -1 (auto) or in [0, 2^31)");
      g->p_bf = v;
      return SSSP_OK;
    case SSSP_PARAM_LOCAL_LIMIT:
      if (v < 1 || v > (i64)LOC_CAP) return fail(SSSP_ERR_INVALID_ARGUMENT, "local limit in [1,%u]", LOC_CAP);
      g->p_local_lim = v;
      return SSSP_OK;
    case SSSP_PARAM_CLAIM_MAX:
      if (v < 1 || v > (i64)BATCH) return fail(SSSP_ERR_INVALID_ARGUMENT, "claim max in [1,%u]", BATCH);
      g->p_claim = v;
      return SSSP_OK;
  }
  return fail(SSSP_ERR_INVALID_ARGUMENT, "unknown parameter %d", (int)p);
}

// ------------------------------------------------------------- symmetry --
template <int NF>
static sssp_status radix_pass(sssp_graph_t g, Fields<NF>& a, Fields<NF>& b, int kf, i64 n, int sh,
                              u32* hist, u32* tmp);
static int bits_for(u64 maxv);

extern "C" sssp_status sssp_is_symmetric(sssp_graph_t g, int* out) {
  NvtxRange nvtx_("sssp_is_symmetric");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
  if (!(g->pro_flags & SSSP_PRO_WEIGHT))
    return fail(SSSP_ERR_INVALID_STATE, "the symmetry check needs weight-sorted adjacencies (sssp_reorder)");
  if (g->sym_state < 0) {
    DeviceGuard dg(g->device);
    cudaStream_t s = g->stream;
    u32* flag = nullptr;
    u32 h = 0;
    CU(cudaMallocAsync(&flag, sizeof(u32), s));
    CU(cudaMemsetAsync(flag, 0, sizeof(u32), s));
    const int vb = std::max(1, bits_for((u64)(g->V - 1))), wb = bits_for(g->maxw_bits);
    bool sorted_done = false;
    if (g->A > 0 && 2 * vb + wb <= 64) {
      // sort-based: transposed keys, the PRO radix passes, one compare (falls back to the
      // per-run binary searches below if the temporaries do not fit)
      const i64 A = g->A, ntiles = (A + RS_TILE - 1) / RS_TILE;
      u32 *f[4] = {}, *hist = nullptr, *tmp = nullptr;
      bool ok = true;
      for (int i = 0; i < 4 && ok; ++i) ok = dalloc(&f[i], sizeof(u32) * A) == cudaSuccess;
      ok = ok && dalloc(&hist, sizeof(u32) * 256 * ntiles) == cudaSuccess;
      ok = ok && dalloc(&tmp, sizeof(u32) * scan_tmp_elems(256 * ntiles)) == cudaSuccess;
      if (ok) {
        const SymPack pk{vb, wb};
        const unsigned nbv = (unsigned)std::min<i64>((g->V + 7) / 8, (i64)g->num_sms * 64);
        k_sym_keys<<<nbv, 256, 0, s>>>(g->rowp, g->arcs, g->V, pk, f[0], f[1]);
        Fields<2> a{{f[0], f[1]}}, b{{f[2], f[3]}};
        for (int sh = 0; sh < 2 * vb + wb && !st; sh += 8) st = radix_pass<2>(g, a, b, sh >= 32 ? 1 : 0, A, sh & 31, hist, tmp);
        if (!st) k_sym_compare<<<nbv, 256, 0, s>>>(g->rowp, g->arcs, g->V, pk, a.f[0], a.f[1], flag);
        CU(cudaGetLastError());
        cudaStreamSynchronize(s);  // before the temporaries are freed
        sorted_done = !st;
      }
      cudaGetLastError();
      for (u32* x : {f[0], f[1], f[2], f[3], hist, tmp})
        if (x) dfree(x);
      if (st) return st;
    }
    if (g->A > 0 && !sorted_done) {
      const i64 nb = std::min<i64>((g->A + SYM_PER_BLOCK - 1) / SYM_PER_BLOCK, (i64)g->num_sms * 16);
      k_check_symmetric<<<(unsigned)nb, 256, 0, s>>>(g->rowp, g->arcs, g->V, g->A, flag);
      CU(cudaGetLastError());
    }
    CU(cudaMemcpyAsync(&h, flag, sizeof(u32), cudaMemcpyDeviceToHost, s));
    CU(cudaFreeAsync(flag, s));
    CU(cudaStreamSynchronize(s));
    g->sym_state = h ? 0 : 1;
  }
  *out = g->sym_state;
  return SSSP_OK;
}

// --------------------------------------------------------------- reorder --
template <int NF>
static sssp_status radix_pass(sssp_graph_t g, Fields<NF>& a, Fields<NF>& b, int kf, i64 n, int sh,
                              u32* hist, u32* tmp) {
  cudaStream_t s = g->stream;
  const u32 ntiles = (u32)((n + RS_TILE - 1) / RS_TILE);
  k_rs_hist<<<ntiles, RS_THREADS, 0, s>>>(a.f[kf], n, sh, hist, ntiles);
  scan_exclusive_rec<u32>(hist, hist, (i64)256 * ntiles, tmp, s);
  const size_t smem = (size_t)NF * RS_TILE * sizeof(u32);
  static bool attr_set = false;  // per NF instantiation
  if (!attr_set) {
    CU(cudaFuncSetAttribute(k_rs_scatter_smem<NF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr_set = true;
  }
  k_rs_scatter_smem<NF><<<ntiles, RS_THREADS, smem, s>>>(a, b, kf, n, sh, hist, ntiles);
  std::swap(a, b);
  CU(cudaGetLastError());
  return SSSP_OK;
}

static int bits_for(u64 maxv) {
  int b = 0;
  while (b < 64 && (maxv >> b) != 0) ++b;
  return b;
}

extern "C" sssp_status sssp_reorder_ex(sssp_graph_t g, unsigned flags) {
  NvtxRange nvtx_("sssp_reorder");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (flags & ~(SSSP_PRO_DEGREE | SSSP_PRO_WEIGHT)) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad PRO flags 0x%x", flags);
  if ((flags & ~g->pro_flags) == 0) return SSSP_OK;  // idempotent
  if (g->pro_flags != 0)
    return fail(SSSP_ERR_INVALID_STATE, "graph already reordered with flags 0x%x", g->pro_flags);
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  const i64 V = g->V, A = g->A;
  const bool deg = flags & SSSP_PRO_DEGREE, wsort = flags & SSSP_PRO_WEIGHT;
  // Every temporary is allocated before the timed window and freed after it, with
  // plain cudaMalloc (one-off, ~24 B per arc: not worth keeping in a stream pool),
  // and no host round trip happens inside the window: reorder_ms is device time.
  const i64 nmax = std::max<i64>(std::max(V, A), 1);
  const i64 ntiles_max = (nmax + RS_TILE - 1) / RS_TILE;
  const i64 hist_n = 256 * ntiles_max;
  const u32 nh_cap = (u32)(A / EXPAND_HUB + 1);
  std::vector<void*> temps;
  auto alloc = [&](void** ptr, size_t bytes) -> cudaError_t {
    cudaError_t e = dalloc(ptr, std::max<size_t>(bytes, 4));
    if (e == cudaSuccess) temps.push_back(*ptr);
    return e;
  };
  auto free_all = [&]() {
    for (void* t : temps) dfree(t);
    temps.clear();
  };
  u32 *hist = nullptr, *tmp = nullptr, *f[6] = {}, *dmax = nullptr, *key0 = nullptr, *key1 = nullptr,
      *id1 = nullptr, *hubs = nullptr, *cst = nullptr, *ctmp = nullptr;
  u64 *ndeg = nullptr, *stmp = nullptr;
  {
    cudaError_t e = cudaSuccess;
    auto A_ = [&](cudaError_t x) {
      if (e == cudaSuccess) e = x;
    };
    A_(alloc((void**)&hist, sizeof(u32) * hist_n));
    A_(alloc((void**)&tmp, sizeof(u32) * scan_tmp_elems(hist_n)));
    A_(alloc((void**)&dmax, sizeof(u32)));
    if (deg) {
      if (!g->new2old) A_(dalloc(&g->new2old, sizeof(u32) * V));
      if (!g->old2new) A_(dalloc(&g->old2new, sizeof(u32) * V));
      A_(alloc((void**)&key0, sizeof(u32) * V));
      A_(alloc((void**)&key1, sizeof(u32) * V));
      A_(alloc((void**)&id1, sizeof(u32) * V));
      A_(alloc((void**)&ndeg, sizeof(u64) * (V + 1)));
      A_(alloc((void**)&stmp, sizeof(u64) * scan_tmp_elems(V)));
    }
    if (A > 0) {
      for (int i = 0; i < 6; ++i) A_(alloc((void**)&f[i], sizeof(u32) * A));
      A_(alloc((void**)&hubs, sizeof(u32) * (nh_cap + 1)));
      A_(alloc((void**)&cst, sizeof(u32) * (nh_cap + 1)));
      A_(alloc((void**)&ctmp, sizeof(u32) * scan_tmp_elems(nh_cap + 1)));
    }
    if (e != cudaSuccess) {
      free_all();
      cudaGetLastError();
      return fail(e == cudaErrorMemoryAllocation ? SSSP_ERR_OUT_OF_MEMORY : SSSP_ERR_CUDA,
                  "reorder temporaries: %s", cudaGetErrorString(e));
    }
  }
#define CT(call)                \
  do {                          \
    cudaError_t e_ = (call);    \
    if (e_ != cudaSuccess) {    \
      free_all();               \
      g->sticky_cuda = true;    \
      return fail(SSSP_ERR_CUDA, "reorder: %s: %s", #call, cudaGetErrorString(e_)); \
    }                           \
  } while (0)
  CT(cudaMemsetAsync(dmax, 0, sizeof(u32), s));
  CT(cudaEventRecord(g->ev[2], s));
  if (deg) {
    // a1: stable radix sort of (maxdeg - deg, id) -> new2old (desc degree, asc id). maxdeg <= A,
    // so bits_for(A) passes cover it without reading maxdeg back to the host.
    k_max_degree<<<grid_for(V), 256, 0, s>>>(g->rowp, V, dmax);
    k_degree_keys<<<grid_for(V), 256, 0, s>>>(g->rowp, V, dmax, key0, g->new2old);
    Fields<2> a{{key0, g->new2old}}, b{{key1, id1}};
    const int nb = std::max(1, bits_for((u64)A));
    for (int sh = 0; sh < nb; sh += 8) {
      if ((st = radix_pass<2>(g, a, b, 0, V, sh, hist, tmp))) {
        free_all();
        return st;
      }
    }
    if (a.f[1] != g->new2old) CT(cudaMemcpyAsync(g->new2old, a.f[1], sizeof(u32) * V, cudaMemcpyDeviceToDevice, s));
    k_invert_perm<<<grid_for(V), 256, 0, s>>>(g->new2old, g->rowp, V, g->old2new, ndeg);
    scan_exclusive_rec<u64>(ndeg, ndeg, V, stmp, s);  // new row starts
    CT(cudaGetLastError());
  }
  if (A > 0) {
    // a2+a3: one stable LSD radix sort of all arcs by (new src, w, new dst)
    // arcs of vertices with <= EXPAND_HUB arcs: warp-flattened; hubs: 4096-arc
    // chunks over all blocks. The hub count is bounded by A / EXPAND_HUB, so
    // the chunk scan runs over that capacity with no host round trip.
    CT(cudaMemsetAsync(hubs + nh_cap, 0, sizeof(u32), s));
    // (src', w, dst') as one 64-bit key when src', w and dst' fit (S = w's end rounded up to
    // whole 8-bit digits): each radix pass then moves 8 bytes per arc instead of 12
    const int vb = std::max(1, bits_for((u64)(V - 1))), wb = bits_for(g->maxw_bits);
    const int S = (vb + wb + 7) / 8 * 8;
    ArcPack pk{(S + vb <= 64) ? 1 : 0, vb, S};
    k_list_hubs<<<grid_for(V), 256, 0, s>>>(g->rowp, V, hubs, hubs + nh_cap);
    k_expand_arcs_flat<<<grid_for(V), 256, 0, s>>>(g->rowp, g->arcs, V, deg ? g->old2new : nullptr,
                                                   f[0], f[1], f[2], pk);
    k_hub_chunks<<<(nh_cap + 256) / 256, 256, 0, s>>>(g->rowp, hubs, hubs + nh_cap, nh_cap, cst);
    scan_exclusive_rec<u32>(cst, cst, (i64)nh_cap + 1, ctmp, s);
    k_expand_hubs<<<g->num_sms * 8, 256, 0, s>>>(g->rowp, g->arcs, hubs, nh_cap, cst,
                                                 deg ? g->old2new : nullptr, f[0], f[1], f[2], pk);
    CT(cudaGetLastError());
    if (pk.packed) {
      // LSD over the key's digits: (w, dst') when weight-sorting, then src' (stable)
      Fields<2> a{{f[0], f[1]}}, b{{f[3], f[4]}};
      const int from = wsort ? 0 : S;
      for (int sh = from; sh < S + vb && !st; sh += 8) st = radix_pass<2>(g, a, b, sh >= 32 ? 1 : 0, A, sh & 31, hist, tmp);
      if (st) {
        free_all();
        return st;
      }
      k_unpack_sorted<<<grid_for(A), 256, 0, s>>>(a.f[0], a.f[1], A, pk, g->arcs);
    } else {
      Fields<3> a{{f[0], f[1], f[2]}}, b{{f[3], f[4], f[5]}};
      auto pass3 = [&](int kf, int sh) { return radix_pass<3>(g, a, b, kf, A, sh, hist, tmp); };
      if (wsort) {
        for (int sh = 0; sh < vb && !st; sh += 8) st = pass3(2, sh);
        for (int sh = 0; sh < wb && !st; sh += 8) st = pass3(1, sh);
      }
      if (deg || wsort)
        for (int sh = 0; sh < vb && !st; sh += 8) st = pass3(0, sh);
      if (st) {
        free_all();
        return st;
      }
      k_pack_sorted<<<grid_for(A), 256, 0, s>>>(a.f[1], a.f[2], A, g->arcs);
    }
    CT(cudaGetLastError());
  }
  if (deg) k_set_rowp<<<grid_for(V + 1), 256, 0, s>>>(ndeg, V, A, g->rowp);
  CT(cudaEventRecord(g->ev[3], s));
  CT(cudaGetLastError());
  if (deg) {
    g->h_old2new.resize(V);
    CT(cudaMemcpyAsync(g->h_old2new.data(), g->old2new, sizeof(u32) * V, cudaMemcpyDeviceToHost, s));
  }
  CT(cudaStreamSynchronize(s));
  free_all();
#undef CT
  g->pro_flags |= flags;
  g->heavy_valid = false;
  g->rowc_valid = false;
  g->rowc_lv_valid = false;
  g->hubdist_bits = 0xFFFFFFFFu;
  g->hub_ids_cached = -1;
  g->sym_state = -1;
  g->v_nz = -1;
  g->have_result = false;
  g->reorder_timed = true;
  return SSSP_OK;
}

extern "C" sssp_status sssp_reorder(sssp_graph_t g) {
  return sssp_reorder_ex(g, SSSP_PRO_DEGREE | SSSP_PRO_WEIGHT);
}

// ------------------------------------------------------------------ run ---
struct DeltaParams {
  u32 delta_u, delta_bits;
  float inv;
  double ahead;  // max weight / Delta (buckets a heavy push can skip ahead)
  AdaptInit ai;  // fixed Delta: mode 0, one ring slot per bucket
};

// Adaptive Delta (NEXT-1): ring slots become fine slots of width g = Delta_0 / 4
// (u32: max(1, floor(Delta_0 / 4))); a bucket spans m in [Delta_0/4, 4 Delta_0] / g
// of them (at most 16), and delta_u / inv / delta_bits describe g instead of Delta.
static void adapt_params(sssp_graph_t g, int mode, DeltaParams* dp) {
  dp->ai = AdaptInit{0u, 1.f, 1u, 1u, 1u, 0u, 0u};
  if (!mode || dp->delta_bits == 0xFFFFFFFFu || (g->wtype == SSSP_WEIGHT_F32 && dp->inv == 0.f)) return;
  double d0;
  if (g->wtype == SSSP_WEIGHT_U32) {
    const u32 D = dp->delta_u, gu = std::max<u32>(1u, D / 4);
    dp->delta_u = dp->delta_bits = gu;
    d0 = (double)D / gu;
    dp->ahead = (double)g->maxw_bits / gu;
  } else {
    float df;
    memcpy(&df, &dp->delta_bits, 4);
    const float gf = df * 0.25f;  // exact (power-of-two scale) unless subnormal
    if (!(gf > 0.f) || gf * 4.f != df) return;
    memcpy(&dp->delta_bits, &gf, 4);
    dp->inv = (float)(1.0 / (double)gf);
    d0 = 4.0;
    dp->ahead *= 4.0;
  }
  const u32 mmin = std::max<u32>(1u, (u32)std::lrint(d0 / 4)), mmax = std::min<u32>(16u, (u32)std::lrint(4 * d0));
  const u32 m0 = std::min(std::max((u32)std::lrint(d0), mmin), mmax);
  u32 l = 0;
  while ((1u << l) < m0) ++l;
  dp->ai = AdaptInit{(u32)mode, (float)d0, m0, mmin, mmax, l, 0u};
}

static sssp_status delta_params(sssp_graph_t g, double delta, DeltaParams* dp) {
  dp->ai = AdaptInit{0u, 1.f, 1u, 1u, 1u, 0u, 0u};
  if (std::isnan(delta) || delta <= 0.0) return fail(SSSP_ERR_INVALID_ARGUMENT, "delta must be > 0 (got %g)", delta);
  if (g->wtype == SSSP_WEIGHT_U32) {
    double c = std::ceil(delta);
    dp->delta_u = (std::isinf(delta) || c >= 4294967295.0) ? 0xFFFFFFFFu : (u32)std::max(1.0, c);
    dp->delta_bits = dp->delta_u;
    dp->inv = 0.f;
    dp->ahead = (double)g->maxw_bits / dp->delta_u;
  } else {
    float df = (float)delta;
    if (df <= 0.f) return fail(SSSP_ERR_INVALID_ARGUMENT, "delta rounds to 0 in binary32");
    u32 bits;
    memcpy(&bits, &df, 4);
    dp->delta_bits = bits;
    dp->delta_u = 1;
    dp->inv = std::isinf(df) ? 0.f : (float)(1.0 / (double)df);
    float mw;
    memcpy(&mw, &g->maxw_bits, 4);
    dp->ahead = std::isinf(df) ? 0.0 : (double)mw / (double)df;
  }
  return SSSP_OK;
}

static sssp_status ensure_run_buffers(sssp_graph_t g, u32 K, u32 cap) {
  cudaStream_t s = g->stream;
  const u32 hub_cap = (u32)std::min<i64>(g->A / 2048 + 4096, 0x7FFFFFFF);
  if (K > g->K_alloc || cap != g->cap_alloc) {
    if (g->items) CU(cudaStreamSynchronize(s));  // earlier runs may still read the old queues
    if (g->items) CU(dfree(g->items));
    if (g->sc) CU(dfree(g->sc));
    if (g->p2o) CU(dfree(g->p2o));
    g->items = nullptr;
    g->sc = nullptr;
    g->p2o = nullptr;
    CU(dalloc(&g->items, sizeof(u64) * (size_t)K * cap));
    CU(dalloc(&g->p2o, sizeof(u32) * (((size_t)cap + 1) & ~(size_t)1) + sizeof(uint2) * (size_t)cap));
    CU(dalloc(&g->sc, sizeof(SlotCtl) * K));
    CU(cudaMemsetAsync(g->sc, 0, sizeof(SlotCtl) * K, s));
    g->K_alloc = K;
    g->cap_alloc = cap;
    g->need_full_reset = true;
  }
  if (!g->hub_items) {
    CU(dalloc(&g->hub_items, sizeof(u64) * hub_cap));
    g->hub_cap = hub_cap;
    g->need_full_reset = true;
  }
  if (g->need_full_reset) {
    CU(cudaMemsetAsync(g->items, 0xFF, sizeof(u64) * (size_t)g->K_alloc * g->cap_alloc, s));
    CU(cudaMemsetAsync(g->hub_items, 0xFF, sizeof(u64) * g->hub_cap, s));
    g->need_full_reset = false;
  }
  return SSSP_OK;
}

typedef void (*ds_kernel_t)(Params);
static ds_kernel_t pick_kernel(bool f32, bool pro, bool abl) {
  if (abl) {
    if (f32) return pro ? k_delta_step<true, true, true> : k_delta_step<true, false, true>;
    return pro ? k_delta_step<false, true, true> : k_delta_step<false, false, true>;
  }
  if (f32) return pro ? k_delta_step<true, true, false> : k_delta_step<true, false, false>;
  return pro ? k_delta_step<false, true, false> : k_delta_step<false, false, false>;
}

static sssp_status launch_run(sssp_graph_t g, u32 src_internal, const DeltaParams& dp, bool timed) {
  cudaStream_t s = g->stream;
  const bool pro = (g->pro_flags & SSSP_PRO_WEIGHT) != 0;
  const bool f32 = g->wtype == SSSP_WEIGHT_F32;
  // a4: heavy offsets for this Delta (only with weight-sorted adjacencies)
  if (pro && (!g->heavy_valid || g->heavy_bits != dp.delta_bits)) {
    k_heavy_offsets<<<grid_for(g->V), 256, 0, s>>>(g->rowp, g->arcs, g->V, dp.delta_bits);
    CU(cudaGetLastError());
    g->heavy_valid = true;
    g->heavy_bits = dp.delta_bits;
    g->rowc_valid = false;
  }
  if (!g->rowc_valid) {
    k_make_rowc<<<grid_for(g->V + 1), 256, 0, s>>>(g->rowp, g->V, g->rowc);
    CU(cudaGetLastError());
    g->rowc_valid = true;
  }
  // ring size: enough slots for the farthest heavy push (+ the recycled slot)
  u32 K = (u32)g->p_ring;
  if (K == 0) {
    double need = std::ceil(dp.ahead) + dp.ai.mmax + 2.0;
    K = 8;
    while (K < need && K < (dp.ai.mode ? 64u : 32u)) K <<= 1;
  }
  u32 cap = (u32)g->p_cap;
  if (cap == 0)  // 2.5 V: far buckets collect repeated improvements; adaptive: 4x the slots, 1.5 V each
    cap = (u32)std::min<i64>((dp.ai.mode ? g->V + g->V / 2 : 2 * g->V + g->V / 2) + 65536, 0x7FFFFFFF);
  sssp_status st = ensure_run_buffers(g, K, cap);
  if (st) return st;
  g->K_used = K;
  if (g->l2_window_bytes < 0) {
    // Persisting L2 set-aside for dist[] (4 B per vertex). The set-aside is a
    // device-wide limit; it is only ever raised, never lowered.
    g->l2_window_bytes = 0;
    int max_persist = 0, max_window = 0;
    cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, g->device);
    cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, g->device);
    const i64 want = (i64)sizeof(u32) * g->V;
    if (g->p_l2 && max_persist > 0 && max_window > 0) {
      size_t cur = 0;
      cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
      const size_t set_aside = (size_t)std::min<i64>(want, max_persist);
      if (cur < set_aside) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, set_aside);
      cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
      g->l2_window_bytes = std::min<i64>(want, max_window);
      g->l2_hit_ratio = (float)std::min(1.0, (double)cur / (double)g->l2_window_bytes);
    }
    cudaGetLastError();
  }
  const bool adapt = dp.ai.mode != 0;
  if (adapt && pro && (!g->rowc_lv_valid || g->rowc_lv_g != dp.delta_bits)) {
    // heavy offsets for the light levels g << l (u32) / g * 2^l (f32), l = 0..4
    if (!g->rowc_lv) CU(dalloc(&g->rowc_lv, sizeof(uint2) * 5 * (size_t)(g->V + 1)));
    for (u32 l = 0; l < 5; ++l) {
      const u32 th = f32 ? dp.delta_bits + (l << 23) : dp.delta_bits << l;
      k_heavy_offsets<<<grid_for(g->V), 256, 0, s>>>(g->rowp, g->arcs, g->V, th);
      k_make_rowc<<<grid_for(g->V + 1), 256, 0, s>>>(g->rowp, g->V, g->rowc_lv + (size_t)l * (g->V + 1));
      g->heavy_bits = th;
    }
    CU(cudaGetLastError());
    g->rowc_lv_valid = true;
    g->rowc_lv_g = dp.delta_bits;
    g->rowc_valid = false;
  }
  ds_kernel_t kern = pick_kernel(f32, pro, g->p_adwl == 0 || g->p_sync != 0 || adapt || g->p_p2eb >= 0);
  int per_sm = 0;
  CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, DS_THREADS, 0));
  if (per_sm < 1) return fail(SSSP_ERR_INTERNAL, "persistent kernel cannot be resident");
  if (g->p_ctas > 0) per_sm = std::min<int>(per_sm, (int)g->p_ctas);
  g->grid_ctas = per_sm * g->num_sms;
  Params p;
  p.rowc = (adapt && pro) ? g->rowc_lv : g->rowc;
  p.arcs = g->arcs;
  p.dist = g->dist;
  p.xd = g->xd;
  p.ctl = g->ctl;
  p.sc = g->sc;
  p.items = g->items;
  p.hub_items = g->hub_items;
  p.stats = g->stats;
  p.trace = g->trace;
  p.V = (u32)g->V;
  p.K = K;
  p.kmask = K - 1;
  p.cap = cap;
  p.hub_cap = g->hub_cap;
  p.delta_u = dp.delta_u;
  p.inv_delta = dp.inv;
  p.delta_bits = dp.delta_bits;
  p.claim_max = (u32)g->p_claim;
  // CTA-local chase only while no arc is heavy (phase 2 then needs no settled list); auto
  // (1) also asks for a sparse graph (A <= 8 V: thin, long frontiers as on road networks),
  // where the chase cuts per-hop latency; on dense graphs it measured slower (C1 2x)
  if (g->p_local && !adapt && !g->p_sync && g->maxw_bits < dp.delta_bits && (g->p_local == 2 || g->A <= 8 * g->V))
    p.claim_max |= LOCAL_CHASE | ((u32)g->p_local_lim << LOCAL_LIM_SHIFT);
  p.p2o = g->p2o;
  p.flags = (g->p_adwl ? 1u : 0u) | (g->p_sync ? 2u : 0u);
  // edge-balanced phase 2 (not in the static thread-per-vertex ablation)
  if (g->p_p2eb >= 0 && g->p_adwl) p.flags |= 4u | ((u32)std::min<i64>(g->p_p2eb, 0x7FFFFF) << 8);
  if (adapt) p.flags |= (dp.ai.mode == 2 ? 16u : 8u) | (pro ? 64u : 0u);
  if (f32) p.flags |= 32u;
  if (g->p_pull && pro && !adapt && (f32 ? dp.inv != 0.f : dp.delta_u != 0xFFFFFFFFu)) {  // symmetric, checked
    if (g->sym_state < 0) {
      int sym = 0;
      if ((st = sssp_is_symmetric(g, &sym))) return st;
    }
    if (g->sym_state == 0) return fail(SSSP_ERR_INVALID_STATE, "pull phases need a symmetric graph; this one is not");
    p.flags |= 128u;
    if (f32) p.delta_u = dp.delta_bits;  // pull_phase needs Delta itself (bucket_of uses inv_delta)
  }
  // The first pull scans ids [0, first_n): with PRO's degree order the isolated vertices
  // (never reached, unless the source) are the id tail, found once per reorder.
  if ((g->pro_flags & SSSP_PRO_DEGREE) && g->v_nz < 0) {
    u32 lo = 0, hi = (u32)g->V;  // first id with degree 0 (degrees non-increasing)
    longlong2 r[2];
    while (lo < hi) {
      const u32 mid = lo + (hi - lo) / 2;
      CU(cudaMemcpy(r, g->rowp + mid, 2 * sizeof(longlong2), cudaMemcpyDeviceToHost));
      if (r[1].x > r[0].x) lo = mid + 1; else hi = mid;
    }
    g->v_nz = lo;
  }
  AdaptInit ai = dp.ai;
  ai.first_n = (g->pro_flags & SSSP_PRO_DEGREE) ? (u32)std::max<i64>(g->v_nz, (i64)src_internal + 1) : (u32)g->V;
  // fixed Delta, asynchronous phase 1 only; auto (-1): on dense graphs (A > 8 V). On sparse,
  // road-like ones the remaining vertices form long chains that label-correcting re-relaxes
  // (C2: 6 % slower with it).
  const i64 bf = g->p_bf >= 0 ? g->p_bf : (g->A > 8 * g->V ? (i64)SSSP_BF_TAIL_DEFAULT : 0);
  ai.bf_t = (ai.mode != 0 || g->p_sync) ? 0u : (u32)bf;
  // a5: init (Alg. 2 l.1-3)
  k_fill_u32<<<grid_for(g->V), 256, 0, s>>>(g->dist, g->V, f32 ? 0x7F800000u : 0xFFFFFFFFu);
  k_seed<<<1, 64, 0, s>>>(p, src_internal, ai);
  CU(cudaGetLastError());
  cudaEvent_t e0, e1;
  for (int i = 0; i < 2; ++i) {
    cudaEvent_t e;
    if (g->ev_pool.empty()) {
      CU(cudaEventCreate(&e));
    } else {
      e = g->ev_pool.back();
      g->ev_pool.pop_back();
    }
    (i ? e1 : e0) = e;
  }
  g->ev_pending.emplace_back(e0, e1);
  CU(cudaEventRecord(e0, s));
  if (timed) CU(cudaEventRecord(g->ev[0], s));
  // Cooperative launch (all CTAs co-resident: the grid barrier and the work
  // queues need forward progress) with an L2 access-policy window that keeps
  // dist[] persisting in L2 while arcs and queue entries stream through.
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(g->grid_ctas);
  cfg.blockDim = dim3(DS_THREADS);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute attrs[2];
  int na = 0;
  attrs[na].id = cudaLaunchAttributeCooperative;
  attrs[na].val.cooperative = 1;
  ++na;
  if (g->l2_window_bytes > 0) {
    attrs[na].id = cudaLaunchAttributeAccessPolicyWindow;
    attrs[na].val.accessPolicyWindow.base_ptr = g->dist;
    attrs[na].val.accessPolicyWindow.num_bytes = (size_t)g->l2_window_bytes;
    attrs[na].val.accessPolicyWindow.hitRatio = g->l2_hit_ratio;
    attrs[na].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    attrs[na].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    ++na;
  }
  cfg.attrs = attrs;
  cfg.numAttrs = na;
  CU(cudaLaunchKernelEx(&cfg, kern, p));
  if (timed) CU(cudaEventRecord(g->ev[1], s));
  CU(cudaEventRecord(e1, s));
  g->run_timed = timed;
  return SSSP_OK;
}

extern "C" sssp_status sssp_run(sssp_graph_t g, int64_t source, double delta) {
  NvtxRange nvtx_("sssp_run");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (source < 0 || source >= g->V) return fail(SSSP_ERR_INVALID_ARGUMENT, "source %lld out of range", (long long)source);
  DeltaParams dp;
  if ((st = delta_params(g, delta, &dp))) return st;
  adapt_params(g, (int)g->p_adapt, &dp);
  DeviceGuard dg(g->device);
  const u32 src = g->h_old2new.empty() ? (u32)source : g->h_old2new[source];
  g->have_result = false;
  if ((st = launch_run(g, src, dp, true))) return st;
  g->have_result = true;
  return SSSP_OK;
}

// ------------------------------------------------------------ results -----
// Errors of every persistent run since the last report: the kernel ORs its err word into
// Ctl::err_acc as it exits (k_seed never clears err_acc), so a run whose errors nobody has
// read yet is never lost. Synchronises the handle's stream, reports, clears.
static sssp_status take_run_errors(sssp_graph_t g) {
  u32 e = 0;
  u32* acc = &g->ctl->err_acc;
  CU(cudaMemcpyAsync(&e, acc, sizeof e, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaMemsetAsync(acc, 0, sizeof e, g->stream));
  CU(cudaStreamSynchronize(g->stream));
  if (e & ERR_INTERNAL) {
    g->need_full_reset = true;
    return fail(SSSP_ERR_INTERNAL, "scheduler queue overflow");
  }
  if (e & ERR_OVERFLOW) return fail(SSSP_ERR_OVERFLOW, "u32 distance overflow");
  return SSSP_OK;
}

extern "C" sssp_status sssp_distances(sssp_graph_t g, void* out, sssp_memory where) {
  NvtxRange nvtx_("sssp_distances");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
  if (where != SSSP_MEM_HOST && where != SSSP_MEM_DEVICE) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad memory kind");
  if (!g->have_result) return fail(SSSP_ERR_INVALID_STATE, "no successful sssp_run since create/reorder");
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  u32* dst = (u32*)out;
  bool staged = false;
  if (where == SSSP_MEM_HOST) {
    // Pinned, device-mapped host memory (cudaHostAlloc / torch pin_memory) is
    // written directly by the output gather over the host link: a8 fused with
    // the D2H copy. Pageable memory goes through a persistent device staging
    // buffer and one cudaMemcpyAsync (no per-call allocation).
    cudaPointerAttributes pa;
    if (cudaPointerGetAttributes(&pa, out) == cudaSuccess && pa.type == cudaMemoryTypeHost &&
        pa.devicePointer != nullptr) {
      dst = (u32*)pa.devicePointer;
    } else {
      cudaGetLastError();
      if (!g->out_tmp) CU(dalloc(&g->out_tmp, sizeof(u32) * g->V));
      staged = true;
    }
  }
  k_output<<<grid_for(g->V), 256, 0, s>>>(g->dist, g->old2new, g->V, staged ? g->out_tmp : dst);
  CU(cudaGetLastError());
  if (staged) CU(cudaMemcpyAsync(out, g->out_tmp, sizeof(u32) * g->V, cudaMemcpyDeviceToHost, s));
  return take_run_errors(g);
}

extern "C" sssp_status sssp_distances_async(sssp_graph_t g, void* out, sssp_memory where) {
  NvtxRange nvtx_("sssp_distances_async");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
  if (where != SSSP_MEM_HOST && where != SSSP_MEM_DEVICE) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad memory kind");
  if (!g->have_result) return fail(SSSP_ERR_INVALID_STATE, "no successful sssp_run since create/reorder");
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  if (where == SSSP_MEM_DEVICE) {  // a8 straight into the caller's device buffer
    k_output<<<grid_for(g->V), 256, 0, s>>>(g->dist, g->old2new, g->V, (u32*)out);
    CU(cudaGetLastError());
    return SSSP_OK;
  }
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, out) != cudaSuccess || pa.type != cudaMemoryTypeHost) {
    cudaGetLastError();
    return fail(SSSP_ERR_INVALID_ARGUMENT, "sssp_distances_async needs pinned host memory");
  }
  if (!g->d2h) {
    CU(cudaStreamCreateWithFlags(&g->d2h, cudaStreamNonBlocking));
    CU(cudaEventCreateWithFlags(&g->ev_ran, cudaEventDisableTiming));
    for (auto& e : g->ev_out) CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  const int j = g->stage_next;
  g->stage_next ^= 1;
  if (!g->stage[j]) CU(dalloc(&g->stage[j], sizeof(u32) * g->V));
  if (g->stage_used[j]) CU(cudaStreamWaitEvent(s, g->ev_out[j], 0));  // its previous copy is done
  // a8 into the staging buffer (HBM speed, run stream), then the copy engine moves it to
  // the host on d2h while the next sssp_run computes
  k_output<<<grid_for(g->V), 256, 0, s>>>(g->dist, g->old2new, g->V, g->stage[j]);
  CU(cudaGetLastError());
  CU(cudaEventRecord(g->ev_ran, s));
  CU(cudaStreamWaitEvent(g->d2h, g->ev_ran, 0));
  CU(cudaMemcpyAsync(out, g->stage[j], sizeof(u32) * g->V, cudaMemcpyDeviceToHost, g->d2h));
  CU(cudaEventRecord(g->ev_out[j], g->d2h));
  g->stage_used[j] = true;
  return SSSP_OK;
}

extern "C" sssp_status sssp_wait(sssp_graph_t g) {
  NvtxRange nvtx_("sssp_wait");
  sssp_status st = check_handle(g);
  if (st) return st;
  DeviceGuard dg(g->device);
  CU(cudaStreamSynchronize(g->stream));
  if (g->d2h) CU(cudaStreamSynchronize(g->d2h));
  return take_run_errors(g);
}

extern "C" sssp_status sssp_run_batch(sssp_graph_t g, const int64_t* sources, int64_t n, double delta,
                                      void* out_dev, int64_t ld) {
  NvtxRange nvtx_("sssp_run_batch");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (n < 0 || (n > 0 && (!sources || !out_dev)) || ld < g->V)
    return fail(SSSP_ERR_INVALID_ARGUMENT, "bad batch arguments");
  DeltaParams dp;
  if ((st = delta_params(g, delta, &dp))) return st;
  adapt_params(g, (int)g->p_adapt, &dp);
  for (i64 i = 0; i < n; ++i)
    if (sources[i] < 0 || sources[i] >= g->V) return fail(SSSP_ERR_INVALID_ARGUMENT, "source[%lld] out of range", (long long)i);
  DeviceGuard dg(g->device);
  std::vector<u32> src(n);
  for (i64 i = 0; i < n; ++i) src[i] = g->h_old2new.empty() ? (u32)sources[i] : g->h_old2new[sources[i]];
  for (i64 i = 0; i < n; ++i) {
    g->have_result = false;
    if ((st = launch_run(g, src[i], dp, i == n - 1))) return st;
    g->have_result = true;
    k_output<<<grid_for(g->V), 256, 0, g->stream>>>(g->dist, g->old2new, g->V, (u32*)out_dev + (size_t)i * ld);
    CU(cudaGetLastError());
  }
  return take_run_errors(g);  // synchronises: errors of any of the n runs
}

// NEXT-4: up to 32 sources per persistent launch (multi_source.cuh).
extern "C" sssp_status sssp_run_multi(sssp_graph_t g, const int64_t* sources, int64_t n, double delta,
                                      void* out_dev, int64_t ld) {
  NvtxRange nvtx_("sssp_run_multi");
  sssp_status st = check_handle(g);
  if (st) return st;
  if (n < 0 || (n > 0 && (!sources || !out_dev)) || ld < g->V)
    return fail(SSSP_ERR_INVALID_ARGUMENT, "bad batch arguments");
  DeltaParams dp;
  if ((st = delta_params(g, delta, &dp))) return st;
  for (i64 i = 0; i < n; ++i)
    if (sources[i] < 0 || sources[i] >= g->V) return fail(SSSP_ERR_INVALID_ARGUMENT, "source[%lld] out of range", (long long)i);
  if (n == 0) return SSSP_OK;
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  const bool f32 = g->wtype == SSSP_WEIGHT_F32;
  if (!g->rowc_valid) {  // only the .x (row start) column is used here
    k_make_rowc<<<grid_for(g->V + 1), 256, 0, s>>>(g->rowp, g->V, g->rowc);
    CU(cudaGetLastError());
    g->rowc_valid = true;
  }
  u32 K = 8;
  while (K < std::ceil(dp.ahead) + 2.0 && K < 64) K <<= 1;
  const u32 cap = (u32)std::min<i64>(g->V + g->V / 2 + g->A / 128 + 65536, 0x7FFFFFFF);
  if (!g->ms_D) {
    CU(dalloc(&g->ms_D, sizeof(u32) * MS_LANES * (size_t)g->V));
    CU(dalloc(&g->ms_Q, sizeof(u32) * (size_t)g->V));
    CU(dalloc(&g->ms_ctl, sizeof(MCtl)));
    CU(cudaMemsetAsync(g->ms_ctl, 0, sizeof(MCtl), s));
    CU(dalloc(&g->ms_stats, sizeof(unsigned long long) * MST_N));
    CU(dalloc(&g->ms_src, sizeof(u32) * 2 * MS_LANES));
  }
  if (K > g->ms_K || cap > g->ms_cap) {
    if (g->ms_items) CU(cudaStreamSynchronize(s));
    if (g->ms_items) CU(dfree(g->ms_items));
    if (g->ms_sc) CU(dfree(g->ms_sc));
    g->ms_items = nullptr;
    g->ms_sc = nullptr;
    CU(dalloc(&g->ms_items, sizeof(u64) * (size_t)K * cap));
    CU(dalloc(&g->ms_sc, sizeof(SlotCtl) * K));
    CU(cudaMemsetAsync(g->ms_items, 0xFF, sizeof(u64) * (size_t)K * cap, s));
    CU(cudaMemsetAsync(g->ms_sc, 0, sizeof(SlotCtl) * K, s));
    g->ms_K = K;
    g->ms_cap = cap;
  }
  MParams p;
  p.rowc = g->rowc;
  p.arcs = g->arcs;
  p.D = g->ms_D;
  p.Q = g->ms_Q;
  p.ctl = g->ms_ctl;
  p.sc = g->ms_sc;
  p.items = g->ms_items;
  p.stats = g->ms_stats;
  p.shift = g->ms_src + MS_LANES;
  p.V = (u32)g->V;
  p.K = g->ms_K;
  p.kmask = g->ms_K - 1;
  p.cap = g->ms_cap;
  p.delta_u = dp.delta_u;
  p.inv_delta = dp.inv;
  p.f32 = f32 ? 1u : 0u;
  p.inf = f32 ? 0x7F800000u : 0xFFFFFFFFu;
  p.hub_ids = 0;
  p.hub_delay = (u32)g->p_hub_delay;
  if (g->p_hub_delay > 0 && !g->h_old2new.empty()) {  // degree-sorted ids: count degree > 1024
    if (g->hub_ids_cached < 0) {
      std::vector<longlong2> r(2);
      u32 lo = 0, hi = (u32)g->V;  // first id with degree <= 1024 (degrees non-increasing)
      while (lo < hi) {
        const u32 mid = lo + (hi - lo) / 2;
        CU(cudaMemcpy(r.data(), g->rowp + mid, 2 * sizeof(longlong2), cudaMemcpyDeviceToHost));
        if (r[1].x - r[0].x > 1024) lo = mid + 1; else hi = mid;
      }
      g->hub_ids_cached = lo;
    }
    p.hub_ids = (u32)g->hub_ids_cached;
  }
  int per_sm = 0;
  const void* mk = f32 ? (const void*)k_ms_step<true> : (const void*)k_ms_step<false>;
  CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mk, MS_THREADS, 0));
  if (per_sm < 1) return fail(SSSP_ERR_INTERNAL, "multi-source kernel cannot be resident");
  if (g->p_ctas > 0) per_sm = std::min<int>(per_sm, (int)g->p_ctas);
  const int grid = per_sm * g->num_sms;
  if (g->p_align && g->hubdist_bits != dp.delta_bits) {
    // Lane alignment: distances from the highest-degree vertex (one single-source run,
    // cached per graph; it replaces the last sssp_run result).
    u32 hub = 0;
    if (g->h_old2new.empty()) {
      std::vector<long long> rp(g->V + 1);
      std::vector<longlong2> tmp(g->V + 1);
      CU(cudaMemcpyAsync(tmp.data(), g->rowp, sizeof(longlong2) * (g->V + 1), cudaMemcpyDeviceToHost, s));
      CU(cudaStreamSynchronize(s));
      long long best = -1;
      for (i64 v = 0; v < g->V; ++v)
        if (tmp[v + 1].x - tmp[v].x > best) best = tmp[v + 1].x - tmp[v].x, hub = (u32)v;
    }  // degree-sorted (PRO): internal id 0 has the highest degree
    DeltaParams dh = dp;
    dh.ai = AdaptInit{0u, 1.f, 1u, 1u, 1u, 0u, 0u};
    g->have_result = false;
    u32 err_prev = 0;  // errors of earlier, not yet reported sssp_run calls survive this run
    CU(cudaMemcpyAsync(&err_prev, &g->ctl->err_acc, sizeof(u32), cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));
    if ((st = launch_run(g, hub, dh, false))) return st;
    g->h_hubdist.resize(g->V);
    CU(cudaMemcpyAsync(g->h_hubdist.data(), g->dist, sizeof(u32) * g->V, cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));
    // the alignment run's own errors are not the batch's (its keys only order the queue)
    CU(cudaMemcpy(&g->ctl->err_acc, &err_prev, sizeof(u32), cudaMemcpyHostToDevice));
    g->hubdist_bits = dp.delta_bits;
  }
  std::vector<u32> src(2 * MS_LANES, 0u);
  u32 err_all = 0;
  for (i64 g0 = 0; g0 < n; g0 += MS_LANES) {
    const u32 nn = (u32)std::min<i64>(MS_LANES, n - g0);
    for (u32 l = 0; l < nn; ++l)
      src[l] = g->h_old2new.empty() ? (u32)sources[g0 + l] : g->h_old2new[sources[g0 + l]];
    // key shift of lane l: M - d(hub, source l) (0 for unreachable sources / alignment off)
    std::fill(src.begin() + MS_LANES, src.end(), 0u);
    if (g->p_align && !g->h_hubdist.empty()) {
      if (f32) {
        float M = 0.f;
        for (u32 l = 0; l < nn; ++l) {
          float d;
          memcpy(&d, &g->h_hubdist[src[l]], 4);
          if (std::isfinite(d)) M = std::max(M, d);
        }
        for (u32 l = 0; l < nn; ++l) {
          float d, sh;
          memcpy(&d, &g->h_hubdist[src[l]], 4);
          sh = std::isfinite(d) ? M - d : 0.f;
          memcpy(&src[MS_LANES + l], &sh, 4);
        }
      } else {
        u32 M = 0;
        for (u32 l = 0; l < nn; ++l)
          if (g->h_hubdist[src[l]] != 0xFFFFFFFFu) M = std::max(M, g->h_hubdist[src[l]]);
        for (u32 l = 0; l < nn; ++l)
          src[MS_LANES + l] = g->h_hubdist[src[l]] != 0xFFFFFFFFu ? M - g->h_hubdist[src[l]] : 0u;
      }
    }
    CU(cudaMemcpyAsync(g->ms_src, src.data(), sizeof(u32) * 2 * MS_LANES, cudaMemcpyHostToDevice, s));
    k_ms_init<<<grid_for(g->V * (MS_LANES / 4)), 256, 0, s>>>(g->ms_D, g->ms_Q, g->V, p.inf);
    k_ms_seed<<<1, 32, 0, s>>>(p, g->ms_src, nn);
    CU(cudaGetLastError());
    cudaEvent_t e0, e1;
    for (int i = 0; i < 2; ++i) {
      cudaEvent_t e;
      if (g->ev_pool.empty()) {
        CU(cudaEventCreate(&e));
      } else {
        e = g->ev_pool.back();
        g->ev_pool.pop_back();
      }
      (i ? e1 : e0) = e;
    }
    g->ev_pending.emplace_back(e0, e1);
    CU(cudaEventRecord(e0, s));
    void* args[] = {&p};
    CU(cudaLaunchCooperativeKernel(mk, dim3(grid), dim3(MS_THREADS), args, 0, s));
    CU(cudaEventRecord(e1, s));
    k_ms_output<<<grid_for(g->V), 256, 0, s>>>(g->ms_D, g->old2new, g->V, nn, (u32*)out_dev + (size_t)g0 * ld, ld);
    CU(cudaGetLastError());
    // k_ms_seed clears err for every group: read this group's before the next one starts
    u32 e = 0;
    CU(cudaMemcpyAsync(&e, &g->ms_ctl->err, sizeof e, cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));  // the source buffer is reused by the next group
    err_all |= e;
  }
  if (err_all & ERR_OVERFLOW) return fail(SSSP_ERR_OVERFLOW, "u32 distance overflow");
  return SSSP_OK;
}

extern "C" sssp_status sssp_multi_stats(sssp_graph_t g, uint64_t* out, int64_t n) {
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out || n < 0) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad output");
  if (!g->ms_stats) return fail(SSSP_ERR_INVALID_STATE, "no sssp_run_multi yet");
  DeviceGuard dg(g->device);
  unsigned long long h[MST_N];
  MCtl c;
  CU(cudaMemcpyAsync(h, g->ms_stats, sizeof h, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaMemcpyAsync(&c, g->ms_ctl, sizeof c, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaStreamSynchronize(g->stream));
  const uint64_t v[7] = {h[MST_UPDATES], h[MST_ARCS], h[MST_EXPAND], h[MST_STALE], h[MST_CHUNKS], c.buckets, c.rescans};
  for (int64_t i = 0; i < n && i < 7; ++i) out[i] = v[i];
  return SSSP_OK;
}

extern "C" sssp_status sssp_get_stats(sssp_graph_t g, sssp_stats* out) {
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out) return fail(SSSP_ERR_INVALID_ARGUMENT, "out is NULL");
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  memset(out, 0, sizeof *out);
  unsigned long long h[ST_N];
  Ctl c;
  unsigned long long* cnt = nullptr;
  CU(cudaMallocAsync(&cnt, sizeof(unsigned long long), s));
  CU(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long), s));
  k_count_finite<<<grid_for(g->V), 256, 0, s>>>(g->dist, g->V, g->wtype == SSSP_WEIGHT_F32 ? 0x7F800000u : 0xFFFFFFFFu, cnt);
  unsigned long long reach = 0;
  CU(cudaMemcpyAsync(&reach, cnt, sizeof reach, cudaMemcpyDeviceToHost, s));
  CU(cudaMemcpyAsync(h, g->stats, sizeof h, cudaMemcpyDeviceToHost, s));
  CU(cudaMemcpyAsync(&c, g->ctl, sizeof c, cudaMemcpyDeviceToHost, s));
  CU(cudaFreeAsync(cnt, s));
  CU(cudaStreamSynchronize(s));
  out->updates = h[ST_UPDATES];
  out->light_arcs = h[ST_LIGHT];
  out->heavy_arcs = h[ST_HEAVY];
  out->vertices_settled = h[ST_SETTLED];
  out->stale_items = h[ST_STALE];
  out->heavy_vertices = h[ST_HEAVYV];
  out->hub_chunks = h[ST_CHUNKS];
  out->bin_thread = h[ST_BIN_T];
  out->bin_warp = h[ST_BIN_W];
  out->bin_cta = h[ST_BIN_C];
  out->buckets = c.epochs;
  out->rescans = c.rescans + c.sweeps;
  out->levels = c.rounds;
  out->reachable = g->have_result ? reach : 0;
  out->ring_slots = g->K_used;
  out->grid_ctas = (u32)g->grid_ctas;
  if (g->run_timed) CU(cudaEventElapsedTime(&out->run_ms, g->ev[0], g->ev[1]));
  if (g->reorder_timed) CU(cudaEventElapsedTime(&out->reorder_ms, g->ev[2], g->ev[3]));
  return SSSP_OK;
}

extern "C" sssp_status sssp_export_csr(sssp_graph_t g, double delta, int64_t* rowlist, uint32_t* adj,
                                       void* val, uint32_t* new2old) {
  sssp_status st = check_handle(g);
  if (st) return st;
  DeltaParams dp;
  if ((st = delta_params(g, delta, &dp))) return st;
  DeviceGuard dg(g->device);
  cudaStream_t s = g->stream;
  const i64 V = g->V, A = g->A;
  if (rowlist) {
    std::vector<longlong2> r(V + 1);
    if (g->pro_flags & SSSP_PRO_WEIGHT) {
      longlong2* tmp = nullptr;
      CU(cudaMallocAsync(&tmp, sizeof(longlong2) * (V + 1), s));
      CU(cudaMemcpyAsync(tmp, g->rowp, sizeof(longlong2) * (V + 1), cudaMemcpyDeviceToDevice, s));
      k_heavy_offsets<<<grid_for(V), 256, 0, s>>>(tmp, g->arcs, V, dp.delta_bits);
      CU(cudaGetLastError());
      CU(cudaMemcpyAsync(r.data(), tmp, sizeof(longlong2) * (V + 1), cudaMemcpyDeviceToHost, s));
      CU(cudaFreeAsync(tmp, s));
    } else {
      CU(cudaMemcpyAsync(r.data(), g->rowp, sizeof(longlong2) * (V + 1), cudaMemcpyDeviceToHost, s));
      for (auto& x : r) x.y = x.x;  // no weight order: no heavy offset
    }
    CU(cudaStreamSynchronize(s));
    for (i64 i = 0; i < V; ++i) {
      rowlist[2 * i] = r[i].x;
      rowlist[2 * i + 1] = r[i].y;
    }
    rowlist[2 * V] = r[V].x;
  }
  if ((adj || val) && A > 0) {
    std::vector<uint2> a(A);
    CU(cudaMemcpyAsync(a.data(), g->arcs, sizeof(uint2) * A, cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));
    for (i64 i = 0; i < A; ++i) {
      if (adj) adj[i] = a[i].x;
      if (val) ((u32*)val)[i] = a[i].y;
    }
  }
  if (new2old) {
    if (g->new2old) {
      CU(cudaMemcpyAsync(new2old, g->new2old, sizeof(u32) * V, cudaMemcpyDeviceToHost, s));
      CU(cudaStreamSynchronize(s));
    } else {
      for (i64 i = 0; i < V; ++i) new2old[i] = (u32)i;
    }
  }
  return SSSP_OK;
}

extern "C" sssp_status sssp_kernel_time(sssp_graph_t g, double* total_ms, int64_t* launches, int reset) {
  sssp_status st = check_handle(g);
  if (st) return st;
  DeviceGuard dg(g->device);
  for (auto& pr : g->ev_pending) {
    CU(cudaEventSynchronize(pr.second));
    float ms = 0.f;
    CU(cudaEventElapsedTime(&ms, pr.first, pr.second));
    g->kt_total_ms += ms;
    g->kt_launches += 1;
    g->ev_pool.push_back(pr.first);
    g->ev_pool.push_back(pr.second);
  }
  g->ev_pending.clear();
  if (total_ms) *total_ms = g->kt_total_ms;
  if (launches) *launches = g->kt_launches;
  if (reset) {
    g->kt_total_ms = 0.0;
    g->kt_launches = 0;
  }
  return SSSP_OK;
}

extern "C" sssp_status sssp_get_trace(sssp_graph_t g, sssp_trace_entry* out, int64_t max_entries,
                                      int64_t* n_entries) {
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!n_entries || (max_entries > 0 && !out)) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad trace buffer");
  static_assert(sizeof(sssp_trace_entry) == sizeof(TraceEnt), "trace layout");
  DeviceGuard dg(g->device);
  Ctl c;
  CU(cudaMemcpyAsync(&c, g->ctl, sizeof c, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaStreamSynchronize(g->stream));
  const int64_t n = std::min<int64_t>(c.trace_n, TRACE_CAP);
  *n_entries = n;
  const int64_t k = std::min<int64_t>(n, std::max<int64_t>(max_entries, 0));
  if (k > 0) {
    CU(cudaMemcpyAsync(out, g->trace, sizeof(TraceEnt) * k, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
  }
  return SSSP_OK;
}

extern "C" sssp_status sssp_get_samples(sssp_graph_t g, sssp_trace_entry* out, int64_t max_entries,
                                        int64_t* n_entries) {
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!n_entries || (max_entries > 0 && !out)) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad sample buffer");
  DeviceGuard dg(g->device);
  Ctl c;
  CU(cudaMemcpyAsync(&c, g->ctl, sizeof c, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaStreamSynchronize(g->stream));
  const int64_t n = std::min<int64_t>(c.sample_n, SAMPLE_CAP);
  *n_entries = n;
  const int64_t k = std::min<int64_t>(n, std::max<int64_t>(max_entries, 0));
  if (k > 0) {
    CU(cudaMemcpyAsync(out, g->trace + TRACE_CAP, sizeof(TraceEnt) * k, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
  }
  return SSSP_OK;
}

extern "C" sssp_status sssp_get_profile(sssp_graph_t g, uint64_t* out, int n) {
  sssp_status st = check_handle(g);
  if (st) return st;
  if (!out || n < 0) return fail(SSSP_ERR_INVALID_ARGUMENT, "bad profile buffer");
  DeviceGuard dg(g->device);
  unsigned long long h[ST_N];
  CU(cudaMemcpyAsync(h, g->stats, sizeof h, cudaMemcpyDeviceToHost, g->stream));
  CU(cudaStreamSynchronize(g->stream));
  for (int i = 0; i < n && i < (int)(ST_N - ST_P_CLAIM); ++i) out[i] = h[ST_P_CLAIM + i];
  return SSSP_OK;
}
