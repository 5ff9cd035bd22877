// multi_source.cuh -- NEXT-4 (beyond the paper): batched
// multi-source SSSP in one persistent sm_100a kernel, so one arc read serves
// up to 32 sources and every dist probe is one coalesced 128-byte row.
//
// Layout: D[v][32] u32 (f32 as IEEE bits), lane l = source l of the group;
// Q[v] u32 = the ring bucket v is queued for (NONE = not queued).
// Scheduling is the bucket structure of PAPER §2.2 / Alg. 2 (P:260-270,
// P:1071-1098) with vertices, not (vertex, source) pairs, as work items: a
// vertex is queued in the bucket of the smallest distance that improved it
// (floor(nd / Delta), R2) and, when a warp pops it, every finite lane is
// relaxed over all its arcs (Alg. 1 per lane: nd = D[u][l] + w; atomicMin when
// nd < D[v][l]). Relaxing a lane whose value did not change costs no extra
// traffic (the row is read whole) and is always safe: D[u][l] is the length of
// a real path, so any order of such relaxations converges to the unique
// shortest distances (label-correcting; for f32 the min over left-to-right
// binary32 path sums, reading R-F32). There is no light/heavy split: the
// bucket order only bounds the re-expansions. Buckets advance through a grid
// barrier when the current one is quiescent (pend == 0), like phase 3.
//
// Improvement protocol (no lost wake-ups): the improver does atomicMin(D),
// __syncwarp, a release atomicMin(Q[v], bucket) and pushes v iff Q dropped; the
// expander does an acquire atomicExch(Q[v], NONE), then reads D[v]. Either the expander
// sees the new D, or the improver sees Q == NONE and queues v again.
#pragma once
#include "delta_step.cuh"

namespace sssp {

constexpr int MS_LANES = 32;
constexpr int MS_THREADS = 256;
constexpr int MS_WARPS = MS_THREADS / 32;
#ifndef SSSP_MS_CHUNK
#define SSSP_MS_CHUNK 256
#endif
constexpr u32 MS_CHUNK = SSSP_MS_CHUNK;  // arcs per work item: longer adjacencies are split
#ifndef SSSP_MS_U
#define SSSP_MS_U 2
#endif
constexpr int MS_U = SSSP_MS_U;  // warp steps (4 arcs each) whose rows are in flight together
#ifndef SSSP_MS_CLAIM
#define SSSP_MS_CLAIM 16
#endif
constexpr u32 MS_CLAIM = SSSP_MS_CLAIM;  // queue items per warp claim
constexpr u32 MS_PB = 96;      // staged pushes per warp

enum : u32 { MS_RUN = 0, MS_DONE = 2, MS_RESCAN_CLEAR = 3, MS_RESCAN_FILL = 4 };
enum { MST_UPDATES = 0, MST_ARCS, MST_EXPAND, MST_STALE, MST_CHUNKS, MST_N };

struct __align__(128) MCtl {
  u32 cur, lim, mode, far_min;
  u32 err, buckets, rescans, base;
  u32 pad0[24];
  u32 bar_count, pad1[31];
  u32 bar_gen, pad2[31];
};

struct MParams {
  const uint2* rowc;  // [V+1] .x = first arc of v (u32 offsets)
  const uint2* arcs;  // [A] {dst, wbits}
  u32* D;             // [V][32]
  u32* Q;             // [V]
  MCtl* ctl;
  SlotCtl* sc;        // [K]
  u64* items;         // [K * cap]: v, or (chunk << 32 | CHUNK_FLAG | v)
  unsigned long long* stats;  // [MST_N]
  const u32* shift;           // [32] per-source queue-key shift (lane alignment, see ms_relax)
  u32 V, K, kmask, cap;
  u32 delta_u;      // u32: integer Delta
  float inv_delta;  // f32: fl32(1 / Delta)
  u32 f32, inf;     // weight type; INF bits
  u32 hub_ids;      // internal ids < hub_ids are high-degree vertices (PRO degree order) ...
  u32 hub_delay;    // ... queued hub_delay buckets late, so more sources reach them first
};

#ifndef SSSP_MS_DEFER
#define SSSP_MS_DEFER 0  // 1: D updates fire-and-forget (red.min), Q publications batched per warp (measured slower)
#endif
constexpr u32 MS_CB = 64;  // deferred (bucket << 32 | v) Q publications per warp

struct MSmem {
  u64 pb[MS_WARPS][MS_PB];
  u32 pb_n[MS_WARPS];
  u64 cb[MS_WARPS][MS_CB];
  u32 cb_n[MS_WARPS];
  unsigned long long st[MST_N];
  u32 mode, cur, lim, base;
};

__device__ __forceinline__ u32 ms_bucket_f(const MParams& p, u32 d) {  // f32: floor(d / Delta), R2
  const u32 b = __float2uint_rz(__fmul_rn(__uint_as_float(d), p.inv_delta));
  return b >= NONE ? NONE - 1 : b;
}

// Publish warp w's staged (bucket << 32 | v) pushes: one reservation per
// distinct ring slot per 32 entries (tail and pend in one atomicAdd). Beyond
// the ring horizon or a full queue: dropped, recorded in far_min (rescan).
__device__ __noinline__ void ms_flush(const MParams p, MSmem& sm) {
  const u32 lane = lane_id(), w = threadIdx.x >> 5;
  const u32 n = sm.pb_n[w];
  for (u32 i0 = 0; i0 < n; i0 += 32) {
    const u32 i = i0 + lane;
    bool ok = i < n;
    const u64 e = ok ? sm.pb[w][i] : 0ULL;
    const u32 x = (u32)(e >> 32);
    if (ok && x > sm.lim) {
      atomicMin(&p.ctl->far_min, x);
      ok = false;
    }
    const u32 m = __ballot_sync(SSSP_FULL_MASK, ok);
    if (ok) {
      const u32 s = x & p.kmask;
      const u32 peers = __match_any_sync(m, s);
      const u32 leader = __ffs(peers) - 1;
      const u32 cnt = __popc(peers);
      u64 old = 0;
      if (lane == leader) old = atomicAdd(&p.sc[s].word, ((u64)cnt << 32) | cnt);
      old = __shfl_sync(peers, old, leader);
      const u32 idx = (u32)(old >> 32) + __popc(peers & lanemask_lt());
      if (idx < p.cap) {
        st_relaxed_u64(p.items + (u64)s * p.cap + idx, (u64)(u32)e);
      } else {
        atomicAdd(&p.sc[s].word, ~0ULL);  // undo the pending count; rescan recovers it
        atomicMin(&p.ctl->far_min, x);
      }
    }
  }
  __syncwarp();
  if (lane == 0) sm.pb_n[w] = 0;
  __syncwarp();
}

// Filter probe of 4 lanes of a D row (16 B; a stale L1 value is >= the
// current one: at most an extra atomic, never a missed improvement).
__device__ __forceinline__ uint4 ms_probe4(const u32* a, bool pred) {
  uint4 v;
  asm volatile(
      "{\n .reg .pred q;\n setp.ne.b32 q, %4, 0;\n mov.b32 %0, 0;\n mov.b32 %1, 0;\n"
      " mov.b32 %2, 0;\n mov.b32 %3, 0;\n"
      " @q ld.global.cg.v4.u32 {%0, %1, %2, %3}, [%5];\n}"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
      : "r"((u32)pred), "l"(a));
  return v;
}

// Q[v] publication: the improver's min is a release (the warp's D atomics,
// ordered before it by __syncwarp, become visible with it; SASS: MEMBAR.ALL.GPU
// + ATOM, no L1 invalidate), the expander's exchange an acquire (ATOM +
// CCTL.IVALL), so an expander that sees the new Q value also sees the new D.
#ifndef SSSP_MS_FENCE
#define SSSP_MS_FENCE 1
#endif
// Predicated atomicMin; returns 0 (so "nd < old" is false) when !pred.
__device__ __forceinline__ u32 ms_atomic_min(u32* a, u32 v, bool pred) {
  u32 old;
  asm volatile(
      "{\n .reg .pred q;\n setp.ne.b32 q, %3, 0;\n mov.b32 %0, 0;\n"
      " @q atom.relaxed.gpu.global.min.u32 %0, [%1], %2;\n}"
      : "=r"(old)
      : "l"(a), "r"(v), "r"((u32)pred)
      : "memory");
  return old;
}

__device__ __forceinline__ u32 ms_q_min_release(u32* a, u32 v) {
  u32 old;
#if SSSP_MS_FENCE
  asm volatile("atom.release.gpu.global.min.u32 %0, [%1], %2;" : "=r"(old) : "l"(a), "r"(v) : "memory");
#else
  old = atomicMin(a, v);
#endif
  return old;
}
__device__ __forceinline__ u32 ms_q_take_acquire(u32* a) {
  u32 old;
  asm volatile("atom.acquire.gpu.global.exch.b32 %0, [%1], %2;" : "=r"(old) : "l"(a), "r"(NONE) : "memory");
  return old;
}

__device__ __forceinline__ void ms_red_min(u32* a, u32 v, bool pred) {
  asm volatile(
      "{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n"
      " @q red.relaxed.gpu.global.min.u32 [%0], %1;\n}" ::"l"(a), "r"(v), "r"((u32)pred)
      : "memory");
}

// Stage this warp's queue pushes (lanes with push) for ms_flush.
__device__ __forceinline__ void ms_stage_pushes(const MParams& p, MSmem& sm, bool push, u32 key, u32 v) {
  const u32 m = __ballot_sync(SSSP_FULL_MASK, push);
  if (m) {
    const u32 w = threadIdx.x >> 5;
    if (sm.pb_n[w] + __popc(m) > MS_PB) ms_flush(p, sm);
    if (push) sm.pb[w][sm.pb_n[w] + __popc(m & lanemask_lt())] = ((u64)key << 32) | v;
    __syncwarp();
    if (lane_id() == 0) sm.pb_n[w] += __popc(m);
    __syncwarp();
  }
}

// Deferred Q publications of warp w: Q[v] = min(Q[v], bucket) as release
// atomics (after __syncwarp, so every red.min the warp issued before is
// visible to the acquiring expander), queueing v where Q dropped.
__device__ __noinline__ void ms_publish(const MParams p, MSmem& sm) {
  const u32 lane = lane_id(), w = threadIdx.x >> 5;
  const u32 n = sm.cb_n[w];
  __syncwarp();
  for (u32 i0 = 0; i0 < n; i0 += 32) {
    const u32 i = i0 + lane;
    const u64 e = i < n ? sm.cb[w][i] : ~0ULL;
    const u32 key = (u32)(e >> 32), v = (u32)e;
    const bool push = i < n && ms_q_min_release(p.Q + v, key) > key;
    ms_stage_pushes(p, sm, push, key, v);
  }
  __syncwarp();
  if (lane == 0) sm.cb_n[w] = 0;
  __syncwarp();
}

// Queue keys use "aligned time" nd + shift[lane] instead of nd: the host
// sets shift[l] = M - d(hub, source l) (M = the largest such distance), so the
// 32 sources' wavefronts, which all pass through the hubs, reach a vertex in
// about the same bucket and it is expanded about once for all of them. Any
// key is correct (label-correcting); the shift only orders the work.
template <bool F32>
__device__ __forceinline__ u32 ms_time(u32 nd, u32 sh) {
  if (F32) return __float_as_uint(__fadd_rn(__uint_as_float(nd), __uint_as_float(sh)));
  const u64 t = (u64)nd + sh;
  return t >= (u64)NONE ? NONE - 1 : (u32)t;
}

// Relax arcs [b, e) of vertex u for every finite source of the group. Lane l
// holds sources 4*(l&7) .. 4*(l&7)+3 (du = D[u][those]); the 8 lanes of
// group l>>3 relax one arc together, so a warp step covers 4 arcs and each
// probe instruction reads four whole 128-byte rows.
template <bool F32>
__device__ __forceinline__ void ms_relax(const MParams& p, MSmem& sm, u32 b, u32 e, const u32 (&du)[4],
                                         const u32 (&sh)[4], u32& c_upd) {
  const u32 lane = lane_id(), grp = lane >> 3, sub = lane & 7, cur = sm.cur;
  const u64 pol_stream = policy_evict_first();
  bool ovf = false;
  uint2 arc_next = ld_arc(p.arcs + b + lane, b + lane < e, pol_stream);
  for (u32 a0 = b; a0 < e; a0 += 32) {
    const u32 na = min(32u, e - a0);
    const uint2 arc = arc_next;  // this chunk's arcs; the next chunk's load starts now
    arc_next = ld_arc(p.arcs + a0 + 32 + lane, a0 + 32 + lane < e, pol_stream);
    for (u32 t = 0; t < na; t += 4 * MS_U) {
      u32 dst[MS_U], nd[MS_U][4];
      uint4 pr[MS_U];
      bool ok[MS_U];
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        const u32 j = t + 4 * k + grp;
        ok[k] = j < na;
        dst[k] = __shfl_sync(SSSP_FULL_MASK, arc.x, j & 31);
        const u32 w = __shfl_sync(SSSP_FULL_MASK, arc.y, j & 31);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if (F32) {  // Alg. 1 l.1 in binary32 (inf + w = inf: never below a probe)
            nd[k][c] = __float_as_uint(__fadd_rn(__uint_as_float(du[c]), __uint_as_float(w)));
          } else {  // exact u32: a wrap or the INF value itself means "no candidate"
            const u32 x = du[c] + w;
            const bool bad = x < du[c] || x == NONE;
            ovf |= ok[k] && bad && du[c] != NONE;
            nd[k][c] = bad ? NONE : x;
          }
        }
        pr[k] = ms_probe4(p.D + (u64)dst[k] * MS_LANES + 4 * sub, ok[k]);
      }
      u32 mn[MS_U];
#if SSSP_MS_DEFER
      // Alg. 1 l.2-3 as a fire-and-forget red.min wherever the probe says the
      // candidate is smaller; the candidate counts as an update (it may lose to
      // a concurrent smaller one: then v is only queued once too often).
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        const u32 pv[4] = {pr[k].x, pr[k].y, pr[k].z, pr[k].w};
        u32* row = p.D + (u64)dst[k] * MS_LANES + 4 * sub;
        mn[k] = NONE;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const bool want = ok[k] && nd[k][c] < pv[c];
          ms_red_min(row + c, nd[k][c], want);
          c_upd += want;
          mn[k] = want ? min(mn[k], ms_time<F32>(nd[k][c], sh[c])) : mn[k];
        }
      }
#else
      // all 4 * MS_U atomics in flight before any result is consumed
      u32 old[MS_U][4];
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        const u32 pv[4] = {pr[k].x, pr[k].y, pr[k].z, pr[k].w};
        u32* row = p.D + (u64)dst[k] * MS_LANES + 4 * sub;
#pragma unroll
        for (int c = 0; c < 4; ++c)  // Alg. 1 l.2, then l.3 (0 when not issued)
          old[k][c] = ms_atomic_min(row + c, nd[k][c], ok[k] && nd[k][c] < pv[c]);
      }
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        mn[k] = NONE;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const bool imp = nd[k][c] < old[k][c];
          c_upd += imp;
          mn[k] = imp ? min(mn[k], ms_time<F32>(nd[k][c], sh[c])) : mn[k];
        }
      }
#endif
      // smallest improved distance of each arc over its 32 sources (8 lanes)
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        mn[k] = min(mn[k], __shfl_xor_sync(SSSP_FULL_MASK, mn[k], 1));
        mn[k] = min(mn[k], __shfl_xor_sync(SSSP_FULL_MASK, mn[k], 2));
        mn[k] = min(mn[k], __shfl_xor_sync(SSSP_FULL_MASK, mn[k], 4));
      }
      // lane i < 4*MS_U publishes arc i = 4k + g (group g, step k): Q[v] = min(Q[v], bucket)
      u32 my_dst = 0, my_key = NONE;
#pragma unroll
      for (int k = 0; k < MS_U; ++k) {
        const u32 src_lane = 8 * (lane & 3);
        const u32 m = __shfl_sync(SSSP_FULL_MASK, mn[k], src_lane);
        const u32 d = __shfl_sync(SSSP_FULL_MASK, dst[k], src_lane);
        if ((lane >> 2) == (u32)k && m != NONE) {
          my_dst = d;
          my_key = max(F32 ? ms_bucket_f(p, m) : m / p.delta_u, cur) + (d < p.hub_ids ? p.hub_delay : 0u);
        }
      }
#if SSSP_MS_DEFER
      const u32 cm = __ballot_sync(SSSP_FULL_MASK, my_key != NONE);
      if (cm) {  // defer: one release fence per batch of publications (ms_publish)
        const u32 w = threadIdx.x >> 5;
        if (sm.cb_n[w] + __popc(cm) > MS_CB) ms_publish(p, sm);
        if (my_key != NONE) sm.cb[w][sm.cb_n[w] + __popc(cm & lanemask_lt())] = ((u64)my_key << 32) | my_dst;
        __syncwarp();
        if (lane == 0) sm.cb_n[w] += __popc(cm);
        __syncwarp();
      }
#else
      if (__any_sync(SSSP_FULL_MASK, my_key != NONE)) {
        __syncwarp();
        bool push = false;
        if (my_key != NONE) push = ms_q_min_release(p.Q + my_dst, my_key) > my_key;
        ms_stage_pushes(p, sm, push, my_key, my_dst);
      }
#endif
    }
  }
  if (!F32 && ovf) atomicOr(&p.ctl->err, ERR_OVERFLOW);
}

__device__ void ms_grid_barrier(const MParams& p, MSmem& sm);

template <bool F32>
__device__ void ms_bucket_run(const MParams& p, MSmem& sm) {
  const u32 lane = lane_id();
  const u32 slot = sm.cur & p.kmask;
  SlotCtl* sc = p.sc + slot;
  u64* q = p.items + (u64)slot * p.cap;
  u32 my_next = 0, my_end = 0;  // lane 0: claimed tickets
  u32 c_upd = 0, c_arcs = 0, c_exp = 0, c_stale = 0, c_chunks = 0;
  for (;;) {
    u32 h = 0, n = 0;
    if (lane == 0) {
      u32 ns = 32;
      for (;;) {
        const u64 wv = ld_relaxed_u64(&sc->word);
        const u32 tail = min((u32)(wv >> 32), p.cap);
        if (my_next >= my_end && my_end < p.cap) {
          my_next = atomicAdd(&sc->head, MS_CLAIM);
          my_end = my_next + MS_CLAIM;
        }
        const u32 ae = min(my_end, tail);
        if (my_next < ae) {
          h = my_next;
          n = ae - my_next;
          my_next = ae;
          break;
        }
        if ((u32)wv == 0) break;  // quiescent
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
      }
    }
    n = __shfl_sync(SSSP_FULL_MASK, n, 0);
    h = __shfl_sync(SSSP_FULL_MASK, h, 0);
    if (n == 0) break;
    // Prologue of the whole claim at once (lane i: item i): wait for the entry, recycle it,
    // read its arc range and take Q[v] -- one round trip of each for up to MS_CLAIM items
    // instead of per item (the items are then relaxed one after another).
    static_assert(MS_CLAIM <= 32, "one lane per claimed item");
    u32 iv = 0, ib = 0, ie = 0, ix = NONE, ich = 0;
    if (lane < n) {
      u64 e;
      u32 ns = 16;
      while ((e = ld_relaxed_u64(q + h + lane)) == SENTINEL) {  // reserved, not yet written
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
      }
      st_relaxed_u64(q + h + lane, SENTINEL);
      const u32 lo = (u32)e;
      iv = lo & ~CHUNK_FLAG;
      ich = (lo & CHUNK_FLAG) ? 1u : 0u;
      ib = p.rowc[iv].x;
      ie = p.rowc[iv + 1].x;
      if (ich) {
        ib += (u32)(e >> 32) * MS_CHUNK;
        ie = min(ie, ib + MS_CHUNK);
      } else {
        ix = ms_q_take_acquire(p.Q + iv);  // NONE: already expanded through another entry
      }
    }
    __syncwarp();  // every take precedes the row reads below (acquire, then warp order)
    for (u32 i = 0; i < n; ++i) {
      const u32 v = __shfl_sync(SSSP_FULL_MASK, iv, i);
      const u32 b = __shfl_sync(SSSP_FULL_MASK, ib, i), en = __shfl_sync(SSSP_FULL_MASK, ie, i);
      const u32 x = __shfl_sync(SSSP_FULL_MASK, ix, i), ch = __shfl_sync(SSSP_FULL_MASK, ich, i);
      if (!ch) {
        if (x == NONE) {
          ++c_stale;
          continue;
        }
        ++c_exp;
        if (en - b > MS_CHUNK) {  // split: ceil(deg / 256) items any warp may claim
          const u32 nc = (en - b + MS_CHUNK - 1) / MS_CHUNK;
          c_chunks += nc;
          u32 base = 0;
          if (lane == 0) base = (u32)(atomicAdd(&sc->word, ((u64)nc << 32) | nc) >> 32);
          base = __shfl_sync(SSSP_FULL_MASK, base, 0);
          for (u32 c = lane; c < nc; c += 32) {
            if (base + c < p.cap) {
              st_relaxed_u64(q + base + c, ((u64)c << 32) | CHUNK_FLAG | v);
            } else {
              atomicAdd(&sc->word, ~0ULL);
              atomicMin(&p.ctl->far_min, sm.cur);  // lost work of this bucket: rescan
              atomicExch(p.Q + v, sm.cur);         // v must be found by the rescan
            }
          }
          continue;
        }
      }
      const uint4 d4 = __ldcg(reinterpret_cast<const uint4*>(p.D + (u64)v * MS_LANES) + (lane & 7));
      const u32 du[4] = {d4.x, d4.y, d4.z, d4.w};
      const uint4 s4 = __ldg(reinterpret_cast<const uint4*>(p.shift) + (lane & 7));
      const u32 sh[4] = {s4.x, s4.y, s4.z, s4.w};
      c_arcs += en - b;
      ms_relax<F32>(p, sm, b, en, du, sh, c_upd);
    }
#if SSSP_MS_DEFER
    if (sm.cb_n[threadIdx.x >> 5]) ms_publish(p, sm);
#endif
    if (sm.pb_n[threadIdx.x >> 5]) ms_flush(p, sm);  // publish before completing
    if (lane == 0) atomicAdd(&sc->word, (u64)0 - (u64)n);
  }
  const u32 upd = __reduce_add_sync(SSSP_FULL_MASK, c_upd);
  if (lane == 0) {
    atomicAdd(&sm.st[MST_UPDATES], (unsigned long long)upd);
    atomicAdd(&sm.st[MST_ARCS], (unsigned long long)c_arcs);
    atomicAdd(&sm.st[MST_EXPAND], (unsigned long long)c_exp);
    atomicAdd(&sm.st[MST_STALE], (unsigned long long)c_stale);
    atomicAdd(&sm.st[MST_CHUNKS], (unsigned long long)c_chunks);
  }
}

// Serial scheduler step of the last CTA at a barrier (phase 3 of Alg. 2).
__device__ void ms_decide(const MParams& p) {
  volatile MCtl* c = p.ctl;
  volatile SlotCtl* sc = p.sc;
  const u32 mode = c->mode;
  if (mode == MS_RUN) {
    const u32 cur = c->cur, fm = c->far_min;
    u32 nxt = NONE;
    for (u32 x = cur + 1; x <= c->lim && x != NONE; ++x)
      if ((u32)(sc[x & p.kmask].word >> 32) != 0) {
        nxt = x;
        break;
      }
    if (fm != NONE && (fm <= cur || nxt == NONE || fm <= nxt)) {  // dropped pushes: rebuild
      c->base = cur;
      c->mode = MS_RESCAN_CLEAR;
      return;
    }
    if (nxt == NONE) {
      c->mode = MS_DONE;
      return;
    }
    const u32 s = cur & p.kmask;
    sc[s].word = 0;
    sc[s].head = 0;
    c->lim = (u32)min((u64)cur + p.K - 1, (u64)NONE - 1);
    c->cur = nxt;
    c->buckets = c->buckets + 1;
  } else if (mode == MS_RESCAN_CLEAR) {
    for (u32 s = 0; s < p.K; ++s) {
      sc[s].word = 0;
      sc[s].head = 0;
    }
    const u32 r = c->base;
    c->far_min = NONE;
    c->cur = r;
    c->lim = (u32)min((u64)r + p.K - 1, (u64)NONE - 1);
    c->mode = MS_RESCAN_FILL;
  } else if (mode == MS_RESCAN_FILL) {
    c->rescans = c->rescans + 1;
    c->buckets = c->buckets + 1;
    c->mode = MS_RUN;
  }
}

__device__ void ms_grid_barrier(const MParams& p, MSmem& sm) {
  __syncthreads();
  if (threadIdx.x == 0) {
    MCtl* c = p.ctl;
    u32 target;
    if (grid_arrive(&c->bar_count, &target)) {
      ms_decide(p);
      grid_release(&c->bar_gen, target);
    } else {
      grid_wait(&c->bar_gen, target);
    }
    volatile MCtl* vc = c;
    sm.mode = vc->mode;
    sm.cur = vc->cur;
    sm.lim = vc->lim;
    sm.base = vc->base;
  }
  __syncthreads();
}

// Rescan: clear every queue, then queue each pending vertex (Q != NONE) in
// bucket max(Q, base), clamped to the ring horizon (early is always safe).
__device__ void ms_rescan_clear(const MParams& p) {
  const i64 t = (i64)blockIdx.x * blockDim.x + threadIdx.x, nt = (i64)gridDim.x * blockDim.x;
  for (u32 s = 0; s < p.K; ++s) {
    const u32 tail = min((u32)(ld_relaxed_u64(&p.sc[s].word) >> 32), p.cap);
    u64* q = p.items + (u64)s * p.cap;
    for (i64 i = t; i < tail; i += nt) st_relaxed_u64(q + i, SENTINEL);
  }
}

__device__ void ms_rescan_fill(const MParams& p, MSmem& sm) {
  const i64 t0 = ((i64)blockIdx.x * blockDim.x + threadIdx.x) & ~31LL, nt = (i64)gridDim.x * blockDim.x;
  const u32 lane = lane_id(), w = threadIdx.x >> 5;
  for (i64 b = t0; b < p.V; b += nt) {
    const i64 v = b + lane;
    u32 key = NONE;
    if (v < p.V) {
      const u32 qv = ld_cg(p.Q + v);
      if (qv != NONE) {
        key = min(max(qv, sm.base), sm.lim);
        p.Q[v] = key;
      }
    }
    const u32 m = __ballot_sync(SSSP_FULL_MASK, key != NONE);
    if (m) {
      if (sm.pb_n[w] + 32 > MS_PB) ms_flush(p, sm);
      if (key != NONE) sm.pb[w][sm.pb_n[w] + __popc(m & lanemask_lt())] = ((u64)key << 32) | (u32)v;
      __syncwarp();
      if (lane == 0) sm.pb_n[w] += __popc(m);
      __syncwarp();
    }
  }
  if (sm.pb_n[w]) ms_flush(p, sm);
}

#ifndef SSSP_MS_MINB
#define SSSP_MS_MINB 6
#endif
template <bool F32>
__global__ void __launch_bounds__(MS_THREADS, SSSP_MS_MINB) k_ms_step(MParams p) {
  __shared__ MSmem sm;
  if (threadIdx.x < MST_N) sm.st[threadIdx.x] = 0;
  if (threadIdx.x < MS_WARPS) sm.pb_n[threadIdx.x] = sm.cb_n[threadIdx.x] = 0;
  if (threadIdx.x == 0) {
    volatile MCtl* vc = p.ctl;
    sm.mode = vc->mode;
    sm.cur = vc->cur;
    sm.lim = vc->lim;
    sm.base = vc->base;
  }
  __syncthreads();
  for (;;) {
    const u32 mode = sm.mode;
    if (mode == MS_DONE) break;
    if (mode == MS_RUN)
      ms_bucket_run<F32>(p, sm);
    else if (mode == MS_RESCAN_CLEAR)
      ms_rescan_clear(p);
    else
      ms_rescan_fill(p, sm);
    ms_grid_barrier(p, sm);
  }
  __syncthreads();
  if (threadIdx.x < MST_N && sm.st[threadIdx.x]) atomicAdd(p.stats + threadIdx.x, sm.st[threadIdx.x]);
}

// D[:][:] = INF, Q[:] = NONE (a5 for the whole group).
__global__ void k_ms_init(u32* __restrict__ D, u32* __restrict__ Q, i64 V, u32 inf) {
  const i64 stride = (i64)gridDim.x * blockDim.x;
  const uint4 f = make_uint4(inf, inf, inf, inf);
  uint4* D4 = reinterpret_cast<uint4*>(D);
  for (i64 i = (i64)blockIdx.x * blockDim.x + threadIdx.x; i < V * (MS_LANES / 4); i += stride) D4[i] = f;
  for (i64 i = (i64)blockIdx.x * blockDim.x + threadIdx.x; i < V; i += stride) Q[i] = NONE;
}

// D[src_l][l] = 0 for the group's sources; bucket 0 holds each distinct source.
__global__ void k_ms_seed(MParams p, const u32* __restrict__ src, u32 n) {
  if (threadIdx.x != 0) return;
  for (u32 s = 0; s < p.K; ++s) {
    p.sc[s].word = 0;
    p.sc[s].head = 0;
  }
  u32 cnt = 0;
  for (u32 l = 0; l < n; ++l) {
    const u32 v = src[l];
    p.D[(u64)v * MS_LANES + l] = 0;
    if (p.Q[v] != 0) {
      p.Q[v] = 0;
      p.items[cnt++] = v;
    }
  }
  p.sc[0].word = ((u64)cnt << 32) | cnt;
  for (u32 i = 0; i < MST_N; ++i) p.stats[i] = 0;
  MCtl* c = p.ctl;
  c->cur = 0;
  c->lim = p.K - 1;
  c->mode = MS_RUN;
  c->far_min = NONE;
  c->err = 0;
  c->buckets = 1;
  c->rescans = 0;
  c->base = 0;
  c->bar_count = 0;
  c->bar_gen = 0;
}

// out[l * ld + o] = D[old2new[o]][l] for l < n (a8 for the group; f32 bits as is).
__global__ void k_ms_output(const u32* __restrict__ D, const u32* __restrict__ old2new, i64 V, u32 n,
                            u32* __restrict__ out, i64 ld) {
  const i64 stride = (i64)gridDim.x * blockDim.x;
  for (i64 o = (i64)blockIdx.x * blockDim.x + threadIdx.x; o < V; o += stride) {
    const u64 v = old2new ? old2new[o] : (u64)o;
    const uint4* row = reinterpret_cast<const uint4*>(D + v * MS_LANES);
    for (u32 l4 = 0; l4 < (n + 3) / 4; ++l4) {
      const uint4 x = row[l4];
      const u32 xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
      for (u32 k = 0; k < 4; ++k)
        if (l4 * 4 + k < n) out[(i64)(l4 * 4 + k) * ld + o] = xs[k];
    }
  }
}

}  // namespace sssp
