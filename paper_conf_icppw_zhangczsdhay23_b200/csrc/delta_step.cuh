// delta_step.cuh -- the persistent bucket-aware asynchronous Delta-stepping
// kernel (sm_100a). One cooperative launch runs the whole bucket loop of
// PAPER Alg. 2 on the device:
//
//   phase 1 (Alg. 2 l.6-9): asynchronous light-arc relaxation of the current
//     bucket. CTAs pull batches of (v, d) entries from the bucket's queue,
//     bin them by light degree l: l < 32 -> thread bin (arcs of
//     a warp's small vertices spread over its lanes by a warp prefix sum,
//     ranges staged in shared memory), 32 <= l < 256 -> warp per vertex,
//     256 <= l <= 4096 -> CTA per vertex, l > 4096 -> ceil(l/4096) chunks any
//     CTA may claim (reading R11). Improved vertices are pushed
//     into the near queue (same bucket: visible without a level barrier,
//     P:1100-1103) or a far bucket queue. The phase ends at quiescence:
//     pend (pushed - completed) == 0 (manager/worker end rule).
//   phases 2&3 (Alg. 2 l.13-19): after a grid barrier, heavy arcs
//     of the bucket's settled vertices (entries with d == dist[v]) are relaxed
//     once, hubs split into 4096-arc chunks; then the next non-empty bucket
//     is chosen by the last CTA to arrive at the barrier (fused phase 3).
//
// Data (all device memory): dist[V] u32 (f32 as IEEE bits: order-preserving
// for w >= 0, so one atomicMin.u32 serves both weight types, Alg. 1 l.3);
// a ring of K bucket queues of packed u64 entries (d << 32 | v). Each queue
// has its own 128-byte control line: word = (tail << 32 | pend), so one
// atomicAdd both reserves entries and counts pending work, and head, the
// consumers' ticket counter. Consumers claim position ranges with atomicAdd
// (never fails; a range may run ahead of tail and is filled as producers
// publish); entries are published by value (SENTINEL = empty). Producers
// stage pushes per warp in shared memory (one global reservation per flush).
// Pushes beyond the ring horizon or beyond a queue's capacity are dropped and
// recorded in far_min; the scheduler then rebuilds the ring from dist[]
// (topological rescan, as the paper's phase 3 loops over all V, Alg. 2 l.13)
// or, for the current bucket, finishes it with Bellman-Ford sweeps.
#pragma once
#include "common.cuh"

namespace sssp {

#ifndef SSSP_MINB
#define SSSP_MINB 4  // persistent CTAs per SM the register budget is sized for
#endif
#ifndef SSSP_DS_THREADS
#define SSSP_DS_THREADS 256
#endif
constexpr int DS_THREADS = SSSP_DS_THREADS;
constexpr int DS_WARPS = DS_THREADS / 32;
constexpr u32 BIN_WARP = 32;     // beta
constexpr u32 BIN_CTA = 256;     // alpha
constexpr u32 HUB_CHUNK = 4096;
#ifndef SSSP_UNROLL
#define SSSP_UNROLL 2  // arcs per lane per warp task (B200 A/B: 2 beats 4 and 1 on C4 and C3, profiles/r02)
#endif
#ifndef SSSP_PROBE_L1
#define SSSP_PROBE_L1 1  // dist probes through L1 (a stale value is a safe filter)
#endif
#ifndef SSSP_PREFETCH
#define SSSP_PREFETCH 0  // 1: L2 bulk prefetch of each claimed vertex's arc range (session 3: 4 % slower on C4)
#endif
#ifndef SSSP_LAT
#define SSSP_LAT 0  // per-stage latency accounting in the task loop (diagnostics build)
#endif
#ifndef SSSP_DEFER_ATOMICS
#define SSSP_DEFER_ATOMICS 1  // relaxations' atomicMin issued by pb_flush, a staged batch at once
#endif
#ifndef SSSP_STATIC_TASKS
#define SSSP_STATIC_TASKS 1  // batch tasks dealt round-robin to the warps (no shared-memory claim atomic)
#endif
#ifndef SSSP_BATCH_SAMPLES
#define SSSP_BATCH_SAMPLES 0  // per-batch stage/task/tail cycles in sssp_get_samples (diagnostics build)
#endif
constexpr int UNROLL = SSSP_UNROLL;
#ifndef SSSP_IPT
#define SSSP_IPT 2  // queue items decoded per thread per phase-1 batch
#endif
#ifndef SSSP_IPT2
#define SSSP_IPT2 2  // ... per phase-2 batch (static, all items ready)
#endif
constexpr int IPT = SSSP_IPT;
constexpr int IPT2 = SSSP_IPT2;
constexpr int IPT_MAX = IPT > IPT2 ? IPT : IPT2;
#ifndef SSSP_PULL_DIV
#define SSSP_PULL_DIV 128u  // pull phases 2&3 when a bucket holds >= V / 128 entries (A/B on C4, C3: 128 beats 8-64, = 256; profiles/r02/ab_pull_div.txt)
#endif
#ifndef SSSP_CLAIM_MINPART
#define SSSP_CLAIM_MINPART 64u  // take a partial batch once this many entries are ready ...
#endif
#ifndef SSSP_CLAIM_WAIT_NS
#define SSSP_CLAIM_WAIT_NS 200u  // ... or after waiting this long for a full one (2000: C2 -4 %, C1 -8 %)
#endif
constexpr u64 SENTINEL = ~0ULL;
constexpr u32 NONE = 0xFFFFFFFFu;
constexpr u32 CHUNK_FLAG = 0x80000000u;
constexpr u32 APPLIED_FLAG = 0x80000000u;  // in a staged push's vertex field (V < 2^31), see stage_pushes

enum : u32 {
  MODE_PHASE1 = 0,
  MODE_PHASE2 = 1,
  MODE_DONE = 2,
  MODE_RESCAN_CLEAR = 3,
  MODE_RESCAN_FILL = 4,
  MODE_SWEEP_LIGHT = 5,
  MODE_SWEEP_HEAVY = 6,
  MODE_P2_COMPACT = 7,  // edge-balanced phase 2, step 1: settled entries -> heavy-arc offsets
  MODE_P2_RELAX = 8,    // ... step 2: equal heavy-arc ranges per warp
  MODE_MERGE = 9,       // adaptive Delta: fold the slots (cur, cur_end) into slot cur
  MODE_PULL = 10,       // phases 2&3 as a pull over the unsettled vertices (symmetric graphs)
  MODE_PULL_LONG = 11   // ... second step: long heavy-arc scans, one warp per vertex
};
enum : u32 { ERR_OVERFLOW = 1, ERR_INTERNAL = 2 };
enum : u32 { SYNC_P1 = 0, SYNC_P2 = 1, SYNC_RC = 2, SYNC_RF = 3, SYNC_SL = 4, SYNC_SH = 5, SYNC_P2C = 6,
              SYNC_MG = 7, TRACE_ADAPT = 8, SYNC_PL = 9 };
enum : u32 { SRC_QUEUE = 0, SRC_STATIC = 1, SRC_HUB = 2, SRC_SWEEP = 3 };

enum {
  ST_UPDATES = 0,
  ST_LIGHT,
  ST_HEAVY,
  ST_SETTLED,
  ST_STALE,
  ST_HEAVYV,
  ST_CHUNKS,
  ST_BIN_T,
  ST_BIN_W,
  ST_BIN_C,
  // cycle accounting of thread 0 of every CTA (diagnostics, sssp_get_profile)
  ST_P_CLAIM,  // waiting for / claiming queue entries
  ST_P_STAGE,  // batch decode + task-pool staging (until the pool barrier)
  ST_P_TASK,   // warp 0 in the task loop
  ST_P_TAIL,   // warp 0 after its last task until the batch barrier (flush + wait)
  ST_P_BAR,    // grid barriers
  ST_P_NB,     // batches
  ST_P_NT,     // tasks
  ST_L_ARC,    // warp 0: cycles waiting for a task's arcs (issued one task ahead)
  ST_L_PROBE,  // ... for its dist probes
  ST_L_ATOM,   // ... for its atomics
  ST_L_STAGE,  // ... staging the pushes
  ST_L_N,      // tasks measured
  ST_ATOMS,    // atomicMin issued (diagnostics builds)
  ST_N
};

struct __align__(128) SlotCtl {
  u64 word;  // (tail << 32) | pend
  u32 head;  // consumer tickets
  u32 p2;    // prefix already handled by phase 2
  u32 pad[28];
};

struct __align__(128) Ctl {
  u32 cur, lim, mode, far_min;
  u32 p2_begin, p2_end, err, epochs;
  u32 rescans, rescan_base, changed, sweep_first;
  u32 sweeps, trace_n, round_end, rounds;  // round_end: level-synchronous mode (ablation)
  // Bucket = fine ring slots [cur, cur_end) (units of the fine width g = delta_u / 1/inv_delta).
  // Fixed Delta: cur_end = cur + 1. Adaptive Delta (NEXT-1, Eq. (1)-(2) P:1006-1028): the
  // width m (fine slots) follows Delta_i = Delta_{i-1} + eps_i, see adapt_next().
  u32 cur_end;
  u32 a_mode;        // 0 fixed, 1 Eq. (2) cumulative (reading A), 2 Delta0 + eps_i (reading B)
  u32 a_i;           // buckets completed
  u32 a_c1, a_c2;    // C_{i-1}, C_{i-2}: converged (settled) vertices of the previous buckets
  u32 a_t1, a_t2;    // T_{i-1}, T_{i-2}: threads (phase-1 queue items) of the previous buckets
  float a_dlt;       // Delta_{i-1} in fine units
  float a_d0;        // Delta_0 in fine units
  u32 a_mmin, a_mmax, a_m;  // width clamp and current width (fine slots)
  u32 lvl;           // light/heavy level of the current bucket: light iff w < g << lvl
  u32 csum;          // settled vertices of the current bucket (phase 2 / pull count them)
  u32 err_acc;       // OR of err over every run since the host last read it (k_seed keeps it)
  u32 bf;            // Bellman-Ford end: 0 off, 1 running (all arcs, one queue), 2 final clear
  // pull phases 2&3: candidate lists (unsettled vertices with arcs) in xd[V..3V); pull_sel = the
  // input list (2 = every vertex, the first pull), pull_n = list lengths
  u32 pull_sel, pull_n[2];
  u32 closed_c, closed_b;    // C_i and index of the bucket the last scheduler step closed (trace)
  u32 bf_t;          // switch to the Bellman-Ford end once the ring holds <= bf_t entries (0: never)
  u32 bf_peak;       // most entries any closed bucket held (the end phase waits for the peak)
  u32 pad_t;
  u64 t_first;               // earliest arrival at the current grid barrier (%globaltimer, trace)
  u32 long_n, long_head;     // pull: long scans handed to whole warps (count, claim tickets)
  u32 sample_n;              // phase-1 claim samples written (diagnostics)
  u32 first_n;               // the first pull's candidates: ids [0, first_n) (isolated ids excluded)
  u32 pad_b[18];
  u32 bar_count, pad3[31];   // own line: arrivals
  u32 bar_gen, pad4[31];     // own line: spun on
  u32 p2_head, pad5[31];     // own line: phase-2 static tickets
  u64 hub_word;              // phase-2 chunk queue: (tail << 32) | pend; edge-balanced
                             // phase 2: (compacted entries << 32) | heavy arcs
  u32 hub_head, pad6[29];
};

constexpr u32 TRACE_CAP = 4096;
constexpr u32 SAMPLE_CAP = 16384;  // phase-1 claim samples after the trace (sssp_get_samples)
constexpr u32 SAMPLE_EVERY = 37;   // CTAs with blockIdx % 37 == 0 record theirs
struct TraceEnt {
  u64 t_ns;   // %globaltimer when the last CTA arrived
  u32 which;  // SYNC_* (99 = kernel start)
  u32 cur;    // current bucket
  u32 tail;   // entries in the current bucket's queue
  u32 mode;   // mode chosen by the scheduler
  u32 far_min, pad;
  u32 closed_b, closed_c;  // bucket this step closed and its settled-vertex count C (else NONE, 0)
  u64 t_first;             // first CTA's arrival at this barrier
  u64 t_rel;               // release (after the scheduler step and this record)
};

__device__ __forceinline__ u64 globaltimer() {
  u64 t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

struct Params {
  const uint2* rowc;      // [V+1] {start, heavy} (u32 arc offsets)
  const uint2* arcs;      // [A] {dst, wbits}
  u32* dist;              // [V]
  u32* xd;                // [5V] sweep fall-back marks [0, V); pull candidate lists [V, 3V);
                          // pull long-scan items uint4 [V/2] from 3V rounded up to 4 (+4 slack)
  Ctl* ctl;
  SlotCtl* sc;            // [K]
  u64* items;             // [K * cap]
  u64* hub_items;         // [hub_cap]
  unsigned long long* stats;  // [ST_N]
  TraceEnt* trace;            // [TRACE_CAP] barrier timeline of the last run, then [SAMPLE_CAP]
                              // phase-1 claim samples
  u32* p2o;  // [cap] edge-balanced phase 2: first heavy-arc rank of each compacted entry,
             // followed by uint2 [cap] {arc index - rank, d} (see p2_compact)
  u32 V, K, kmask, cap, hub_cap;
  u32 delta_u;       // u32 graphs: integer Delta >= 1
  float inv_delta;   // f32 graphs: fl32(1/Delta)
  u32 delta_bits;    // light iff wbits < delta_bits
  u32 claim_max;
  // ablation flags (bit 0 ADWL: adaptive thread/warp/CTA bins + hub chunks, 0 = thread per
  // vertex; bit 1 SYNC: level-synchronous phase 1, a grid barrier per frontier level = BL;
  // bit 2 EB: edge-balanced phase 2 for settled ranges of >= (flags >> 8) & 0x7FFFFF entries;
  // bit 7 PULL: pull-style phases 2&3 for large buckets (symmetric graphs, PRO; f32 graphs
  // then carry Delta's bits in delta_u);
  // bits 3/4 adaptive Delta reading A/B (NEXT-1); bit 5 f32 weights (theta level bits)).
  // Params stays <= 128 bytes: larger, it spills around the out-of-line pb_flush call.
  u32 flags;
};

static_assert(sizeof(Params) <= 128, "Params > 128 B spills around the out-of-line pb_flush call");

constexpr u32 TASK = 32 * UNROLL;  // arcs per warp task
constexpr u32 BATCH = DS_THREADS * IPT;        // queue items per phase-1 CTA batch
constexpr u32 BATCH_MAX = DS_THREADS * IPT_MAX;
constexpr u32 SB_CAP = 32 * IPT_MAX;           // thread-bin entries per warp
#ifndef SSSP_PB_CAP
#define SSSP_PB_CAP 128u  // (128 beats 256 and 64, profiles/r02)
#endif
constexpr u32 PB_CAP = SSSP_PB_CAP;  // staged pushes per warp (>= 32 * UNROLL)
constexpr u32 LOC_CAP = BATCH;       // CTA-local chase list: one phase-1 batch
constexpr u32 LOCAL_CHASE = 1u << 16;  // Params::claim_max bit (claim_max itself <= BATCH) ...
constexpr u32 LOCAL_LIM_SHIFT = 20;     // ... and bits 20-31: entries kept locally (1..LOC_CAP)
constexpr u32 LOCAL_LIM_MASK = 4095u;
static_assert(BATCH < LOCAL_CHASE, "claim_max must fit below the LOCAL_CHASE bit");
static_assert(LOC_CAP <= LOCAL_LIM_MASK, "local-chase limit field too narrow for LOC_CAP");

// What pb_flush needs, kept in shared memory (Smem::fctx) so the out-of-line call takes no
// parameter registers.
struct FlushCtx {
  SlotCtl* sc;
  u64* items;
  Ctl* ctl;
  u32* xd;
  u32* dist;
  u64 dmul;  // u32 graphs: ceil(2^64 / delta_u), so d / delta_u = umulhi64(d, dmul) exactly
  u32 cap, kmask, delta_u;
  float inv_delta;
};

struct Smem {
  // Task pool of one batch. Tasks [0, S): 128-arc slices of each warp's
  // thread bin (small vertices, arcs spread by a warp prefix sum); tasks
  // [S, S+R): 128-arc slices of the range list (warp-bin vertices, CTA-bin
  // vertices and hub chunks: a 256..4096-arc vertex is spread over the CTA's
  // 8 warps = "CTA per vertex"; a 32..255-arc one takes 1-2 tasks = "warp per
  // vertex"). Any warp may run any task, so warps stay balanced.
  u32 rl_beg[BATCH_MAX];
  u32 rl_len[BATCH_MAX];
  u32 rl_d[BATCH_MAX];
  u32 rl_toff[BATCH_MAX + 1];
  u32 sb_beg[DS_WARPS][SB_CAP];
  u32 sb_off[DS_WARPS][SB_CAP];
  u32 sb_d[DS_WARPS][SB_CAP];
  u32 sb_n[DS_WARPS];
  u32 sb_total[DS_WARPS];
  u32 sb_toff[DS_WARPS + 1];  // first thread-bin task of each warp
  u64 scan_ws[DS_WARPS];
  u32 rl_n, rl_tasks, task_next;
  u64 pb[DS_WARPS][PB_CAP];  // staged pushes (d << 32 | v), bucket resolved at flush
  u32 pb_n[DS_WARPS];
  u32 fc[DS_WARPS][64];      // pb_flush: entries per ring slot, then each slot's next position
  FlushCtx fctx;
  unsigned long long st[ST_N];
  unsigned long long wst[DS_WARPS][ST_N];  // per-warp counters (st_add), summed at kernel end
  u32 claim_h, claim_n, claim_src;
  // CTA-local chase (LOCAL_CHASE): phase-1 pushes into the current bucket kept in shared
  // memory and processed by this CTA next, without the global queue round trip
  u64 loc[LOC_CAP];
  u32 loc_n, loc_on, loc_lim;
  // control snapshot
  u32 mode, cur, lim, p2_begin, p2_end, sweep_first, round_end;
  u32 cur_end, rowc_off, theta_bits;  // bucket end (fine slots), light/heavy level
  u32 pull_sel, pull_n_in;            // pull phases 2&3: input candidate list
  u32 bf;                             // Bellman-Ford end: phase 1 relaxes every arc
};

// ---------------------------------------------------------------- helpers --
#ifndef SSSP_LD_VOLATILE
#define SSSP_LD_VOLATILE 0  // 0: probes and arc loads as plain asm (A/B: C4 -2 %, C3 -2 %, C1 -1 %)
#endif
#if SSSP_LD_VOLATILE
#define SSSP_LD_ASM asm volatile
#else
#define SSSP_LD_ASM asm  // probes and arc loads are pure loads: let the compiler schedule them
#endif
// Filter probe of dist[] before the atomicMin (Alg. 1 l.2). Any value ever
// stored in dist[v] is >= its current value, so a stale (L1-cached) read can
// only cause an extra atomic, never a missed improvement.
__device__ __forceinline__ u32 ld_probe(const u32* p, bool pred, u64 pol) {
  u32 v;
#if SSSP_PROBE_L1
  SSSP_LD_ASM(
      "{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n mov.b32 %0, 0;\n"
      " @q ld.global.ca.L2::cache_hint.u32 %0, [%1], %3;\n}"
      : "=r"(v)
      : "l"(p), "r"((u32)pred), "l"(pol));
#else
  SSSP_LD_ASM(
      "{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n mov.b32 %0, 0;\n"
      " @q ld.global.cg.L2::cache_hint.u32 %0, [%1], %3;\n}"
      : "=r"(v)
      : "l"(p), "r"((u32)pred), "l"(pol));
#endif
  return v;
}

// Predicated arc load (streamed: L1 bypass, L2 evict-first). {0,0} if !pred.
__device__ __forceinline__ uint2 ld_arc(const uint2* p, bool pred, u64 pol) {
  uint2 v;
  SSSP_LD_ASM(
      "{\n .reg .pred q;\n setp.ne.b32 q, %3, 0;\n mov.b32 %0, 0;\n mov.b32 %1, 0;\n"
      " @q ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %4;\n}"
      : "=r"(v.x), "=r"(v.y)
      : "l"(p), "r"((u32)pred), "l"(pol));
  return v;
}

// Predicated atomicMin keeping dist[] L2-resident (evict_last). Returns the
// old value, or 0 when !pred (so "nd < old" is false). All UNROLL atomics of
// a group are issued before any result is consumed.
__device__ __forceinline__ u32 atomic_min_keep(u32* p, u32 v, bool pred, u64 pol) {
  u32 old;
  asm volatile(
      "{\n .reg .pred q;\n setp.ne.b32 q, %3, 0;\n mov.b32 %0, 0;\n"
      " @q atom.relaxed.gpu.global.min.L2::cache_hint.u32 %0, [%1], %2, %4;\n}"
      : "=r"(old)
      : "l"(p), "r"(v), "r"((u32)pred), "l"(pol)
      : "memory");
  return old;
}

__device__ __forceinline__ u64 policy_evict_first() {
  u64 pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

template <bool F32>
__device__ __forceinline__ u32 relax_add(u32 d, u32 w, u32* err) {
  if (F32) {
    return __float_as_uint(__fadd_rn(__uint_as_float(d), __uint_as_float(w)));  // Alg. 1 l.1
  } else {
    u64 s = (u64)d + w;
    if (s >= (u64)NONE) {
      atomicOr(err, ERR_OVERFLOW);
      return NONE;  // treated as "no improvement"
    }
    return (u32)s;
  }
}

template <bool F32>
__device__ __forceinline__ u32 bucket_of(const Params& p, u32 d) {
  if (F32) {
    u32 b = __float2uint_rz(__fmul_rn(__uint_as_float(d), p.inv_delta));
    return b >= NONE ? NONE - 1 : b;
  } else {
    return d / p.delta_u;
  }
}

__device__ __forceinline__ void st_add(Smem& sm, int k, u32 x) {
  u32 s = __reduce_add_sync(SSSP_FULL_MASK, x);
  if (lane_id() == 0 && s) sm.wst[threadIdx.x >> 5][k] += s;  // this warp's row: no atomic
}

// Publish warp w's staged pushes: per 32 entries, one global reservation per
// distinct bucket queue (tail and pend in one atomicAdd). Entries beyond the
// ring horizon or a full queue are dropped and recorded in far_min. In the
// sweep fall-back (nearb != NONE) entries of bucket nearb mark xd[] instead.

template <bool F32>
__device__ __forceinline__ u32 bucket_of_f(const FlushCtx& p, u32 d) {
  if (F32) {
    u32 b = __float2uint_rz(__fmul_rn(__uint_as_float(d), p.inv_delta));
    return b >= NONE ? NONE - 1 : b;
  } else {
    // floor(d / delta_u) as a 64-bit multiply-high: with dmul = ceil(2^64 / D) the error is
    // below d / 2^64 < 2^-32, less than the gap between d / D and the next integer
    return p.delta_u == 1 ? d : (u32)__umul64hi((u64)d, p.dmul);
  }
}

// Publish warp w's staged pushes. Entries beyond the ring horizon or a full queue are
// dropped and recorded in far_min; in the sweep fall-back (nearb != NONE) entries of bucket
// nearb mark xd[] instead; with the CTA-local chase, current-bucket entries stay in the CTA.
// Reservations (tail and pend in one atomicAdd on the slot's control word): every CTA
// pushing into a bucket hits that one word, and on C4 the peak bucket's word saturated the
// L2's same-address atomic rate (ncu: ~28 % of all stall samples waited on it). So a flush
// of more than 32 entries makes two passes -- classify and count per ring slot, one
// atomicAdd per non-empty slot (all in flight together), then place -- instead of one
// reservation per slot per 32 entries; a flush of <= 32 entries (thin frontiers, C2) keeps
// the single pass and its shorter latency. (Measured on C4: one flush waiting a single round
// trip -- reservations issued while the candidates' atomics are in flight, dead entries for
// the losers -- was 7 % slower than this: profiles/r02/ab_flush_merged_negative.txt.)
template <bool F32>
__device__ __noinline__ void pb_flush_impl(Smem& sm, u32 lim, u32 nearb) {
  const FlushCtx& p = sm.fctx;
  const u32 lane = lane_id(), w = threadIdx.x >> 5;
  const u32 n = sm.pb_n[w];
  {  // pass 0: the staged relaxations' atomicMin (Alg. 1 l.3, SSSP_DEFER_ATOMICS), four rounds
     // in flight; an entry that did not lower dist[v] is dropped (SENTINEL), an applied one
     // (stage_pushes<.., true>) only loses its flag
    const u64 pol_keep = policy_evict_last();
    constexpr int AR = 4;
    u32 nsurv = 0;
    for (u32 i0 = 0; i0 < n; i0 += 32 * AR) {
      u64 e[AR];
      u32 old[AR];
#pragma unroll
      for (int r = 0; r < AR; ++r) {
        const u32 i = i0 + r * 32 + lane;
        e[r] = i < n ? sm.pb[w][i] : SENTINEL;
        const bool need = e[r] != SENTINEL && !((u32)e[r] & APPLIED_FLAG);
        old[r] = atomic_min_keep(p.dist + (u32)e[r], (u32)(e[r] >> 32), need, pol_keep);
      }
#pragma unroll
      for (int r = 0; r < AR; ++r) {
        if (e[r] == SENTINEL) continue;
        const u32 i = i0 + r * 32 + lane;
        const bool applied = ((u32)e[r] & APPLIED_FLAG) != 0;
        if (applied || (u32)(e[r] >> 32) < old[r]) {
          if (applied) sm.pb[w][i] = e[r] & ~(u64)APPLIED_FLAG;
          ++nsurv;
        } else {
          sm.pb[w][i] = SENTINEL;
        }
      }
    }
    nsurv = __reduce_add_sync(SSSP_FULL_MASK, nsurv);
    if (lane == 0) sm.wst[w][ST_UPDATES] += nsurv;
    __syncwarp();
  }
  const u32 c0 = sm.cur, ce = sm.cur_end;
  // entry -> (keep for the global queue?, ring slot, bucket); handles the dropped cases
  auto classify = [&](u64 e, bool ok, u32& x, u32& slot) -> bool {
    const u32 v = (u32)e, nd = (u32)(e >> 32);
    x = ok ? bucket_of_f<F32>(p, nd) : 0u;
    const bool in_cur = x - c0 < ce - c0;  // current bucket [cur, cur_end): its queue is slot cur
    if (ok && nearb != NONE && in_cur) {
      st_relaxed_u32(p.xd + v, NONE);
      st_relaxed_u32(&p.ctl->changed, 1u);
      ok = false;
    }
    // CTA-local chase: this CTA relaxes the vertex itself in its next batch. Only enabled
    // when no arc is heavy at this Delta (phase 2 then needs no settled list in the queue).
    const bool lc = ok && in_cur && sm.loc_on;
    const u32 lm = __ballot_sync(SSSP_FULL_MASK, lc);
    if (lm) {
      const u32 ld = __ffs(lm) - 1;
      u32 base = 0;
      if (lane == ld) base = atomicAdd(&sm.loc_n, (u32)__popc(lm));
      base = __shfl_sync(SSSP_FULL_MASK, base, ld);
      const u32 li = base + __popc(lm & lanemask_lt());
      if (lc && li < sm.loc_lim) {  // the rest goes to the global queue, where idle CTAs find it
        sm.loc[li] = e;
        ok = false;
      }
    }
    if (ok && x > lim) {  // beyond the ring horizon: rescan later
      atomicMin(&p.ctl->far_min, x);
      ok = false;
    }
    slot = (in_cur ? c0 : x) & p.kmask;
    return ok;
  };
  auto place = [&](u64 e, u32 x, u32 slot, u32 idx) {
    if (idx < p.cap) {
      st_relaxed_u64(p.items + (u64)slot * p.cap + idx, e);
    } else {  // queue full: undo the pending count, recover later
      atomicAdd(&p.sc[slot].word, ~0ULL);
      atomicMin(&p.ctl->far_min, x);
    }
  };
  if (n <= 32) {
    const u64 e0 = lane < n ? sm.pb[w][lane] : SENTINEL;
    const bool has = e0 != SENTINEL;
    const u64 e = has ? e0 : 0ULL;
    u32 x, slot;
    const bool ok = classify(e, has, x, slot);
    const u32 m = __ballot_sync(SSSP_FULL_MASK, ok);
    if (ok) {
      const u32 peers = __match_any_sync(m, slot);
      const u32 leader = __ffs(peers) - 1;
      const u32 cnt = __popc(peers);
      u64 old = 0;
      if (lane == leader) old = atomicAdd(&p.sc[slot].word, ((u64)cnt << 32) | cnt);
      old = __shfl_sync(peers, old, leader);
      place(e, x, slot, (u32)(old >> 32) + __popc(peers & lanemask_lt()));
    }
  } else {
    u32* fc = sm.fc[w];
    const u32 K = p.kmask + 1;
    for (u32 k = lane; k < K; k += 32) fc[k] = 0;
    __syncwarp();
    for (u32 i0 = 0; i0 < n; i0 += 32) {  // pass 1: classify, count per slot
      const u32 i = i0 + lane;
      const u64 e0 = i < n ? sm.pb[w][i] : SENTINEL;
      const bool has = e0 != SENTINEL;
      const u64 e = has ? e0 : 0ULL;
      u32 x, slot;
      const bool ok = classify(e, has, x, slot);
      if (has && !ok) sm.pb[w][i] = SENTINEL;  // handled (or dropped) here
      const u32 m = __ballot_sync(SSSP_FULL_MASK, ok);
      if (ok) {
        const u32 peers = __match_any_sync(m, slot);
        if (lane == __ffs(peers) - 1) fc[slot] += __popc(peers);
      }
      __syncwarp();
    }
    for (u32 k = lane; k < K; k += 32) {  // one reservation per non-empty slot
      const u32 c = fc[k];
      if (c) fc[k] = (u32)(atomicAdd(&p.sc[k].word, ((u64)c << 32) | c) >> 32);
    }
    __syncwarp();
    for (u32 i0 = 0; i0 < n; i0 += 32) {  // pass 2: place at the reserved positions
      const u32 i = i0 + lane;
      const u64 e = i < n ? sm.pb[w][i] : SENTINEL;
      const bool ok = e != SENTINEL;
      u32 x = 0, slot = 0;
      if (ok) {
        x = bucket_of_f<F32>(p, (u32)(e >> 32));
        slot = (x - c0 < ce - c0 ? c0 : x) & p.kmask;
      }
      const u32 m = __ballot_sync(SSSP_FULL_MASK, ok);
      u32 base = 0, peers = 0;
      if (ok) {
        peers = __match_any_sync(m, slot);
        base = fc[slot];
      }
      __syncwarp();
      if (ok) {
        if (lane == __ffs(peers) - 1) fc[slot] = base + __popc(peers);
        place(e, x, slot, base + __popc(peers & lanemask_lt()));
      }
      __syncwarp();
    }
  }
  __syncwarp();
  if (lane == 0) sm.pb_n[w] = 0;
  __syncwarp();
}

template <bool F32>
__device__ __forceinline__ void pb_flush(const Params& p, Smem& sm, u32 lim, u32 nearb) {
  pb_flush_impl<F32>(sm, lim, nearb);
}

// Stage up to UNROLL pushes per lane into the warp's buffer (all 32 lanes). APPLIED: dist[v]
// already holds nd (the entry only needs queueing); otherwise the entry is a relaxation
// candidate whose atomicMin pb_flush issues (SSSP_DEFER_ATOMICS).
template <bool F32, bool APPLIED = true>
__device__ __forceinline__ void stage_pushes(const Params& p, Smem& sm, u32 lim, u32 nearb,
                                             const bool (&want)[UNROLL], const u32 (&v)[UNROLL],
                                             const u32 (&nd)[UNROLL]) {
  u32 m[UNROLL], tot = 0;
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    m[k] = __ballot_sync(SSSP_FULL_MASK, want[k]);
    tot += __popc(m[k]);
  }
  if (!tot) return;
  const u32 w = threadIdx.x >> 5, lt = lanemask_lt();
  if (sm.pb_n[w] + tot > PB_CAP) pb_flush<F32>(p, sm, lim, nearb);
  u32 base = sm.pb_n[w];
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    if (want[k]) sm.pb[w][base + __popc(m[k] & lt)] = ((u64)nd[k] << 32) | (v[k] | (APPLIED ? APPLIED_FLAG : 0u));
    base += __popc(m[k]);
  }
  __syncwarp();
  if (lane_id() == 0) sm.pb_n[w] = base;
  __syncwarp();
}

// Relax UNROLL arcs per thread (independent loads in flight: arcs, then dist
// probes, then atomics). PH 1 = light arcs, PH 2 = heavy arcs; without PRO the
// light/heavy split is a per-arc predicate (the divergence PRO removes).
// Relax UNROLL arcs per thread in two steps so consecutive tasks overlap:
// arcs_issue() starts the (streamed) arc loads of the next task before
// relax_finish() of the current one waits on its dist probes and atomics.
// PH 1 = light arcs, PH 2 = heavy arcs; without PRO the light/heavy split is
// a per-arc predicate (the divergence PRO removes).
__device__ __forceinline__ void arcs_issue(const Params& p, const u32 (&idx)[UNROLL],
                                           const bool (&valid)[UNROLL], uint2 (&a)[UNROLL]) {
  const u64 pol_stream = policy_evict_first();
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) a[k] = ld_arc(p.arcs + idx[k], valid[k], pol_stream);
}

template <bool F32, bool PRO, int PH>
__device__ __forceinline__ void relax_finish(const Params& p, Smem& sm, u32 lim, u32 nearb,
                                             const uint2 (&a)[UNROLL], const bool (&valid)[UNROLL],
                                             const u32 (&d)[UNROLL]) {
  const u64 pol_keep = policy_evict_last();
  u32 nd[UNROLL], cur[UNROLL];
  bool want[UNROLL];
  bool of = false;
#if SSSP_LAT
  long long t0 = 0, t1 = 0, t2 = 0, t3 = 0;
  if (threadIdx.x == 0) {
    t0 = clock64();
    asm volatile("" ::"r"(a[0].x), "r"(a[UNROLL - 1].x));
    t1 = clock64();
  }
#endif
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    bool take = valid[k];
    if (!PRO) take = take && ((PH == 1) ? (a[k].y < sm.theta_bits) : (a[k].y >= sm.theta_bits));
    if (F32) {
      nd[k] = __float_as_uint(__fadd_rn(__uint_as_float(d[k]), __uint_as_float(a[k].y)));  // Alg. 1 l.1
    } else {
      const u64 sum = (u64)d[k] + a[k].y;  // exact; >= 0xFFFFFFFF is an overflow
      const bool o = take && sum >= (u64)NONE;
      of |= o;
      take = take && !o;
      nd[k] = (u32)sum;
    }
    want[k] = take;
    cur[k] = ld_probe(p.dist + a[k].x, take, pol_keep);
  }
  if (!F32 && of) atomicOr(&p.ctl->err, ERR_OVERFLOW);
#if SSSP_LAT
  if (threadIdx.x == 0) {
    asm volatile("" ::"r"(cur[0]), "r"(cur[UNROLL - 1]));
    t2 = clock64();
  }
  u32 n_atoms = 0;
#endif
  u32 vv[UNROLL];
#if SSSP_DEFER_ATOMICS
  // Alg. 1 l.2 here; the atomicMin of l.3 is issued by pb_flush for every staged candidate
  // of the warp at once (a warp no longer waits one L2 atomic round trip per task)
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    want[k] = want[k] && nd[k] < cur[k];
    vv[k] = a[k].x;
#if SSSP_LAT
    n_atoms += want[k];
#endif
  }
#if SSSP_LAT
  st_add(sm, ST_ATOMS, n_atoms);
#endif
#else
  u32 old[UNROLL];
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    want[k] = want[k] && nd[k] < cur[k];  // check before the atomic (Alg. 1 l.2)
#if SSSP_LAT
    n_atoms += want[k];
#endif
    old[k] = atomic_min_keep(p.dist + a[k].x, nd[k], want[k], pol_keep);  // Alg. 1 l.3
  }
#if SSSP_LAT
  st_add(sm, ST_ATOMS, n_atoms);
#endif
#pragma unroll
  for (int k = 0; k < UNROLL; ++k) {
    want[k] = want[k] && nd[k] < old[k];
    vv[k] = a[k].x;
  }
#endif
#if SSSP_LAT
  if (threadIdx.x == 0) {
#if !SSSP_DEFER_ATOMICS
    asm volatile("" ::"r"(old[0]), "r"(old[UNROLL - 1]));
#endif
    t3 = clock64();
  }
#endif
  stage_pushes<F32, !SSSP_DEFER_ATOMICS>(p, sm, lim, nearb, want, vv, nd);
#if SSSP_LAT
  if (threadIdx.x == 0) {
    const long long t4 = clock64();
    sm.st[ST_L_ARC] += (unsigned long long)(t1 - t0);
    sm.st[ST_L_PROBE] += (unsigned long long)(t2 - t1);
    sm.st[ST_L_ATOM] += (unsigned long long)(t3 - t2);
    sm.st[ST_L_STAGE] += (unsigned long long)(t4 - t3);
    sm.st[ST_L_N] += 1;
  }
#endif
}


// ------------------------------------------------------------ batch -------
// Batch item q (0 <= q < n) lives in thread (x % 8) * 32 + x / 8 of round
// r = q / 256 (x = q % 256): consecutive items are spread over the 8 warps.
__device__ __forceinline__ u32 batch_item_index(u32 r) {
  return r * DS_THREADS + (threadIdx.x & 31) * DS_WARPS + (threadIdx.x >> 5);
}

// Process the CTA's claimed items (IPT per thread; has[i] = holds item i).
// src: SRC_QUEUE phase-1 queue, SRC_STATIC phase-2 static range, SRC_HUB
// phase-2 hub queue, SRC_SWEEP fall-back sweep over dist[] (no queue pushes
// into the current bucket, hubs stay in the range list).
template <bool F32, bool PRO, int PH, int N, bool ADWL = true, bool EXT = false>
__device__ __forceinline__ void process_batch(const Params& p, Smem& sm, const u64 (&it)[N],
                                              const bool (&has)[N], u32 lim, u32 src, u32 slot) {
  const u32 tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const bool sweep = src == SRC_SWEEP;
  const u32 nearb = sweep ? sm.cur : NONE;
  const long long t_enter = tid == 0 ? clock64() : 0;
#if SSSP_LAT && SSSP_BATCH_SAMPLES
  const unsigned long long lat0_probe = tid == 0 ? sm.st[ST_L_PROBE] : 0ULL;
  const unsigned long long lat0_stage = tid == 0 ? sm.st[ST_L_STAGE] : 0ULL;
#endif
  // ---- decode: all dist probes and row loads of the thread's items in flight at once
  u32 cls[N], beg[N], len[N], d[N];
  u32 cd[N];
#pragma unroll
  for (int i = 0; i < N; ++i) {
    const u32 lo = (u32)it[i];
    cls[i] = 0;
    cd[i] = has[i] ? ld_cg(p.dist + (lo & ~CHUNK_FLAG)) : 0u;
  }
  // item range for phase PH: PRO -> light [start, heavy) / heavy [heavy, end); no PRO -> the
  // whole adjacency (predicate per arc). (Loading the rows with the dist probe, for stale
  // entries too, measured 4 % slower on C4.)
  const uint2* rowc = EXT ? p.rowc + sm.rowc_off : p.rowc;  // heavy offsets of the bucket's level
  const bool bf_all = PH == 1 && sm.bf;  // Bellman-Ford end: phase 1 relaxes every arc
  auto range_of = [&](int i, i64& b, i64& e) {
    const u32 v = (u32)it[i] & ~CHUNK_FLAG;
    const uint2 r = rowc[v];
    if (PRO && PH == 1 && !bf_all) {
      b = r.x;
      e = r.y;
    } else {  // heavy range, the whole adjacency (no PRO) or, in the Bellman-Ford end, all arcs
      e = rowc[v + 1].x;
      b = (PRO && PH == 2) ? r.y : r.x;
    }
  };
  u32 c_settled = 0, c_stale = 0, c_arcs = 0, c_chunks = 0, c_w = 0, c_c = 0, c_t = 0;
#pragma unroll
  for (int i = 0; i < N; ++i) {
    beg[i] = 0;
    len[i] = 0;
    d[i] = 0;
    if (!has[i]) continue;
    const u32 lo = (u32)it[i], hi = (u32)(it[i] >> 32);
    const bool is_chunk = (lo & CHUNK_FLAG) != 0;
    const u32 v = lo & ~CHUNK_FLAG;
    if (is_chunk) {
      // Chunk items in the phase-2 static range are phase-1 work already done.
      if (!(PH == 2 && src == SRC_STATIC)) {
        i64 rb, re;
        range_of(i, rb, re);
        const i64 b = rb + (i64)hi * HUB_CHUNK;
        beg[i] = (u32)b;
        len[i] = (u32)min((i64)HUB_CHUNK, re - b);
        d[i] = cd[i];  // current distance: a valid path length (<= spawning d)
        c_arcs += len[i];
        cls[i] = 2;
      }
    } else {
      d[i] = hi;
      const bool live = (PH == 1) ? (hi <= cd[i]) : (hi == cd[i]);  // stale / settled-final filter
      if (!live) {
        c_stale += (PH == 1);
      } else {
        c_settled += 1;
        i64 rb, re;
        range_of(i, rb, re);
        const i64 l = re - rb;
        if (!ADWL) {  // ablation: the vertex's own thread walks all its arcs
          beg[i] = (u32)rb;
          len[i] = (u32)l;
          cls[i] = l > 0 ? 3 : 0;
          c_arcs += (u32)l;
          c_t += l > 0;
        } else if (l > (i64)HUB_CHUNK && !sweep) {  // hub: ceil(l/4096) chunks any CTA may claim
          const u32 nc = (u32)((l + HUB_CHUNK - 1) / HUB_CHUNK);
          c_chunks += nc;
          u64* word = (PH == 1) ? &p.sc[slot].word : &p.ctl->hub_word;
          u64* q = (PH == 1) ? p.items + (u64)slot * p.cap : p.hub_items;
          const u32 qcap = (PH == 1) ? p.cap : p.hub_cap;
          const u32 base = (u32)(atomicAdd(word, ((u64)nc << 32) | nc) >> 32);
          for (u32 c = 0; c < nc; ++c) {
            if (base + c < qcap) {
              st_relaxed_u64(q + base + c, ((u64)c << 32) | CHUNK_FLAG | v);
            } else {
              atomicAdd(word, ~0ULL);
              if (PH == 1)
                atomicMin(&p.ctl->far_min, sm.cur);  // lost phase-1 work: sweep this bucket
              else
                atomicOr(&p.ctl->err, ERR_INTERNAL);
            }
          }
        } else if (l >= (i64)BIN_WARP) {
          beg[i] = (u32)rb;
          len[i] = (u32)l;
          cls[i] = 2;
          c_arcs += (u32)l;
          if (l >= (i64)BIN_CTA)
            ++c_c;
          else
            ++c_w;
        } else if (l > 0) {
          beg[i] = (u32)rb;
          len[i] = (u32)l;
          cls[i] = 1;
          c_arcs += (u32)l;
          ++c_t;
        }
      }
    }
  }
#if SSSP_PREFETCH
#pragma unroll
  for (int i = 0; i < N; ++i)
    if (cls[i]) prefetch_l2(p.arcs + beg[i], len[i] * (u32)sizeof(uint2));
#endif
  if (!ADWL) {  // ablation (no ADWL): static thread-per-vertex relaxation
#pragma unroll 1
    for (int i = 0; i < N; ++i) {
      const u32 l = cls[i] == 3 ? len[i] : 0u;
      const u32 maxl = __reduce_max_sync(SSSP_FULL_MASK, l);
      for (u32 j0 = 0; j0 < maxl; j0 += UNROLL) {
        u32 idx[UNROLL], dd[UNROLL];
        bool valid[UNROLL];
        uint2 a[UNROLL];
#pragma unroll
        for (int k = 0; k < UNROLL; ++k) {
          valid[k] = j0 + k < l;
          idx[k] = beg[i] + j0 + k;
          dd[k] = d[i];
        }
        arcs_issue(p, idx, valid, a);
        relax_finish<F32, PRO, PH>(p, sm, lim, nearb, a, valid, dd);
      }
    }
  }
  // ---- stats (warp-aggregated)
  st_add(sm, PH == 1 ? ST_SETTLED : ST_HEAVYV, c_settled);
  if (PH == 2) {  // C_i: vertices settled in bucket cur (trace; adaptive Delta, Eq. (1))
    const u32 cs = __reduce_add_sync(SSSP_FULL_MASK, c_settled);
    if (lane == 0 && cs) atomicAdd(&p.ctl->csum, cs);
  }
  if (PH == 1) st_add(sm, ST_STALE, c_stale);
  st_add(sm, PH == 1 ? ST_LIGHT : ST_HEAVY, c_arcs);
  st_add(sm, ST_CHUNKS, c_chunks);
  st_add(sm, ST_BIN_T, c_t);
  st_add(sm, ST_BIN_W, c_w);
  st_add(sm, ST_BIN_C, c_c);

  // ---- stage: thread bin (warp prefix sums) and range list (block scan)
  {
    u32 ns = 0, ls = 0, nl = 0, tl = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      ns += cls[i] == 1;
      ls += cls[i] == 1 ? len[i] : 0u;
      nl += cls[i] == 2;
      tl += cls[i] == 2 ? (len[i] + TASK - 1) / TASK : 0u;
    }
    u32 tot_ns, tot_ls;
    u32 pos = warp_exclusive_scan(ns, &tot_ns);
    u32 off = warp_exclusive_scan(ls, &tot_ls);
#pragma unroll
    for (int i = 0; i < N; ++i) {
      if (cls[i] == 1) {
        sm.sb_beg[w][pos] = beg[i];
        sm.sb_off[w][pos] = off;
        sm.sb_d[w][pos] = d[i];
        ++pos;
        off += len[i];
      }
    }
    const u64 x = ((u64)nl << 32) | tl;
    u64 wt;
    const u64 ex = warp_exclusive_scan(x, &wt);
    if (lane == 31) {
      sm.scan_ws[w] = wt;
      sm.sb_n[w] = tot_ns;
      sm.sb_total[w] = tot_ls;
    }
    __syncthreads();
    u64 acc = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < DS_WARPS; ++i) {
      const u64 sv = sm.scan_ws[i];
      if (i < (int)w) acc += sv;
      tot += sv;
    }
    u32 li = (u32)((ex + acc) >> 32), lt = (u32)(ex + acc);
#pragma unroll
    for (int i = 0; i < N; ++i) {
      if (cls[i] == 2) {
        sm.rl_beg[li] = beg[i];
        sm.rl_len[li] = len[i];
        sm.rl_d[li] = d[i];
        sm.rl_toff[li] = lt;
        ++li;
        lt += (len[i] + TASK - 1) / TASK;
      }
    }
    if (tid <= DS_WARPS) {  // thread-bin task offsets per warp
      u32 a = 0;
      for (int i = 0; i < (int)tid; ++i) a += (sm.sb_total[i] + TASK - 1) / TASK;
      sm.sb_toff[tid] = a;
    }
    if (tid == 0) {
      sm.rl_n = (u32)(tot >> 32);
      sm.rl_tasks = (u32)tot;
      sm.rl_toff[(u32)(tot >> 32)] = (u32)tot;
      sm.task_next = 0;
    }
  }
  __syncthreads();  // task pool complete
  long long t_pool = 0;
  if (tid == 0) {
    t_pool = clock64();
    sm.st[ST_P_STAGE] += (unsigned long long)(t_pool - t_enter);
    sm.st[ST_P_NB] += 1;
  }

  const u32 S = sm.sb_toff[DS_WARPS];
  const u32 ntask = S + sm.rl_tasks, nl = sm.rl_n;
  if (tid == 0) sm.st[ST_P_NT] += ntask;
  // Task descriptor -> per-lane arc indices / distances (smem lookups only).
  u32 rl_cur = 0;  // SSSP_STATIC_TASKS: this warp's current range-list entry
  auto setup = [&](u32 t, u32 (&idx)[UNROLL], bool (&valid)[UNROLL], u32 (&dd)[UNROLL]) {
    if (t >= ntask) {
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        valid[k] = false;
        idx[k] = 0;
        dd[k] = 0;
      }
    } else if (t < S) {  // thread-bin slice of warp ww
      u32 ww = 0;
#pragma unroll
      for (int i = 1; i < DS_WARPS; ++i) ww += (t >= sm.sb_toff[i]);
      const u32 j0 = (t - sm.sb_toff[ww]) * TASK, total = sm.sb_total[ww], ne = sm.sb_n[ww];
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        const u32 j = j0 + k * 32 + lane;
        valid[k] = j < total;
        u32 o = 0;  // owner: last entry with sb_off <= j
#pragma unroll
        for (u32 step = SB_CAP / 2; step; step >>= 1)
          if (o + step < ne && sm.sb_off[ww][o + step] <= j) o += step;
        idx[k] = sm.sb_beg[ww][o] + (j - sm.sb_off[ww][o]);
        dd[k] = sm.sb_d[ww][o];
      }
    } else {  // range-list slice
      const u32 tr = t - S;
#if SSSP_STATIC_TASKS
      // a warp's tasks ascend by DS_WARPS: walk on from its previous entry
      u32 lo = rl_cur;
      while (lo + 1 < nl && sm.rl_toff[lo + 1] <= tr) ++lo;
      rl_cur = lo;
#else
      u32 lo = 0, hi = nl;  // entry i with toff[i] <= tr < toff[i+1]
      while (hi - lo > 1) {
        const u32 mid = (lo + hi) >> 1;
        if (sm.rl_toff[mid] <= tr)
          lo = mid;
        else
          hi = mid;
      }
#endif
      const u32 sub = (tr - sm.rl_toff[lo]) * TASK;
      const u32 b = sm.rl_beg[lo] + sub;
      const u32 l = sm.rl_len[lo] - sub;
      const u32 dv = sm.rl_d[lo];
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        const u32 j = k * 32 + lane;
        valid[k] = j < l;
        idx[k] = b + j;
        dd[k] = dv;
      }
    }
  };
#if SSSP_STATIC_TASKS
  u32 t_next = w;  // round-robin: tasks cost about the same (<= 64 arcs, latency-bound)
  auto claim = [&]() {
    const u32 t = t_next;
    t_next += DS_WARPS;
    return t;
  };
#else
  auto claim = [&]() {
    u32 t = 0;
    if (lane == 0) t = atomicAdd(&sm.task_next, 1u);
    return __shfl_sync(SSSP_FULL_MASK, t, 0);
  };
#endif
  u32 idx[UNROLL], dd[UNROLL];
  bool valid[UNROLL];
  uint2 a[UNROLL];
  u32 t = claim();
  setup(t, idx, valid, dd);
  arcs_issue(p, idx, valid, a);
  while (t < ntask) {
    const u32 t2 = claim();
    u32 idx2[UNROLL], dd2[UNROLL];
    bool valid2[UNROLL];
    uint2 a2[UNROLL];
    setup(t2, idx2, valid2, dd2);
    arcs_issue(p, idx2, valid2, a2);  // next task's arcs in flight ...
    relax_finish<F32, PRO, PH>(p, sm, lim, nearb, a, valid, dd);  // ... while this one completes
    t = t2;
#pragma unroll
    for (int k = 0; k < UNROLL; ++k) {
      a[k] = a2[k];
      valid[k] = valid2[k];
      dd[k] = dd2[k];
    }
  }
  long long t_task = 0;
  if (tid == 0) {
    t_task = clock64();
    sm.st[ST_P_TASK] += (unsigned long long)(t_task - t_pool);
  }
  if (sm.pb_n[w]) pb_flush<F32>(p, sm, lim, nearb);  // publish before reporting completion
  __syncthreads();
  if (tid == 0) {
    const long long t_end = clock64();
    sm.st[ST_P_TAIL] += (unsigned long long)(t_end - t_task);
    if (SSSP_BATCH_SAMPLES && blockIdx.x % SAMPLE_EVERY == 0) {  // batch timeline (which = 101)
      const u32 k = atomicAdd(&p.ctl->sample_n, 1u);
      if (k < SAMPLE_CAP) {
        TraceEnt e;
        e.t_ns = globaltimer();
        e.which = 101;
        e.cur = sm.cur;
        e.tail = ntask;
#if SSSP_LAT
        e.mode = (u32)(sm.st[ST_L_PROBE] - lat0_probe);  // warp 0's probe-wait cycles in this batch
        e.far_min = (u32)(sm.st[ST_L_STAGE] - lat0_stage);  // ... and push-staging cycles
#else
        e.mode = S;
        e.far_min = nl;
#endif
        e.pad = (u32)(t_end - t_task);
        e.closed_b = blockIdx.x;
        e.closed_c = PH * 10 + src;
        e.t_first = (u64)(t_pool - t_enter);
        e.t_rel = (u64)(t_task - t_pool);
        p.trace[TRACE_CAP + k] = e;
      }
    }
  }
}

// --------------------------------------------------------- grid barrier ---
__device__ __forceinline__ void enter_sweep(volatile Ctl* c) {
  c->csum = 0;  // the heavy sweep counts the bucket's vertices afresh
  c->changed = 0;
  c->sweep_first = 1;
  c->sweeps = c->sweeps + 1;
  c->mode = MODE_SWEEP_LIGHT;
}

// Adaptive Delta (NEXT-1): PAPER Eq. (1)-(2), Alg. 2 l.11
// Update_Delta_Epsilon, with reading R7: the garbled bars are
// absolute values,
//   eps_i = |C_{i-2} - C_{i-1}| / (C_{i-2} + C_{i-1})
//           * (T_{i-2} - T_{i-1}) / (T_{i-2} + T_{i-1}) * Delta_0     (i >= 2; else 0)
//   Delta_i = Delta_{i-1} + eps_i   (reading A; reading B: Delta_0 + eps_i, Fig. 6 text)
// clamped to [Delta_0/4, 4 Delta_0]; C = vertices settled in the bucket
// ("converged vertices"), T = phase-1 queue items of the bucket (one
// thread per active vertex in the paper's master kernel). So more work
// per bucket (T up) narrows the next bucket. Runs on the one
// thread that closes a bucket; the next bucket spans round(Delta_i / g) fine
// slots and its light level is the smallest g * 2^l >= that width.
__device__ void adapt_next(const Params& p, u32 t_i, u32 c_i) {
  volatile Ctl* c = p.ctl;
  const u32 i = c->a_i + 1;
  c->a_c2 = c->a_c1;
  c->a_c1 = c_i;
  c->a_t2 = c->a_t1;
  c->a_t1 = t_i;
  c->a_i = i;
  const float d0 = c->a_d0;
  float eps = 0.f;
  if (i >= 2) {
    const float c2 = (float)c->a_c2, c1 = (float)c->a_c1, t2 = (float)c->a_t2, t1 = (float)c->a_t1;
    if (c2 + c1 > 0.f && t2 + t1 > 0.f) eps = fabsf(c2 - c1) / (c2 + c1) * ((t2 - t1) / (t2 + t1)) * d0;
  }
  float dl = (c->a_mode == 2 ? d0 : c->a_dlt) + eps;
  dl = fminf(fmaxf(dl, 0.25f * d0), 4.f * d0);
  c->a_dlt = dl;
  u32 m = (u32)rintf(dl);
  m = min(max(m, c->a_mmin), c->a_mmax);
  c->a_m = m;
  u32 l = 0;
  while ((1u << l) < m) ++l;
  c->lvl = l;
  const u32 tn = c->trace_n;
  if (tn < TRACE_CAP) {  // (C_i, T_i, next width, Delta_i) for sssp_get_trace
    TraceEnt e;
    e.t_ns = globaltimer();
    e.which = TRACE_ADAPT;
    e.cur = c_i;
    e.tail = t_i;
    e.mode = m;
    e.far_min = __float_as_uint(dl);
    e.pad = i;
    e.closed_b = NONE;
    e.closed_c = 0;
    e.t_first = e.t_rel = e.t_ns;
    p.trace[tn] = e;
    c->trace_n = tn + 1;
  }
}

__device__ __forceinline__ uint4 ld_volatile_v4(const void* q) {
  uint4 r;
  asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(q)
               : "memory");
  return r;
}

// Closing a bucket after its phases 2&3 (SYNC_P2), fixed Delta: the same steps as the
// general path in decide(), but every control word is read up front -- the whole first
// Ctl line and the pull selector in one round trip, the bucket's ring word and the next
// eight ring slots in a second -- instead of one dependent volatile load after another
// (the general path's step cost ~4 us per bucket on C4, profiles/r02). Returns false
// (nothing written) when the general path is needed: adaptive Delta, a heavy relaxation
// that landed back in the bucket (reopen), or no non-empty slot among the next eight.
__device__ bool decide_close_fast(const Params& p) {
  volatile Ctl* c = p.ctl;
  volatile SlotCtl* sc = p.sc;
  u32 W[40];
#pragma unroll
  for (int i = 0; i < 10; ++i) {
    const uint4 x = ld_volatile_v4(reinterpret_cast<const uint4*>(const_cast<Ctl*>(p.ctl)) + i);
    W[4 * i] = x.x;
    W[4 * i + 1] = x.y;
    W[4 * i + 2] = x.z;
    W[4 * i + 3] = x.w;
  }
  static_assert(offsetof(Ctl, cur) == 0 && offsetof(Ctl, lim) == 4 && offsetof(Ctl, mode) == 8 &&
                offsetof(Ctl, far_min) == 12 && offsetof(Ctl, p2_end) == 20 && offsetof(Ctl, epochs) == 28 &&
                offsetof(Ctl, cur_end) == 64 && offsetof(Ctl, a_mode) == 68 && offsetof(Ctl, a_m) == 108 &&
                offsetof(Ctl, csum) == 116 && offsetof(Ctl, bf) == 124 && offsetof(Ctl, pull_sel) == 128 &&
                offsetof(Ctl, bf_t) == 148 && offsetof(Ctl, bf_peak) == 152 && offsetof(Ctl, bar_count) == 256,
                "Ctl layout (decide_close_fast)");
  const u32 cur = W[0], lim0 = W[1], mode = W[2], fm = W[3], p2_end = W[5], epochs = W[7];
  const u32 cur_end = W[16], a_mode = W[17], a_m = W[27], csum = W[29], pull_sel = W[32], bf_t = W[37];
  const u32 bf_peak = W[38];
  if (a_mode) return false;
  const u32 s = cur & p.kmask;
  const u64 ws = sc[s].word;
  u32 t[8];
#pragma unroll
  for (u32 k = 0; k < 8; ++k)
    t[k] = (cur_end + k <= lim0 && cur_end + k >= cur_end) ? (u32)(sc[(cur_end + k) & p.kmask].word >> 32) : 0u;
  if ((u32)ws != 0) return false;  // reopen (f32 rounding): general path
  u32 nxt = NONE, nxt_tail = 0;
#pragma unroll
  for (u32 k = 0; k < 8; ++k)
    if (t[k] && nxt == NONE) {
      nxt = cur_end + k;
      nxt_tail = t[k];
    }
  if (nxt == NONE && cur_end + 8 <= lim0 && cur_end + 8 > cur_end) return false;  // scan further: general path
  const u32 peak = max(bf_peak, min((u32)(ws >> 32), p.cap));
  if (bf_t && nxt != NONE && peak >= 8 * bf_t) {
    // past the peak with few entries left: the general path decides on the Bellman-Ford end
    u32 sum = 0;
#pragma unroll
    for (u32 k = 0; k < 8; ++k) sum += t[k];
    if (sum <= bf_t) return false;
  }
  sc[s].p2 = p2_end;
  c->bf_peak = peak;
  if (mode == MODE_PULL || mode == MODE_PULL_LONG) c->pull_sel = pull_sel == 0 ? 1u : 0u;  // its output list
  c->csum = 0;
  c->closed_c = (p.claim_max & LOCAL_CHASE) ? NONE : csum;
  c->closed_b = cur;
  if (nxt == NONE && fm == NONE) {
    c->mode = MODE_DONE;
    return true;
  }
  if (fm <= nxt) {  // a dropped push precedes the ring's next bucket
    c->rescan_base = fm;
    c->mode = MODE_RESCAN_CLEAR;
    return true;
  }
  sc[s].word = 0;  // recycle the finished bucket's queue (entries already SENTINEL)
  sc[s].head = 0;
  sc[s].p2 = 0;
  const u32 lim = (u32)min((u64)nxt + p.K - 1, (u64)NONE - 1);  // see decide(): slots hold [nxt, nxt + K)
  c->lim = lim;
  c->cur = nxt;
  c->cur_end = (u32)min((u64)nxt + a_m, (u64)lim + 1);
  c->epochs = epochs + 1;
  c->round_end = min(nxt_tail, p.cap);
  c->mode = MODE_PHASE1;
  return true;
}

// Last CTA to arrive runs the serial scheduler step (fused phase 3).
__device__ void decide(const Params& p, u32 which) {
  volatile Ctl* c = p.ctl;
  volatile SlotCtl* sc = p.sc;
  const u32 K = p.K;
  c->closed_b = NONE;
  c->closed_c = 0;
  if (which == SYNC_PL) {  // pull done but for the long scans it handed off
    if (c->long_n != 0) {
      c->long_head = 0;
      c->mode = MODE_PULL_LONG;
      return;
    }
    which = SYNC_P2;
  }
  if (which == SYNC_P2C) {  // entries compacted: relax their heavy arcs, if any
    if ((u32)c->hub_word != 0) {
      c->mode = MODE_P2_RELAX;
      return;
    }
    which = SYNC_P2;
  }
  if (which == SYNC_P1 && c->bf) {  // Bellman-Ford end quiescent: distances final
    if (c->far_min != NONE) {  // a push was dropped (queue full): rebuild from dist[], go on
      c->rescan_base = c->cur;
    } else {
      c->bf = 2;  // clear the queues (rescan_clear), then done
    }
    c->mode = MODE_RESCAN_CLEAR;
    return;
  }
  if (which == SYNC_P1) {
    const u32 cur = c->cur, s = cur & p.kmask;
    if (c->far_min < c->cur_end) {  // phase-1 work was dropped (queue full)
      enter_sweep(c);
      return;
    }
    const u32 tail = min((u32)(sc[s].word >> 32), p.cap);
    if ((p.flags & 2u) && tail > c->round_end) {  // level-synchronous: the next frontier level
      sc[s].head = c->round_end;
      c->round_end = tail;
      c->rounds = c->rounds + 1;
      c->mode = MODE_PHASE1;
      return;
    }
    const u32 b = sc[s].p2;
    c->p2_begin = b;
    c->p2_end = tail;
    if ((p.flags & 128u) && tail - b >= p.V / SSSP_PULL_DIV) {  // large bucket: pull phase 2
      c->pull_n[c->pull_sel == 0 ? 1u : 0u] = 0;  // output candidate list
      c->long_n = 0;
      c->mode = MODE_PULL;
      return;
    }
    if ((p.flags & 4u) && tail - b >= ((p.flags >> 8) & 0x7FFFFFu)) {  // edge-balanced phase 2
      c->hub_word = 0;
      c->p2_head = 0;
      c->mode = MODE_P2_COMPACT;
      return;
    }
    c->p2_head = b;
    c->hub_word = (u64)(tail - b);  // pending = static entries; chunks add to it
    c->hub_head = 0;
    c->mode = MODE_PHASE2;
  } else if (which == SYNC_P2 && decide_close_fast(p)) {
    // fixed Delta: done with two round trips of loads (decide_close_fast)
  } else if (which == SYNC_P2) {
    const u32 cur = c->cur, s = cur & p.kmask;
    sc[s].p2 = c->p2_end;
    if (c->mode == MODE_PULL || c->mode == MODE_PULL_LONG) c->pull_sel = c->pull_sel == 0 ? 1u : 0u;  // its output
    const u32 fm = c->far_min;
    if ((u32)sc[s].word != 0) {  // a heavy relaxation landed in bucket cur (f32 rounding, or
                                 // adaptive Delta with a light level below the width)
      if (fm < c->cur_end) {
        enter_sweep(c);
      } else {
        c->round_end = min((u32)(sc[s].word >> 32), p.cap);
        c->mode = MODE_PHASE1;
        c->epochs = c->epochs + 1;
      }
      return;
    }
    // bucket cur is closed: C_i = vertices settled in it (counted by phase 2 / the pull; unknown
    // with the CTA-local chase, whose entries never reach the bucket's queue)
    const u32 c_i = c->csum;
    c->csum = 0;
    c->closed_c = (p.claim_max & LOCAL_CHASE) ? NONE : c_i;
    c->closed_b = cur;
    u32 nxt = NONE;
    {  // lowest non-empty ring slot after the bucket: 8 slot words in flight per step
      const u32 x_end = c->lim;
      for (u32 x0 = c->cur_end; x0 <= x_end && x0 != NONE && nxt == NONE; x0 += 8) {
        u32 t[8];
#pragma unroll
        for (u32 k = 0; k < 8; ++k)
          t[k] = (x0 + k <= x_end && x0 + k >= x0) ? (u32)(sc[(x0 + k) & p.kmask].word >> 32) : 0u;
#pragma unroll
        for (u32 k = 0; k < 8; ++k)
          if (t[k] && nxt == NONE) nxt = x0 + k;
        if (x0 + 8 < x0) break;
      }
    }
    if (nxt == NONE && fm == NONE) {
      c->mode = MODE_DONE;
      return;
    }
    if (fm <= nxt) {  // a dropped push precedes the ring's next bucket
      c->rescan_base = fm;
      c->mode = MODE_RESCAN_CLEAR;
      return;
    }
    const u32 t_items = min((u32)(sc[s].word >> 32), p.cap);  // T_i: items of bucket cur
    sc[s].word = 0;  // recycle the finished bucket's queue (entries already SENTINEL)
    sc[s].head = 0;
    sc[s].p2 = 0;
    // Ring horizon: slots hold buckets [nxt, nxt + K). The slots of bucket cur (reset just now)
    // and of the empty buckets (cur, nxt) are free, so a jump over empty buckets moves the
    // horizon with it (cur + K - 1 here forced needless rescans after such jumps).
    const u64 lim = (u64)nxt + K - 1;
    c->lim = (u32)min(lim, (u64)NONE - 1);
    c->cur = nxt;
    c->bf_peak = max(c->bf_peak, t_items);
    if (c->bf_t && !c->a_mode && !(p.flags & 2u) && fm == NONE && c->bf_peak >= 8 * c->bf_t) {
      // Bellman-Ford end (Delta = inf for what is left): when the ring holds at most
      // bf_t entries after the wave's peak (a closed bucket held >= 8 bf_t), the remaining buckets would each pay two grid barriers and a chain of
      // round trips for a few thousand vertices. Instead every entry moves into bucket nxt's
      // queue (MODE_MERGE), and one phase 1 relaxes all arcs (light and heavy) of every
      // improved vertex until quiescence: a label-correcting fixpoint, so the same distances.
      u32 tt[16], sum = 0, others = 0;
#pragma unroll
      for (u32 k = 0; k < 16; ++k)
        tt[k] = (k < K && nxt + k <= c->lim) ? (u32)(sc[(nxt + k) & p.kmask].word >> 32) : 0u;
#pragma unroll
      for (u32 k = 0; k < 16; ++k) {
        sum += tt[k];
        others += k ? tt[k] : 0u;
      }
      bool more = false;  // a ring of more than 16 slots: the rest must be empty too
      for (u32 k = 16; k < K && nxt + k <= c->lim; ++k) more |= (sc[(nxt + k) & p.kmask].word >> 32) != 0;
      if (!more && sum <= c->bf_t) {
        c->bf = 1;
        c->epochs = c->epochs + 1;
        if (others) {
          c->cur_end = c->lim + 1;  // merge slots (nxt, lim] into slot nxt
          c->mode = MODE_MERGE;
        } else {
          c->cur_end = NONE;
          c->lim = NONE - 1;
          c->round_end = min(tt[0], p.cap);
          c->mode = MODE_PHASE1;
        }
        return;
      }
    }
    if (c->a_mode) adapt_next(p, t_items, c_i);
    c->cur_end = (u32)min((u64)nxt + c->a_m, (u64)c->lim + 1);
    c->epochs = c->epochs + 1;
    for (u32 x = nxt + 1; x < c->cur_end; ++x)
      if ((u32)(sc[x & p.kmask].word >> 32) != 0) {  // entries binned before the width grew
        c->mode = MODE_MERGE;
        return;
      }
    c->round_end = min((u32)(sc[nxt & p.kmask].word >> 32), p.cap);
    c->mode = MODE_PHASE1;
  } else if (which == SYNC_RC) {
    for (u32 s = 0; s < K; ++s) {
      sc[s].word = 0;
      sc[s].head = 0;
      sc[s].p2 = 0;
    }
    if (c->bf == 2) {
      c->bf = 0;
      c->mode = MODE_DONE;
      return;
    }
    const u32 r = c->rescan_base;
    c->far_min = NONE;
    c->cur = r;
    c->lim = (u32)min((u64)r + K - 1, (u64)NONE - 1);
    c->cur_end = (u32)min((u64)r + c->a_m, (u64)c->lim + 1);
    if (c->bf) {  // Bellman-Ford end: one bucket [r, inf)
      c->lim = NONE - 1;
      c->cur_end = NONE;
    }
    c->mode = MODE_RESCAN_FILL;
  } else if (which == SYNC_MG) {  // slots (cur, cur_end) folded into slot cur
    for (u32 x = c->cur + 1; x < c->cur_end; ++x) {
      sc[x & p.kmask].word = 0;
      sc[x & p.kmask].head = 0;
      sc[x & p.kmask].p2 = 0;
    }
    if (c->bf) {  // merged for the Bellman-Ford end: one bucket [cur, inf)
      c->cur_end = NONE;
      c->lim = NONE - 1;
      if (c->far_min != NONE) {  // slot cur overflowed while merging: rebuild from dist[]
        c->rescan_base = c->cur;
        c->mode = MODE_RESCAN_CLEAR;
        return;
      }
    } else if (c->far_min < c->cur_end) {  // slot cur overflowed while merging
      enter_sweep(c);
      return;
    }
    c->round_end = min((u32)(sc[c->cur & p.kmask].word >> 32), p.cap);
    c->mode = MODE_PHASE1;
  } else if (which == SYNC_RF) {
    c->round_end = min((u32)(sc[c->cur & p.kmask].word >> 32), p.cap);
    c->mode = MODE_PHASE1;
    c->epochs = c->epochs + 1;
    c->rescans = c->rescans + 1;
  } else {  // SYNC_SL / SYNC_SH: sweep fall-back of bucket cur
    if (c->changed) {  // something improved inside bucket cur: sweep light arcs again
      c->changed = 0;
      c->sweep_first = 0;
      c->mode = MODE_SWEEP_LIGHT;
    } else if (which == SYNC_SL) {
      c->mode = MODE_SWEEP_HEAVY;
    } else {  // bucket cur is final; rebuild the ring from dist[] for what follows
      c->closed_c = c->csum;  // the heavy sweep counted the bucket's vertices (local chase or not)
      c->csum = 0;
      c->closed_b = c->cur;
      c->rescan_base = c->cur_end;
      c->mode = MODE_RESCAN_CLEAR;
    }
  }
}

// Bucket extent and light/heavy level of the current bucket into shared memory.
__device__ __forceinline__ void load_bucket(const Params& p, Smem& sm, volatile Ctl* vc) {
  sm.cur_end = vc->cur_end;
  sm.pull_sel = vc->pull_sel;
  sm.pull_n_in = sm.pull_sel < 2 ? vc->pull_n[sm.pull_sel] : vc->first_n;
  const u32 l = vc->lvl;
  sm.rowc_off = (p.flags & 64u) ? l * (p.V + 1) : 0u;  // levels built only with PRO
  sm.theta_bits = l == 0 ? p.delta_bits : ((p.flags & 32u) ? p.delta_bits + (l << 23) : p.delta_bits << l);
  sm.bf = vc->bf;
  if (sm.bf) sm.theta_bits = NONE;  // without PRO: every arc counts as light
}

__device__ void grid_barrier(const Params& p, Smem& sm, u32 which) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const long long t_b = clock64();
    Ctl* c = p.ctl;
    atomicMin(&c->t_first, globaltimer());  // trace only (fire and forget)
    u32 target;
    if (grid_arrive(&c->bar_count, &target)) {
      const u64 t = globaltimer();
      decide(p, which);
      volatile Ctl* vc = c;
      const u64 t_first = vc->t_first;
      vc->t_first = ~0ULL;
      const u64 t_rel = globaltimer();
      grid_release(&c->bar_gen, target);
      // The record is written after the release, off the critical path: what it reads was
      // set by decide() and stays put until the next barrier, which this thread must reach.
      const u32 tn = vc->trace_n;
      if (tn < TRACE_CAP) {
        TraceEnt e;
        e.t_ns = t;
        e.which = which;
        e.cur = vc->cur;
        e.tail = (u32)(((volatile SlotCtl*)p.sc)[vc->cur & p.kmask].word >> 32);
        e.mode = vc->mode;
        e.far_min = vc->far_min;
        e.pad = vc->cur_end;
        e.closed_b = vc->closed_b;
        e.closed_c = vc->closed_c;
        e.t_first = t_first;
        e.t_rel = t_rel;
        p.trace[tn] = e;
        vc->trace_n = tn + 1;
      }
    } else {
      grid_wait(&c->bar_gen, target);
    }
    volatile Ctl* vc = c;
    sm.mode = vc->mode;
    sm.cur = vc->cur;
    sm.lim = vc->lim;
    sm.p2_begin = vc->p2_begin;
    sm.p2_end = vc->p2_end;
    sm.sweep_first = vc->sweep_first;
    sm.round_end = vc->round_end;
    load_bucket(p, sm, vc);
    sm.st[ST_P_BAR] += (unsigned long long)(clock64() - t_b);
  }
  __syncthreads();
}

// ------------------------------------------------------------ phases ------
template <bool F32, bool PRO, bool ABL>
__device__ void phase1(const Params& p, Smem& sm) {
  const u32 slot = sm.cur & p.kmask, lim = sm.lim;
  SlotCtl* sc = p.sc + slot;
  u64* q = p.items + (u64)slot * p.cap;
  const u32 G = gridDim.x;
  const u32 claim_max = p.claim_max & (LOCAL_CHASE - 1);  // claim_max <= BATCH
  u32 my_next = 0, my_end = 0;  // thread 0: claimed ticket range
  u32 owed = 0;  // thread 0: completions of claimed entries held back while the CTA chases locally
  if (threadIdx.x == 0) {
    sm.loc_on = (!ABL && (p.claim_max & LOCAL_CHASE)) ? 1u : 0u;
    // >= 1: a zero limit would leave loc_n growing while nothing drains it (pend never 0)
    sm.loc_lim = max(1u, min((p.claim_max >> LOCAL_LIM_SHIFT) & LOCAL_LIM_MASK, LOC_CAP));
  }
  for (;;) {
    if (threadIdx.x == 0) {
      const long long t_c = clock64();
      u32 n = 0, h = 0, ns = 32, waited = 0, loc = 0;
      if (sm.loc_n) {  // the CTA's own pushes first: pend stays > 0 (owed) until they are done
        n = min(sm.loc_n, sm.loc_lim);
        loc = 1;
      } else if (owed) {
        atomicAdd(&sc->word, (u64)0 - (u64)owed);  // completion of the chased-from entries
        owed = 0;
      }
      if (loc) {
      } else if (ABL && (p.flags & 2u)) {  // level-synchronous: only this level's entries, all already written
        const u32 re = sm.round_end;
        const u32 c = min(max(re / (2 * G), 8u), min(claim_max, BATCH));
        h = ld_relaxed_u32(&sc->head) < re ? atomicAdd(&sc->head, c) : re;
        n = h < re ? min(c, re - h) : 0u;
      }
      for (; !loc && !(ABL && (p.flags & 2u));) {
        // word (tail, pend) and the ticket head in one 16-byte load (same control line)
        uint4 cl;
        asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(cl.x), "=r"(cl.y), "=r"(cl.z), "=r"(cl.w)
                     : "l"(sc)
                     : "memory");
        const u64 wv = ((u64)cl.y << 32) | cl.x;
        const u32 tail = min(cl.y, p.cap);
        // Take new tickets only while some entry is unclaimed (head < tail): in a near-empty
        // bucket the whole grid no longer queues 592 atomics on the one head word before the
        // few CTAs that get entries can start (tickets past the tail still fill as pushes land).
        if (my_next >= my_end && my_end < p.cap && cl.z < tail) {
          // claim size grows with the queue: small early (spread work), up to claim_max
          u32 c = min(max(tail / (2 * G), 8u), claim_max);
          my_next = atomicAdd(&sc->head, c);
          my_end = my_next + c;
        }
        const u32 avail_end = min(my_end, tail);
        const u32 avail = my_next < avail_end ? avail_end - my_next : 0u;
        const u32 full = min(my_end - my_next, BATCH);
        // take a full batch at once; a partial one only after a short wait
        if (avail && (avail >= full || avail >= SSSP_CLAIM_MINPART || waited > SSSP_CLAIM_WAIT_NS)) {
          n = min(avail, BATCH);
          h = my_next;
          my_next += n;
          break;
        }
        if ((u32)wv == 0) {  // quiescent: nothing pending anywhere
          n = 0;
          break;
        }
        __nanosleep(ns);
        waited += ns;
        if (ns < 256) ns <<= 1;
      }
      sm.claim_n = n;
      sm.claim_h = h;
      sm.claim_src = loc;
      sm.st[ST_P_CLAIM] += (unsigned long long)(clock64() - t_c);
      if (SSSP_BATCH_SAMPLES && blockIdx.x % SAMPLE_EVERY == 0) {  // claim timeline (which = 100)
        const u32 k = atomicAdd(&p.ctl->sample_n, 1u);
        if (k < SAMPLE_CAP) {
          const u64 wv = ld_relaxed_u64(&sc->word);
          TraceEnt e;
          e.t_ns = globaltimer();
          e.which = 100;
          e.cur = sm.cur;
          e.tail = (u32)(wv >> 32);
          e.mode = n;
          e.far_min = (u32)wv;
          e.pad = h;
          e.closed_b = blockIdx.x;
          e.closed_c = loc;
          e.t_first = e.t_rel = 0;
          p.trace[TRACE_CAP + k] = e;
        }
      }
    }
    __syncthreads();
    const u32 n = sm.claim_n;
    if (n == 0) break;
    const u32 h = sm.claim_h;
    const bool loc = sm.claim_src != 0;
    u64 it[IPT];
    bool has[IPT];
#pragma unroll
    for (int i = 0; i < IPT; ++i) {
      const u32 my = batch_item_index(i);
      has[i] = my < n;
      it[i] = has[i] ? (loc ? sm.loc[my] : ld_relaxed_u64(q + h + my)) : SENTINEL;
    }
    if (loc) {  // list taken: empty it before this batch pushes again
      __syncthreads();
      if (threadIdx.x == 0) sm.loc_n = 0;
      __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < IPT; ++i) {
      u32 ns = 16;
      while (has[i] && it[i] == SENTINEL) {  // reserved, not yet written
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
        it[i] = ld_relaxed_u64(q + h + batch_item_index(i));
      }
    }
    if (!ABL || (p.flags & 1u))
      process_batch<F32, PRO, 1, IPT, true, ABL>(p, sm, it, has, lim, SRC_QUEUE, slot);
    else
      process_batch<F32, PRO, 1, IPT, !ABL, ABL>(p, sm, it, has, lim, SRC_QUEUE, slot);
    if (threadIdx.x == 0 && !loc) {
      if (sm.loc_on)
        owed += n;  // completion deferred until the local list is drained
      else
        atomicAdd(&sc->word, (u64)0 - (u64)n);  // completion
    }
  }
  if (threadIdx.x == 0) sm.loc_on = 0;
}

template <bool F32, bool PRO, bool ABL>
__device__ void phase2(const Params& p, Smem& sm) {
  const u32 slot = sm.cur & p.kmask, lim = sm.lim;
  u64* q = p.items + (u64)slot * p.cap;
  const u32 p2e = sm.p2_end;
  const u32 G = gridDim.x;
  const u32 span = sm.p2_end - sm.p2_begin;
  const u32 CL = min(max((span + 2 * G - 1) / (2 * G), 16u), (u32)(DS_THREADS * IPT2));
  Ctl* c = p.ctl;
  u32 hub_next = 0, hub_end = 0;  // thread 0: hub ticket
  for (;;) {
    if (threadIdx.x == 0) {
      const long long t_c = clock64();
      u32 n = 0, h = 0, src = 0, ns = 32;
      for (;;) {
        if (ld_relaxed_u32(&c->p2_head) < p2e) {
          h = atomicAdd(&c->p2_head, CL);
          if (h < p2e) {
            n = min(CL, p2e - h);
            src = SRC_STATIC;
            break;
          }
        }
        const u64 wv = ld_relaxed_u64(&c->hub_word);
        const u32 tail = min((u32)(wv >> 32), p.hub_cap);
        if (hub_next >= hub_end && hub_end < p.hub_cap && hub_end <= tail) {
          hub_next = atomicAdd(&c->hub_head, 1u);  // one 4096-arc chunk per ticket
          hub_end = hub_next + 1;
        }
        if (hub_next < hub_end && hub_next < tail) {
          h = hub_next;
          n = 1;
          hub_next = hub_end;
          src = SRC_HUB;
          break;
        }
        if ((u32)wv == 0) {
          n = 0;
          break;
        }
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
      }
      sm.claim_n = n;
      sm.claim_h = h;
      sm.claim_src = src;
      sm.st[ST_P_CLAIM] += (unsigned long long)(clock64() - t_c);
    }
    __syncthreads();
    const u32 n = sm.claim_n;
    if (n == 0) break;
    const u32 h = sm.claim_h, src = sm.claim_src;
    u64 it[IPT2];
    bool has[IPT2];
    u64* const base_q = src == SRC_STATIC ? q + h : p.hub_items + h;
#pragma unroll
    for (int i = 0; i < IPT2; ++i) {
      const u32 my = batch_item_index(i);
      has[i] = my < n;
      it[i] = has[i] ? ld_relaxed_u64(base_q + my) : SENTINEL;
    }
#pragma unroll
    for (int i = 0; i < IPT2; ++i) {
      if (!has[i]) continue;
      u32 ns = 16;
      while (it[i] == SENTINEL) {  // hub chunks may be reserved but not yet written
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
        it[i] = ld_relaxed_u64(base_q + batch_item_index(i));
      }
      st_relaxed_u64(base_q + batch_item_index(i), SENTINEL);  // recycle the queue entry
    }
    if (!ABL || (p.flags & 1u))
      process_batch<F32, PRO, 2, IPT2, true, ABL>(p, sm, it, has, lim, src, slot);
    else
      process_batch<F32, PRO, 2, IPT2, !ABL, ABL>(p, sm, it, has, lim, src, slot);
    if (threadIdx.x == 0) atomicAdd(&c->hub_word, (u64)0 - (u64)n);
  }
}

// ------------------------------------------- edge-balanced phase 2 -------
// The paper's phases 2&3 kernel gives every thread the same number of heavy
// edges (static load balancing). Here: (1) p2_compact turns the
// bucket's settled range [p2_begin, p2_end) into a dense list of the entries
// that are final (d == dist[v], Alg. 2 l.14) and have heavy arcs, each with
// the rank of its first heavy arc (one 64-bit atomicAdd per CTA batch hands
// out (entry, arc-rank) bases together, so ranks grow with the list index);
// (2) after a grid barrier, p2_relax splits the rank range [0, T) into
// equal-arc pieces claimed by warps. A warp maps arc rank x to its owner entry
// (the last entry with rank <= x) with a 32-entry window held in registers
// (one coalesced load per 31 entries, shuffle binary search per arc), so hubs
// and small vertices are spread over warps by arcs, not by vertices.
// Measured on B200 (profiles/r01c): no faster than the vertex-bin phase 2 on
// C4 and 15 % slower on C3, so it is off by default (SSSP_PARAM_P2_EDGE_BALANCED).
template <bool F32, bool PRO>
__device__ void p2_compact(const Params& p, Smem& sm) {
  const u32 slot = sm.cur & p.kmask;
  u64* q = p.items + (u64)slot * p.cap;
  const u32 b0 = sm.p2_begin, b1 = sm.p2_end;
  uint2* sd = reinterpret_cast<uint2*>(p.p2o + ((p.cap + 1) & ~1u));
  const u32 tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  constexpr u32 CB = DS_THREADS * IPT2;
  u32 c_live = 0, c_arcs = 0;
  for (u32 base = b0 + blockIdx.x * CB; base < b1; base += gridDim.x * CB) {
    u64 e[IPT2];
    bool has[IPT2];
#pragma unroll
    for (int i = 0; i < IPT2; ++i) {
      const u32 pos = base + i * DS_THREADS + tid;
      has[i] = pos < b1;
      e[i] = has[i] ? ld_relaxed_u64(q + pos) : SENTINEL;
    }
    u32 cd[IPT2];
#pragma unroll
    for (int i = 0; i < IPT2; ++i) {
      if (has[i]) st_relaxed_u64(q + base + i * DS_THREADS + tid, SENTINEL);  // recycle
      has[i] = has[i] && !((u32)e[i] & CHUNK_FLAG);  // phase-1 hub chunks: no vertex
      cd[i] = has[i] ? ld_cg(p.dist + (u32)e[i]) : 0u;
    }
    u32 hl[IPT2], st[IPT2];
    u64 x = 0;
#pragma unroll
    for (int i = 0; i < IPT2; ++i) {
      hl[i] = 0;
      st[i] = 0;
      if (has[i] && (u32)(e[i] >> 32) == cd[i]) {  // final in this bucket
        const u32 v = (u32)e[i];
        const uint2* rowc = p.rowc + sm.rowc_off;
        const uint2 r = rowc[v];
        st[i] = PRO ? r.y : r.x;
        hl[i] = rowc[v + 1].x - st[i];
        ++c_live;
        c_arcs += hl[i];
        if (hl[i]) x += (1ULL << 32) | hl[i];
      }
    }
    u64 tot;
    u64 pre = warp_exclusive_scan(x, &tot);
    if (lane == 31) sm.scan_ws[w] = tot;
    __syncthreads();
    u64 acc = 0, all = 0;
#pragma unroll
    for (int i = 0; i < DS_WARPS; ++i) {
      const u64 sv = sm.scan_ws[i];
      if (i < (int)w) acc += sv;
      all += sv;
    }
    if (tid == 0 && all) {
      const u64 g = atomicAdd(&p.ctl->hub_word, all);
      sm.claim_h = (u32)(g >> 32);
      sm.claim_n = (u32)g;
    }
    __syncthreads();
    if (all) {
      pre += acc;
      u32 idx = sm.claim_h + (u32)(pre >> 32), rank = sm.claim_n + (u32)pre;
#pragma unroll
      for (int i = 0; i < IPT2; ++i) {
        if (hl[i]) {
          p.p2o[idx] = rank;
          sd[idx] = make_uint2(st[i] - rank, (u32)(e[i] >> 32));  // arc index = rank + .x
          ++idx;
          rank += hl[i];
        }
      }
    }
    __syncthreads();  // scan_ws / claim_* reused by the next batch
  }
  st_add(sm, ST_HEAVYV, c_live);
  st_add(sm, ST_HEAVY, c_arcs);
  {
    const u32 cs = __reduce_add_sync(SSSP_FULL_MASK, c_live);
    if (lane == 0 && cs) atomicAdd(&p.ctl->csum, cs);
  }
}

template <bool F32, bool PRO>
__device__ void p2_relax(const Params& p, Smem& sm) {
  const u64 hw = ld_relaxed_u64(&p.ctl->hub_word);
  const u32 n = (u32)(hw >> 32), T = (u32)hw;
  const u32 lane = lane_id(), lim = sm.lim;
  const u32* O = p.p2o;
  const uint2* sd = reinterpret_cast<const uint2*>(p.p2o + ((p.cap + 1) & ~1u));
  const u32 W = gridDim.x * DS_WARPS;
  u32* head = &p.ctl->p2_head;
  // window over entries [wb, wb+32): rank, {arc index - rank, d}; NONE past n
  u32 wb = 0, wv = NONE, wx = 0, wy = 0;
  auto load_window = [&]() {
    const u32 j = wb + lane;
    wv = NONE;
    if (j < n) {
      wv = ld_cg(O + j);
      const uint2 t = __ldcg(sd + j);
      wx = t.x;
      wy = t.y;
    }
  };
  auto setup = [&](u32 tb, u32 ce, u32(&idx)[UNROLL], bool(&valid)[UNROLL], u32(&dd)[UNROLL]) {
    bool pend[UNROLL];
#pragma unroll
    for (int k = 0; k < UNROLL; ++k) {
      const u32 xk = tb + k * 32 + lane;
      valid[k] = tb < ce && xk < ce;
      pend[k] = valid[k];
      idx[k] = 0;
      dd[k] = 0;
    }
    for (;;) {
      const u32 wlast = __shfl_sync(SSSP_FULL_MASK, wv, 31);
      bool left = false;
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        const u32 xk = tb + k * 32 + lane;
        u32 j = 0;  // last window entry with rank <= xk (entry 0 always qualifies)
#pragma unroll
        for (u32 s = 16; s; s >>= 1) {
          const u32 t = __shfl_sync(SSSP_FULL_MASK, wv, j + s);
          if (t <= xk) j += s;
        }
        const u32 ax = __shfl_sync(SSSP_FULL_MASK, wx, j);
        const u32 ay = __shfl_sync(SSSP_FULL_MASK, wy, j);
        if (pend[k] && xk < wlast) {
          idx[k] = xk + ax;
          dd[k] = ay;
          pend[k] = false;
        }
        left |= pend[k];
      }
      if (!__any_sync(SSSP_FULL_MASK, left)) break;
      wb += 31;  // every pending rank is >= the window's last rank
      load_window();
    }
  };
  for (;;) {
    u32 c0 = 0, cl = 0;
    if (lane == 0) {
      const u32 seen = ld_relaxed_u32(head);
      const u32 rem = seen < T ? T - seen : 0u;
      cl = min(max((rem / (2 * W)) & ~(TASK - 1), 8 * TASK), 64 * TASK);  // guided self-scheduling
      c0 = atomicAdd(head, cl);
    }
    c0 = __shfl_sync(SSSP_FULL_MASK, c0, 0);
    cl = __shfl_sync(SSSP_FULL_MASK, cl, 0);
    if (c0 >= T) break;
    const u32 ce = min(c0 + cl, T);
    // owner of c0: 32-ary search over the ranks
    u32 lo = 0, hi = n;
    while (hi - lo > 32) {
      const u32 step = (hi - lo + 31) / 32;
      const u32 j = lo + lane * step;
      const u32 v = j < hi ? ld_cg(O + j) : NONE;
      const u32 m = __ballot_sync(SSSP_FULL_MASK, v <= c0);
      lo += (31 - __clz(m)) * step;
      hi = min(lo + step, hi);
    }
    wb = lo;
    load_window();
    u32 idx[UNROLL], dd[UNROLL];
    bool valid[UNROLL];
    uint2 a[UNROLL];
    u32 tb = c0;
    setup(tb, ce, idx, valid, dd);
    arcs_issue(p, idx, valid, a);
    while (tb < ce) {
      const u32 tb2 = tb + TASK;
      u32 idx2[UNROLL], dd2[UNROLL];
      bool valid2[UNROLL];
      uint2 a2[UNROLL];
      setup(tb2, ce, idx2, valid2, dd2);
      arcs_issue(p, idx2, valid2, a2);  // next task's arcs in flight ...
      relax_finish<F32, PRO, 2>(p, sm, lim, NONE, a, valid, dd);  // ... while this one completes
      tb = tb2;
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        a[k] = a2[k];
        valid[k] = valid2[k];
        dd[k] = dd2[k];
      }
    }
  }
  if (sm.pb_n[threadIdx.x >> 5]) pb_flush<F32>(p, sm, lim, NONE);
}

// ------------------------------------------------------ pull phase 2 -----
// Phases 2&3 of a bucket with many settled vertices, turned around (the
// direction-optimising idea, valid because the graph is symmetric: v's arc
// (v, u, w) exists iff u's arc (u, v, w) does). Alg. 2 l.13-17 relaxes the
// heavy arcs (w >= Delta) of every vertex u settled in bucket cur; here every
// vertex v not settled yet (dist[v] >= hi) scans its own heavy arcs, which PRO
// sorted by ascending weight, and takes min(dist[u] + w) over
// neighbours u whose distance lies in bucket cur. A candidate through bucket
// cur is >= lo + w, so the scan stops at the first arc with lo + w >= best:
// most vertices find a hub of the bucket among their lightest heavy arcs and
// stop early. Every heavy arc out of bucket cur that could improve v is still
// examined, so the result is the one push-style phase 2 gives.
// Bucket cur's bounds for the pull: u32 [lo, hi) (INF = 0xFFFFFFFF is never inside, even when
// hi > 2^32 - 1); f32 by bucket_of, with lo_f <= every distance of bucket cur (cur * Delta
// rounded down, less 2^-20 relative), so fl(lo_f + w) bounds fl(du + w) from below for every u
// of the bucket (fl is monotone). f32 graphs carry Delta's bits in delta_u when pulling.
struct PullBounds {
  u64 lo, hi;
  float lo_f;
  u32 cur;
};
template <bool F32>
__device__ __forceinline__ PullBounds pull_bounds(const Params& p, u32 cur) {
  PullBounds b;
  b.cur = cur;
  b.lo = F32 ? 0 : (u64)cur * p.delta_u;
  b.hi = F32 ? 0 : b.lo + p.delta_u;
  b.lo_f = (F32 && cur) ? __fmul_rd(__fmul_rd((float)cur, __uint_as_float(p.delta_u)), 0.99999905f) : 0.f;
  return b;
}
template <bool F32>
__device__ __forceinline__ bool in_bucket(const Params& p, const PullBounds& b, u32 d) {
  if (F32) return bucket_of<true>(p, d) == b.cur;
  return d != NONE && (u64)d >= b.lo && (u64)d < b.hi;
}
template <bool F32>
__device__ __forceinline__ bool unsettled(const Params& p, const PullBounds& b, u32 d) {
  if (F32) return bucket_of<true>(p, d) > b.cur;
  return d == NONE || (u64)d >= b.hi;
}
// A heavy arc of weight w can still beat best (ascending w: once false, false for the rest).
// An unreached v (best = INF) scans on even when lo + w >= INF, so an overflow is reported.
template <bool F32>
__device__ __forceinline__ bool may_win(const PullBounds& b, u32 w, u32 best) {
  if (F32) return __float_as_uint(__fadd_rn(b.lo_f, __uint_as_float(w))) < best;
  return b.lo + w < (u64)best || best == NONE;
}
// Candidate through u (du in bucket cur) over an arc of weight w: best = min(best, du + w).
template <bool F32>
__device__ __forceinline__ void pull_take(u32 du, u32 w, u32& best, bool& of) {
  if (F32) {
    best = min(best, __float_as_uint(__fadd_rn(__uint_as_float(du), __uint_as_float(w))));
  } else {
    const u64 cand = (u64)du + w;
    if (cand >= (u64)NONE)
      of = true;  // same rule as the push relaxation (relax_finish)
    else if (cand < (u64)best)
      best = (u32)cand;
  }
}

constexpr u32 PULL_LANE_STEPS = 4;  // a lane scans <= 4 * 2 heavy arcs of a vertex, then hands it off

template <bool F32, bool PRO>
__device__ void pull_phase(const Params& p, Smem& sm) {
  const u32 cur = sm.cur, lim = sm.lim, lane = lane_id();
  {  // recycle the bucket's queue entries (push-style phase 2 consumes them)
    u64* q = p.items + (u64)(cur & p.kmask) * p.cap;
    for (i64 i = sm.p2_begin + (i64)blockIdx.x * blockDim.x + threadIdx.x; i < sm.p2_end;
         i += (i64)gridDim.x * blockDim.x)
      st_relaxed_u64(q + i, SENTINEL);
  }
  const PullBounds B = pull_bounds<F32>(p, cur);
  // Candidates: every vertex (first pull), else the list the previous pull kept -- the vertices
  // that were unsettled then and have arcs (a vertex settled since is skipped, one settled in
  // bucket cur is counted in C_i). This pull keeps the ones still unsettled after bucket cur.
  const u32 sel = sm.pull_sel, osel = sel == 0 ? 1u : 0u;
  const u32* in = sel == 2 ? nullptr : p.xd + (u64)(1 + sel) * p.V;
  const u32 n_in = sm.pull_n_in;  // first pull: [0, first_n)
  u32* out = p.xd + (u64)(1 + osel) * p.V;
  u32* out_n = &p.ctl->pull_n[osel];
  uint4* longq = reinterpret_cast<uint4*>(p.xd + ((3 * (u64)p.V + 3) & ~3ULL));  // 16-B aligned
  const u32 long_cap = p.V / 2;
  constexpr int NV = 4;       // candidates per lane in flight
  static_assert(NV % UNROLL == 0, "pushes are staged UNROLL at a time");
  constexpr int PU = 2;       // heavy arcs per candidate per step
  u32 c_pull = 0, c_arcs = 0, c_in = 0;
  bool of = false;
  const u64 pol_stream = policy_evict_first(), pol_keep = policy_evict_last();
  const u64 wstride = (u64)gridDim.x * blockDim.x * NV;
  for (u64 wb = ((u64)blockIdx.x * blockDim.x + (threadIdx.x & ~31u)) * NV; wb < n_in; wb += wstride) {
    u32 v[NV], dv[NV], j[NV], e[NV], best[NV];
    bool act[NV], keep[NV];
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const u64 i = wb + (u64)k * 32 + lane;
      v[k] = i < n_in ? (in ? ld_cg(in + i) : (u32)i) : NONE;
    }
#pragma unroll
    for (int k = 0; k < NV; ++k) dv[k] = v[k] != NONE ? ld_cg(p.dist + v[k]) : 0u;
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const bool has = v[k] != NONE;
      c_in += has && in_bucket<F32>(p, B, dv[k]);
      act[k] = has && unsettled<F32>(p, B, dv[k]);
      j[k] = e[k] = 0;
    }
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      if (act[k]) {
        const uint2 r = p.rowc[v[k]];
        e[k] = p.rowc[v[k] + 1].x;
        keep[k] = e[k] > r.x;  // isolated vertices are never reached: drop them
        j[k] = PRO ? r.y : r.x;
      } else {
        keep[k] = false;
      }
      act[k] = act[k] && j[k] < e[k];
      best[k] = dv[k];
    }
    {  // the next pull's candidates: one reservation per warp
      u32 m[NV], tot = 0;
#pragma unroll
      for (int k = 0; k < NV; ++k) {
        m[k] = __ballot_sync(SSSP_FULL_MASK, keep[k]);
        tot += __popc(m[k]);
      }
      u32 base = 0;
      if (lane == 0 && tot) base = atomicAdd(out_n, tot);
      base = __shfl_sync(SSSP_FULL_MASK, base, 0);
      const u32 lt = lanemask_lt();
#pragma unroll
      for (int k = 0; k < NV; ++k) {
        if (keep[k]) out[base + __popc(m[k] & lt)] = v[k];
        base += __popc(m[k]);
      }
    }
    bool any = false;
#pragma unroll
    for (int k = 0; k < NV; ++k) any |= act[k];
    u32 steps = 0;
    while (__any_sync(SSSP_FULL_MASK, any)) {
      if (steps == PULL_LANE_STEPS) {  // long scans: hand them to whole warps (MODE_PULL_LONG)
        u32 m[NV], tot = 0;
#pragma unroll
        for (int k = 0; k < NV; ++k) {
          m[k] = __ballot_sync(SSSP_FULL_MASK, act[k]);
          tot += __popc(m[k]);
        }
        u32 base = 0;
        if (lane == 0) base = atomicAdd(&p.ctl->long_n, tot);
        base = __shfl_sync(SSSP_FULL_MASK, base, 0);
        const u32 lt = lanemask_lt();
        any = false;
#pragma unroll
        for (int k = 0; k < NV; ++k) {
          const u32 idx = base + __popc(m[k] & lt);
          if (act[k] && idx < long_cap) {
            longq[idx] = make_uint4(v[k], j[k], best[k], dv[k]);
            act[k] = false;
            v[k] = NONE;  // its push is the long step's
          }
          base += __popc(m[k]);
          any |= act[k];
        }
        if (lane == 0 && base > long_cap) atomicMin(&p.ctl->long_n, long_cap);  // the rest stay here
        if (!__any_sync(SSSP_FULL_MASK, any)) break;
      }
      ++steps;
      uint2 a[NV][PU];
#pragma unroll
      for (int k = 0; k < NV; ++k)
#pragma unroll
        for (int u = 0; u < PU; ++u) a[k][u] = ld_arc(p.arcs + j[k] + u, act[k] && j[k] + u < e[k], pol_stream);
      u32 du[NV][PU];
      bool ok[NV][PU];
#pragma unroll
      for (int k = 0; k < NV; ++k)
#pragma unroll
        for (int u = 0; u < PU; ++u) {
          bool o = act[k] && j[k] + u < e[k] && may_win<F32>(B, a[k][u].y, best[k]);
          if (!PRO) o = o && a[k][u].y >= p.delta_bits;  // heavy arcs only
          ok[k][u] = o;
          du[k][u] = ld_probe(p.dist + a[k][u].x, o, pol_keep);
        }
      any = false;
#pragma unroll
      for (int k = 0; k < NV; ++k) {
#pragma unroll
        for (int u = 0; u < PU; ++u)
          if (ok[k][u] && in_bucket<F32>(p, B, du[k][u])) pull_take<F32>(du[k][u], a[k][u].y, best[k], of);
        if (act[k]) c_arcs += min((u32)PU, e[k] - j[k]);
        j[k] += PU;
        act[k] = act[k] && j[k] < e[k] && (PRO ? ok[k][PU - 1] : true);
        any |= act[k];
      }
    }
#pragma unroll
    for (int k0 = 0; k0 < NV; k0 += UNROLL) {
      bool want[UNROLL];
      u32 vv[UNROLL], nd[UNROLL];
#pragma unroll
      for (int k = 0; k < UNROLL; ++k) {
        want[k] = v[k0 + k] != NONE && best[k0 + k] < dv[k0 + k];
        vv[k] = v[k0 + k];
        nd[k] = best[k0 + k];
        if (want[k]) {
          atomicMin(p.dist + vv[k], nd[k]);  // v is this thread's alone during the pull
          ++c_pull;
        }
      }
      stage_pushes<F32>(p, sm, lim, NONE, want, vv, nd);
    }
  }
  if (sm.pb_n[threadIdx.x >> 5]) pb_flush<F32>(p, sm, lim, NONE);
  if (!F32 && of) atomicOr(&p.ctl->err, ERR_OVERFLOW);
  st_add(sm, ST_HEAVY, c_arcs);
  st_add(sm, ST_HEAVYV, c_pull);
  {
    const u32 cs = __reduce_add_sync(SSSP_FULL_MASK, c_in);
    if (lane == 0 && cs) atomicAdd(&p.ctl->csum, cs);
  }
}

// Second step of the pull: the vertices whose weight-sorted heavy scan outlasted the lane
// budget, one warp per vertex, 64 arcs per step (two per lane), warp-min of the candidates;
// the scan ends at the first arc that can no longer win (or the segment end).
template <bool F32, bool PRO>
__device__ void pull_long(const Params& p, Smem& sm) {
  const u32 cur = sm.cur, lim = sm.lim, lane = lane_id();
  const PullBounds B = pull_bounds<F32>(p, cur);
  const uint4* longq = reinterpret_cast<const uint4*>(p.xd + ((3 * (u64)p.V + 3) & ~3ULL));
  const u32 n = ld_relaxed_u32(&p.ctl->long_n);
  const u64 pol_stream = policy_evict_first(), pol_keep = policy_evict_last();
  u32 c_pull = 0, c_arcs = 0;
  bool of = false;
  for (;;) {
    u32 i = 0;
    if (lane == 0) i = atomicAdd(&p.ctl->long_head, 1u);
    i = __shfl_sync(SSSP_FULL_MASK, i, 0);
    bool want[UNROLL] = {};
    u32 vv[UNROLL] = {}, nd[UNROLL] = {};
    if (i < n) {
      const uint4 it = __ldcg(longq + i);
      const u32 v = it.x, e = p.rowc[v + 1].x, dv = it.w;
      u32 j = it.y, best = it.z;
      for (;;) {
        uint2 a[2];
        bool ok[2];
        u32 du[2];
#pragma unroll
        for (int u = 0; u < 2; ++u) a[u] = ld_arc(p.arcs + j + u * 32 + lane, j + u * 32 + lane < e, pol_stream);
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          ok[u] = j + u * 32 + lane < e && may_win<F32>(B, a[u].y, best);
          if (!PRO) ok[u] = ok[u] && a[u].y >= p.delta_bits;
          du[u] = ld_probe(p.dist + a[u].x, ok[u], pol_keep);
        }
        u32 b = best;
#pragma unroll
        for (int u = 0; u < 2; ++u)
          if (ok[u] && in_bucket<F32>(p, B, du[u])) pull_take<F32>(du[u], a[u].y, b, of);
        best = __reduce_min_sync(SSSP_FULL_MASK, b);
        if (lane == 0) c_arcs += min(64u, e - j);
        j += 64;
        // an arc that failed the bound (or the segment end) ends the scan: weights ascend
        if (!__all_sync(SSSP_FULL_MASK, ok[0] && ok[1]) || j >= e) break;
      }
      if (lane == 0 && best < dv) {
        atomicMin(p.dist + v, best);
        want[0] = true;
        vv[0] = v;
        nd[0] = best;
        ++c_pull;
      }
    }
    stage_pushes<F32>(p, sm, lim, NONE, want, vv, nd);
    if (i >= n) break;
  }
  if (sm.pb_n[threadIdx.x >> 5]) pb_flush<F32>(p, sm, lim, NONE);
  if (!F32 && of) atomicOr(&p.ctl->err, ERR_OVERFLOW);
  st_add(sm, ST_HEAVY, c_arcs);
  st_add(sm, ST_HEAVYV, c_pull);
}

// Rescan stage 1: clear every queue entry still holding a value.
__device__ void rescan_clear(const Params& p) {
  const i64 t = (i64)blockIdx.x * blockDim.x + threadIdx.x;
  const i64 nt = (i64)gridDim.x * blockDim.x;
  for (u32 s0 = 0; s0 < p.K; s0 += 8) {
    u32 tl[8];  // tails in flight together
#pragma unroll
    for (u32 k = 0; k < 8; ++k) tl[k] = s0 + k < p.K ? min((u32)(ld_relaxed_u64(&p.sc[s0 + k].word) >> 32), p.cap) : 0u;
    for (u32 k = 0; k < 8 && s0 + k < p.K; ++k) {
      u64* q = p.items + (u64)(s0 + k) * p.cap;
      for (i64 i = t; i < tl[k]; i += nt) st_relaxed_u64(q + i, SENTINEL);
    }
  }
}

// Rescan stage 2: every unsettled vertex (bucket(dist) >= base) is pushed anew.
template <bool F32>
__device__ void rescan_fill(const Params& p, Smem& sm) {
  const u32 base = sm.cur, lim = sm.lim;
  const i64 t0 = ((i64)blockIdx.x * blockDim.x + threadIdx.x) & ~31LL;
  const i64 nt = (i64)gridDim.x * blockDim.x;
  const u32 inf = F32 ? 0x7F800000u : NONE;
  for (i64 b = t0; b < p.V; b += nt) {
    const i64 v = b + lane_id();
    bool want[UNROLL] = {};
    u32 vv[UNROLL] = {}, dd[UNROLL] = {};
    if (v < p.V) {
      const u32 d = ld_cg(p.dist + v);
      want[0] = d != inf && bucket_of<F32>(p, d) >= base;
      vv[0] = (u32)v;
      dd[0] = d;
    }
    stage_pushes<F32>(p, sm, lim, NONE, want, vv, dd);
  }
  if (sm.pb_n[threadIdx.x >> 5]) pb_flush<F32>(p, sm, lim, NONE);
}

// Sweep fall-back for a bucket whose queue lost work (capacity): Bellman-Ford
// style sweeps over all v with bucket(dist[v]) == cur until nothing in the
// bucket improves (light arcs; xd[] skips vertices unchanged since their last
// expansion), then one sweep over heavy arcs. Always makes progress.
template <bool F32, bool PRO, int PH, bool EXT>
__device__ void sweep(const Params& p, Smem& sm) {
  const u32 cur = sm.cur, lim = sm.lim;
  const bool first = sm.sweep_first != 0;
  const u32 inf = F32 ? 0x7F800000u : NONE;
  for (i64 base = (i64)blockIdx.x * BATCH; base < p.V; base += (i64)gridDim.x * BATCH) {
    bool has[IPT];
    u64 it[IPT];
#pragma unroll
    for (int i = 0; i < IPT; ++i) {
      const i64 v = base + batch_item_index(i);
      has[i] = false;
      it[i] = SENTINEL;
      if (v < p.V) {
        const u32 d = ld_cg(p.dist + v);
        const u32 bx = d != inf ? bucket_of<F32>(p, d) : NONE;
        if (bx >= cur && bx < sm.cur_end) {
          if (PH == 1) {
            if (first || d < ld_cg(p.xd + v)) {
              st_relaxed_u32(p.xd + v, d);
              has[i] = true;
            }
          } else {
            has[i] = true;
          }
          it[i] = ((u64)d << 32) | (u64)v;
        }
      }
    }
    process_batch<F32, PRO, PH, IPT, true, EXT>(p, sm, it, has, lim, SRC_SWEEP, cur & p.kmask);
  }
}

// Adaptive Delta: the bucket grew over slots (cur, cur_end) that already hold
// entries pushed while they were far buckets. Move the live ones into slot cur
// (pb_flush resolves them to the current bucket); stale ones are dropped (a
// better entry of the same vertex was pushed when dist[] improved).
template <bool F32>
__device__ void merge_slots(const Params& p, Smem& sm) {
  const u32 cur = sm.cur, ce = sm.cur_end, lim = sm.lim, lane = lane_id();
  u32 moved = 0;
  const i64 t0 = ((i64)blockIdx.x * blockDim.x + threadIdx.x) & ~31LL;
  const i64 nt = (i64)gridDim.x * blockDim.x;
  for (u32 x0 = cur + 1; x0 < ce; x0 += 8) {
    // eight slots at a time, their entries laid end to end: the tails in one round trip and
    // every entry of the eight slots in one grid-stride pass (the Bellman-Ford end merges a
    // few thousand entries spread over up to K - 1 slots)
    u32 tl[8], tot = 0;
#pragma unroll
    for (u32 k = 0; k < 8; ++k)
      tl[k] = x0 + k < ce ? min((u32)(ld_relaxed_u64(&p.sc[(x0 + k) & p.kmask].word) >> 32), p.cap) : 0u;
#pragma unroll
    for (u32 k = 0; k < 8; ++k) tot += tl[k];
    for (i64 b = t0; b < tot; b += nt) {
      const i64 i = b + lane;
      bool want[UNROLL] = {};
      u32 vv[UNROLL] = {}, dd[UNROLL] = {};
      if (i < tot) {
        u32 k = 0, o = (u32)i;
#pragma unroll
        for (u32 j = 0; j < 7; ++j)
          if (k == j && o >= tl[j]) {
            o -= tl[j];
            k = j + 1;
          }
        u64* q = p.items + (u64)((x0 + k) & p.kmask) * p.cap + o;
        const u64 e = ld_relaxed_u64(q);
        st_relaxed_u64(q, SENTINEL);
        if (e != SENTINEL && !((u32)e & CHUNK_FLAG)) {
          vv[0] = (u32)e;
          dd[0] = (u32)(e >> 32);
          want[0] = ld_cg(p.dist + vv[0]) == dd[0];
        }
      }
      moved += want[0];
      stage_pushes<F32>(p, sm, lim, NONE, want, vv, dd);
    }
  }
  if (sm.pb_n[threadIdx.x >> 5]) pb_flush<F32>(p, sm, lim, NONE);
  const u32 mv = __reduce_add_sync(SSSP_FULL_MASK, moved);
  if (lane == 0 && mv) sm.wst[threadIdx.x >> 5][ST_UPDATES] -= mv;  // not updates
}

// ABL = extended build: the ablation paths (SSSP_PARAM_ADWL = 0 / SSSP_PARAM_SYNC = 1),
// the edge-balanced phase 2 and the adaptive-Delta slot merge are compiled in; the
// default kernel (ABL = false) carries none of that code (it raised the default
// kernel's register spills from 164 to 288 bytes and cost ~6 % on C4).
template <bool F32, bool PRO, bool ABL>
__global__ void __launch_bounds__(DS_THREADS, SSSP_MINB) k_delta_step(Params p) {
  __shared__ Smem sm;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const u64 t0 = globaltimer();
    TraceEnt e = {t0, 99u, 0u, 0u, 0u, 0u, 0u, NONE, 0u, t0, t0};
    p.trace[0] = e;
    p.ctl->trace_n = 1;
  }
  if (threadIdx.x < ST_N) sm.st[threadIdx.x] = 0;
  for (u32 i = threadIdx.x; i < DS_WARPS * ST_N; i += blockDim.x) (&sm.wst[0][0])[i] = 0;
  if (threadIdx.x < DS_WARPS) sm.pb_n[threadIdx.x] = 0;
  if (threadIdx.x == 0) {
    // dmul = ceil(2^64 / delta_u); delta_u = 1 (2^64 does not fit) is its own case in bucket_of_f
    const u64 dm = p.delta_u > 1 ? (~0ULL / p.delta_u) + 1 : 0ULL;
    sm.fctx = FlushCtx{p.sc, p.items, p.ctl, p.xd, p.dist, dm, p.cap, p.kmask, p.delta_u, p.inv_delta};
    sm.loc_n = 0;
    sm.loc_on = 0;
    volatile Ctl* vc = p.ctl;
    sm.mode = vc->mode;
    sm.cur = vc->cur;
    sm.lim = vc->lim;
    sm.p2_begin = vc->p2_begin;
    sm.p2_end = vc->p2_end;
    sm.sweep_first = vc->sweep_first;
    sm.round_end = vc->round_end;
    load_bucket(p, sm, vc);
  }
  __syncthreads();
  for (;;) {
    const u32 mode = sm.mode;
    if (mode == MODE_DONE) break;
    if (mode == MODE_PHASE1) {
      phase1<F32, PRO, ABL>(p, sm);
      grid_barrier(p, sm, SYNC_P1);
    } else if (mode == MODE_PHASE2) {
      phase2<F32, PRO, ABL>(p, sm);
      grid_barrier(p, sm, SYNC_P2);
    } else if (mode == MODE_PULL) {
      pull_phase<F32, PRO>(p, sm);
      grid_barrier(p, sm, SYNC_PL);
    } else if (mode == MODE_PULL_LONG) {
      pull_long<F32, PRO>(p, sm);
      grid_barrier(p, sm, SYNC_P2);
    } else if (mode == MODE_MERGE) {  // adaptive Delta (extended build) / Bellman-Ford end
      merge_slots<F32>(p, sm);
      grid_barrier(p, sm, SYNC_MG);
    } else if (ABL && mode == MODE_P2_COMPACT) {  // extended build only (edge-balanced phase 2)
      if constexpr (ABL) p2_compact<F32, PRO>(p, sm);
      grid_barrier(p, sm, SYNC_P2C);
    } else if (ABL && mode == MODE_P2_RELAX) {
      if constexpr (ABL) p2_relax<F32, PRO>(p, sm);
      grid_barrier(p, sm, SYNC_P2);
    } else if (mode == MODE_RESCAN_CLEAR) {
      rescan_clear(p);
      grid_barrier(p, sm, SYNC_RC);
    } else if (mode == MODE_RESCAN_FILL) {
      rescan_fill<F32>(p, sm);
      grid_barrier(p, sm, SYNC_RF);
    } else if (mode == MODE_SWEEP_LIGHT) {
      sweep<F32, PRO, 1, ABL>(p, sm);
      grid_barrier(p, sm, SYNC_SL);
    } else {
      sweep<F32, PRO, 2, ABL>(p, sm);
      grid_barrier(p, sm, SYNC_SH);
    }
  }
  __syncthreads();
  if (threadIdx.x < ST_N) {
    unsigned long long x = sm.st[threadIdx.x];
#pragma unroll
    for (int w = 0; w < DS_WARPS; ++w) x += sm.wst[w][threadIdx.x];
    if (x) atomicAdd(p.stats + threadIdx.x, x);
  }
  // Every CTA has passed the last grid barrier, so err is final: fold it into the sticky word
  // that sssp_wait / sssp_run_batch / sssp_distances report (and clear) on the host.
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const u32 e = ld_relaxed_u32(&p.ctl->err);
    if (e) atomicOr(&p.ctl->err_acc, e);
  }
}

// ------------------------------------------------------------- init -------
__global__ void k_fill_u32(u32* __restrict__ a, i64 n, u32 v) {
  i64 i = (i64)blockIdx.x * blockDim.x + threadIdx.x;
  i64 stride = (i64)gridDim.x * blockDim.x;
  for (; i < n; i += stride) a[i] = v;
}

// Alg. 2 l.1-3: dist[s] = 0, bucket 0 queue holds (s, 0), counters reset.
struct AdaptInit {
  u32 mode;        // 0 fixed Delta, 1 / 2 adaptive (readings A / B of Eq. (2))
  float d0;        // Delta_0 in fine units
  u32 m0, mmin, mmax, lvl0;
  u32 first_n;     // ids [0, first_n) hold every vertex with arcs and the source
  u32 bf_t;        // Bellman-Ford end threshold (entries left in the ring; 0 = never)
};
__global__ void k_seed(Params p, u32 src, AdaptInit ai) {
  const u32 t = threadIdx.x;
  for (u32 s = t; s < p.K; s += blockDim.x) {
    p.sc[s].word = 0;
    p.sc[s].head = 0;
    p.sc[s].p2 = 0;
  }
  if (t < ST_N) p.stats[t] = 0;
  __syncthreads();
  if (t == 0) {
    p.dist[src] = 0;
    p.items[0] = (u64)src;  // (d=0 << 32) | src in bucket 0, slot 0
    p.sc[0].word = (1ULL << 32) | 1ULL;
    Ctl* c = p.ctl;
    c->cur = 0;
    c->lim = p.K - 1;
    c->mode = MODE_PHASE1;
    c->far_min = NONE;
    c->p2_begin = c->p2_end = c->p2_head = 0;
    c->err = 0;
    c->bar_count = 0;
    c->bar_gen = 0;
    c->t_first = ~0ULL;
    c->epochs = 1;
    c->rescans = 0;
    c->rescan_base = 0;
    c->changed = 0;
    c->sweep_first = 0;
    c->sweeps = 0;
    c->hub_word = 0;
    c->hub_head = 0;
    c->trace_n = 0;
    c->round_end = 1;
    c->rounds = 0;
    c->cur_end = ai.m0;
    c->a_mode = ai.mode;
    c->a_i = 0;
    c->a_c1 = c->a_c2 = c->a_t1 = c->a_t2 = 0;
    c->a_dlt = ai.d0;
    c->a_d0 = ai.d0;
    c->a_mmin = ai.mmin;
    c->a_mmax = ai.mmax;
    c->a_m = ai.m0;
    c->lvl = ai.lvl0;
    c->csum = 0;
    c->pull_sel = 2;  // the first pull scans every vertex
    c->pull_n[0] = c->pull_n[1] = 0;
    c->closed_b = NONE;
    c->closed_c = 0;
    c->long_n = c->long_head = 0;
    c->sample_n = 0;
    c->first_n = ai.first_n;
    c->bf = 0;
    c->bf_t = ai.bf_t;
    c->bf_peak = 0;
  }
}

}  // namespace sssp
