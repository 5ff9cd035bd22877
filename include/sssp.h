/* sssp.h -- C-ABI of the B200-native bucket-aware asynchronous Delta-stepping
 * SSSP library (libsssp.so, sm_100a).
 *
 * Method: Zhang et al., "A Bucket-aware Asynchronous Single-Source Shortest
 * Path Algorithm on GPU", ICPP-W 2023. "P:n" cites line n of PAPER.md.
 * Problem statement (Alg. 2 header P:1072-1075): given a graph
 * G=(V,E,W), a starting vertex s and Delta, return the final shortest
 * distance array dist.
 *
 * Conventions for every function:
 *  - Return an sssp_status; never abort, never throw across the ABI. A
 *    thread-local detail string is available from sssp_last_error().
 *  - SSSP_ERR_CUDA is sticky for a handle: destroy it.
 *  - All vertex ids at the API are the caller's ORIGINAL ids, also after
 *    sssp_reorder (the relabelling is internal).
 *  - Inputs are copied; the caller keeps ownership of every buffer it passes.
 *    Output buffers are caller-allocated. The handle owns its device memory
 *    until sssp_destroy.
 *  - One host thread per handle at a time; handles are independent.
 *  - Work is stream-ordered on the handle's stream (sssp_set_stream); only
 *    sssp_graph_create, sssp_distances(HOST), sssp_get_stats and the export
 *    helpers synchronise that stream.
 */
#ifndef SSSP_H
#define SSSP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sssp_graph_s* sssp_graph_t; /* opaque, library-owned */

typedef enum {
    SSSP_OK = 0,
    SSSP_ERR_INVALID_ARGUMENT = 1, /* bad size/pointer/id/Delta/CSR/weight */
    SSSP_ERR_OUT_OF_MEMORY = 2,
    SSSP_ERR_CUDA = 3,             /* CUDA runtime failure (sticky) */
    SSSP_ERR_INVALID_STATE = 4,    /* e.g. sssp_distances before a successful sssp_run */
    SSSP_ERR_OVERFLOW = 5,         /* a u32 distance reached 0xFFFFFFFF */
    SSSP_ERR_INTERNAL = 6          /* scheduler safety cap hit (should not happen) */
} sssp_status;

typedef enum { SSSP_WEIGHT_U32 = 0, SSSP_WEIGHT_F32 = 1 } sssp_weight_type;
typedef enum { SSSP_MEM_HOST = 0, SSSP_MEM_DEVICE = 1 } sssp_memory;

/* Create a graph handle on CUDA device `device` from a CSR (DS-1):
 *   row_offsets [V+1] int64: row[0]=0, non-decreasing, row[V]=A;
 *   col_indices [A] uint32: each < V (arcs are directed; pass both directions
 *                for an undirected graph, as the paper's figures do);
 *   weights     [A] uint32, or float32 finite and >= 0 (-0.0 becomes +0.0).
 * `where` says whether the three arrays are host or device pointers.
 * 1 <= V < 2^31 and 0 <= A < 2^32 (arc offsets are kept 64-bit internally).
 * V < 2^31 rather than SURVEY §8(b)'s 2^32-1: bit 31 of a queued vertex id
 * marks a 4096-arc hub chunk in the bucket queues. Every BASELINE
 * config (largest C5: V = 2^26) is far inside this range.
 * cuda_stream: a cudaStream_t (NULL = legacy default stream).
 * Validation runs on the device; the call synchronises the stream and returns
 * SSSP_ERR_INVALID_ARGUMENT on any violation (*out untouched). */
sssp_status sssp_graph_create(sssp_graph_t* out, int device, int64_t num_vertices,
                              int64_t num_arcs, const int64_t* row_offsets,
                              const uint32_t* col_indices, const void* weights,
                              sssp_weight_type wtype, sssp_memory where, void* cuda_stream);

/* Property-driven reordering (PRO, PAPER §4.1, Fig. 4), on the GPU:
 * relabel vertices by descending degree (ties by ascending original id) with
 * a radix sort, permute the CSR, sort every adjacency by ascending weight
 * (ties by ascending new id), and keep a heavy-edge offset per vertex in the
 * row list (recomputed whenever Delta changes).
 * Idempotent. Invalidates the previous sssp_run result. */
sssp_status sssp_reorder(sssp_graph_t g);

#define SSSP_PRO_DEGREE 1u /* relabel by descending degree */
#define SSSP_PRO_WEIGHT 2u /* sort adjacencies by weight + heavy offsets */
/* Ablation variant of sssp_reorder: flags = any subset of the two steps
 * (0 restores nothing: reorder is one-way; 0 is a no-op). A graph with
 * SSSP_PRO_WEIGHT uses the light/heavy split by offset; without it phases 1
 * and 2 both scan whole adjacencies with a per-arc w < Delta predicate. */
sssp_status sssp_reorder_ex(sssp_graph_t g, unsigned flags);

/* Single-source shortest paths from `source` (original id, 0 <= source < V)
 * with bucket width `delta` (> 0; u32 graphs round it UP to an integer >= 1;
 * f32 graphs round it to nearest binary32; +inf = one bucket, i.e. the
 * Bellman-Ford end of Delta-stepping). Light arcs: w < Delta
 * (P:265-266); bucket i holds distances in [i*Delta,(i+1)*Delta).
 * Runs the bucket-aware asynchronous Delta-stepping of Alg. 2
 * in one persistent cooperative kernel: phase 1 (light arcs, asynchronous,
 * adaptive thread/warp/CTA bins),
 * then fused phases 2&3 (heavy arcs + next bucket).
 * Asynchronous w.r.t. the host (stream-ordered): launch errors come back
 * here, run-time errors (u32 overflow, scheduler cap) are recorded on the
 * device and reported by the next sssp_distances / sssp_wait /
 * sssp_run_batch, which synchronise (see "Run errors" below).
 * With SSSP_PARAM_PULL_SYMMETRIC set on a weight-sorted graph, the first run
 * checks the arc multiset for symmetry (once per reorder) and returns
 * SSSP_ERR_INVALID_STATE if it is not symmetric. */
sssp_status sssp_run(sssp_graph_t g, int64_t source, double delta);

/* Copy the last run's distances (V elements of the graph's weight type, in
 * ORIGINAL vertex order; unreachable = 0xFFFFFFFF for u32, +inf for f32) to
 * `out` (host or device per `where`). HOST synchronises the stream; a pinned,
 * device-mapped host buffer (cudaHostAlloc, torch pin_memory) is written
 * directly by the output gather kernel, pageable memory is staged through a
 * library-owned device buffer (allocated on first use, freed by destroy).
 * SSSP_ERR_INVALID_STATE if no successful run since create/reorder;
 * otherwise the run errors (below) of every run since the last report.
 *
 * Run errors. Each persistent run ORs its error bits into a per-handle device
 * word that survives later runs; sssp_distances, sssp_wait and sssp_run_batch
 * synchronise, report that word and clear it, so no run's error is lost:
 *   SSSP_ERR_OVERFLOW: a relaxation d[u] + w of a u32 graph reached
 *     0xFFFFFFFF. Always reported when some reachable vertex's shortest
 *     distance is >= 0xFFFFFFFF (its result would be wrong); may also be
 *     reported when only a longer path's sum overflows (push relaxations
 *     check every sum they form, Alg. 1 l.1).
 *   SSSP_ERR_INTERNAL: a hub-chunk queue overflowed in phase 2 (work was
 *     dropped; the handle's queues are fully reset before the next run). */
sssp_status sssp_distances(sssp_graph_t g, void* out, sssp_memory where);

/* Free every resource of the handle. NULL-safe. */
void sssp_destroy(sssp_graph_t g);

/* ------------------------------------------------------------ helpers --- */
const char* sssp_status_string(sssp_status s);
const char* sssp_last_error(void); /* thread-local detail of the last failure */

/* Make subsequent work on g use cuda_stream (a cudaStream_t; NULL = default). */
sssp_status sssp_set_stream(sssp_graph_t g, void* cuda_stream);

/* Asynchronous sssp_distances: the output gather of the last run (original
 * ids, graph weight type) goes to one of two device staging buffers on the
 * handle's stream, then a copy engine moves it to `out` on the handle's own
 * output stream, so the transfer overlaps the next sssp_run. out: pinned host
 * memory (cudaHostAlloc / torch pin_memory) or device memory (written on the
 * handle's stream); valid, and not touched by the caller, until sssp_wait.
 * Pageable memory: SSSP_ERR_INVALID_ARGUMENT. INVALID_STATE before a run. */
sssp_status sssp_distances_async(sssp_graph_t g, void* out, sssp_memory where);

/* Waits for every output enqueued by sssp_distances_async and for every run
 * enqueued on the handle's stream, then reports (and clears) the run errors
 * of all runs since the last report (see sssp_distances). */
sssp_status sssp_wait(sssp_graph_t g);

/* Multi-source batch (the naturally sharded case of the north star): for
 * i < n run sssp_run(sources[i], delta) and write the distances (original
 * order) to the DEVICE buffer out_dev + i*ld elements (ld >= V). sources is a
 * host array. Enqueues all n runs, then synchronises once and reports the run
 * errors of the batch (and of any earlier unreported run). */
sssp_status sssp_run_batch(sssp_graph_t g, const int64_t* sources, int64_t n, double delta,
                           void* out_dev, int64_t ld);

/* NEXT-4 (beyond the paper): the same batch as sssp_run_batch
 * (row i = distances from sources[i], original ids, out_dev + i*ld, ld >= V,
 * device buffer) computed 32 sources per persistent launch: distances are
 * kept as D[v][32] (128-byte rows), so one arc read and one coalesced row
 * probe serve 32 sources. Work items are vertices queued in Delta-width
 * buckets by their smallest improved distance; an expansion relaxes every
 * finite lane (label-correcting: exact, identical to sssp_run per source for
 * u32 and f32). Allocates 132 B per vertex plus the ring on first use.
 * Synchronises once per group of 32 sources; SSSP_ERR_OVERFLOW if a u32
 * relaxation of any group overflowed (each group's error word is read before
 * the next group starts). */
sssp_status sssp_run_multi(sssp_graph_t g, const int64_t* sources, int64_t n, double delta,
                           void* out_dev, int64_t ld);

/* Counters of the last sssp_run_multi group: out[0] successful lane updates,
 * [1] arcs relaxed (each for all 32 lanes), [2] vertex expansions, [3] stale
 * queue items, [4] split items (256-arc pieces), [5] buckets, [6] rescans.
 * Writes min(n, 7) values. SSSP_ERR_INVALID_STATE before the first call. */
sssp_status sssp_multi_stats(sssp_graph_t g, uint64_t* out, int64_t n);

/* Counters of the last run (the work-efficiency metric of P:410-413 and
 * updates = successful atomicMin writes; a valid update is one
 * that writes the final distance, so valid = reachable - 1). Synchronises. */
typedef struct sssp_stats {
    uint64_t updates;          /* successful atomicMin improvements (total updates) */
    uint64_t light_arcs;       /* light arcs relaxed in phase 1 */
    uint64_t heavy_arcs;       /* heavy arcs relaxed in phase 2 */
    uint64_t vertices_settled; /* phase-1 vertex items processed (non-stale) */
    uint64_t stale_items;      /* phase-1 items skipped as stale */
    uint64_t heavy_vertices;   /* phase-2 vertices whose heavy arcs were relaxed */
    uint64_t hub_chunks;       /* 4096-arc chunks of vertices with > 4096 arcs in range */
    uint64_t bin_thread;       /* vertices relaxed by the thread bin (< 32 arcs) */
    uint64_t bin_warp;         /* ... warp bin (32..255) */
    uint64_t bin_cta;          /* ... CTA bin (256..4096) */
    uint64_t buckets;          /* phase-1 epochs run (buckets + reopenings) */
    uint64_t rescans;          /* overflow fall-back rescans of dist[] */
    uint64_t reachable;        /* vertices with a finite distance (filled by sssp_distances) */
    uint64_t levels;           /* extra phase-1 frontier levels (SSSP_PARAM_SYNC=1 only) */
    uint32_t ring_slots;       /* K: bucket-queue ring size used */
    uint32_t grid_ctas;        /* persistent grid size */
    float run_ms;              /* device time of the last sssp_run (CUDA events) */
    float reorder_ms;          /* device time of the last sssp_reorder */
} sssp_stats;
sssp_status sssp_get_stats(sssp_graph_t g, sssp_stats* s);

/* Export the internal CSR (for parity tests against the paper's Fig. 4):
 * rowlist [2V+1] int64 interleaved (start_v, heavy_v) + end with heavy offsets
 * for `delta` (Fig. 4c layout); adj [A] uint32 internal ids;
 * val [A] weights (4-byte, graph type); new2old [V] uint32 (identity if not
 * reordered). Host pointers; any may be NULL. Synchronises. */
sssp_status sssp_export_csr(sssp_graph_t g, double delta, int64_t* rowlist, uint32_t* adj,
                            void* val, uint32_t* new2old);

/* Tunables (defaults in brackets). Values are validated; takes effect at the
 * next sssp_run. */
#define SSSP_BF_TAIL_DEFAULT 262144  /* entries: SSSP_PARAM_BF_TAIL's default */
typedef enum {
    SSSP_PARAM_RING_SLOTS = 0,     /* K bucket queues, power of two in [4,64]; 0 = auto [0] */
    SSSP_PARAM_CTAS_PER_SM = 1,    /* persistent CTAs per SM; 0 = max co-resident [0] */
    SSSP_PARAM_SLOT_CAPACITY = 2,  /* entries per bucket queue; 0 = auto (2.5 V + 64Ki) [0] */
    SSSP_PARAM_CLAIM_MAX = 3,      /* max queue entries one CTA claims at once (1..512) [512] */
    SSSP_PARAM_L2_PERSIST = 4,     /* 1: keep dist[] in a persisting L2 window (raises the
                                      device's persisting-L2 limit; never lowers it) [1] */
    SSSP_PARAM_ADWL = 5,           /* ablation: 1 adaptive thread/warp/CTA bins + hub chunks
                                      (P:733-780); 0 static thread per vertex [1] */
    SSSP_PARAM_SYNC = 6,           /* ablation: 1 level-synchronous phase 1 (a grid barrier per
                                      frontier level, the paper's BL); 0 the
                                      bucket-aware asynchronous phase 1 (BASYN) [0] */
    SSSP_PARAM_P2_EDGE_BALANCED = 7, /* phases 2&3 with equal heavy arcs per warp
                                      for buckets with >= value (< 2^23) settled entries; smaller
                                      buckets (and -1 = never) relax heavy arcs through the
                                      phase-1 vertex bins [-1] */
    SSSP_PARAM_ADAPTIVE_DELTA = 8, /* NEXT-1, Eq. (1)-(2) P:1006-1028 (Alg. 2 l.11): 0 fixed
                                      Delta; 1 Delta_i = Delta_{i-1} + eps_i (Eq. (2) as
                                      printed); 2 Delta_i = Delta_0 + eps_i (Fig. 6 text,
                                      P:1033-1037). eps_i from the converged-vertex and thread
                                      counts of the previous two buckets (reading R7: |.| bars),
                                      Delta_i clamped to [Delta_0/4, 4 Delta_0]. The delta of
                                      sssp_run is Delta_0. Distances do not change (Delta-
                                      stepping is exact for every Delta) [0] */
    SSSP_PARAM_MULTI_ALIGN = 9,    /* sssp_run_multi: 1 orders the queue by distance + (M -
                                      d(hub, source)) per source, so the 32 wavefronts that all
                                      pass through the highest-degree vertex reach each vertex in
                                      about the same bucket (one SSSP from that vertex per graph
                                      and Delta, which replaces the last sssp_run result); 0 by
                                      plain distance. Results are identical [1] */
    SSSP_PARAM_MULTI_HUB_DELAY = 10, /* sssp_run_multi on a degree-reordered graph: vertices
                                      of degree > 1024 are queued this many buckets late, so
                                      more of the 32 sources reach a hub before its (long)
                                      adjacency is expanded; 0..16. Results are identical [0] */
    SSSP_PARAM_PULL_SYMMETRIC = 11, /* 1 = the caller asserts the graph is symmetric (every arc
                                      (u,v,w) has its reverse (v,u,w), as the generators' graphs
                                      are, R13): graphs after a weight-sorting sssp_reorder
                                      then run phases 2&3 of buckets holding >= V/128 entries as a
                                      pull (each unsettled vertex scans its weight-sorted heavy
                                      arcs up to the first that cannot win). Same distances.
                                      The assertion is verified once per reorder (sssp_is_
                                      symmetric): setting 1 on a reordered asymmetric graph,
                                      or running with it, returns SSSP_ERR_INVALID_STATE [0] */
    SSSP_PARAM_LOCAL_CHASE = 12,   /* 2: when no arc is heavy at the run's Delta (max weight <
                                      Delta, fixed Delta), a phase-1 push into
                                      the current bucket stays in the pushing CTA's shared
                                      memory (up to one batch) and that CTA relaxes it next,
                                      skipping the global queue round trip; the bucket's
                                      pending count stays > 0 until the CTA's chain is done
                                      (P:1063-1065 leaves the near-list layout open, R10).
                                      1 = the same, only on sparse graphs (A <= 8 V, e.g. road
                                      networks: thin frontiers; on dense ones the CTA-local
                                      depth-first order re-relaxes more). Same distances;
                                      0 = always through the global queue [1] */
    SSSP_PARAM_LOCAL_LIMIT = 13,   /* local-chase entries a CTA keeps (1..512); pushes beyond
                                      go to the global queue, where idle CTAs can take them [512] */
    SSSP_PARAM_BF_TAIL = 14        /* Bellman-Ford end: when a bucket closes, the ring's
                                      queues hold at most this many entries, an earlier bucket
                                      held at least 8x as many (the wave is past its peak) and
                                      no push was dropped beyond the ring, the rest of the run is one
                                      bucket [cur, inf): every queued vertex moves into it and
                                      phase 1 relaxes all arcs (light and heavy) to quiescence.
                                      Delta-stepping with Delta = inf is Bellman-Ford,
                                      so the distances are the same; per-bucket statistics
                                      (trace C_i, heavy relaxations) then stop at the switch.
                                      Fixed Delta and the asynchronous phase 1 only; 0 = never;
                                      -1 = auto: SSSP_BF_TAIL_DEFAULT on graphs with more than
                                      8 arcs per vertex, never on sparser (road-like) ones [-1] */
} sssp_param;
sssp_status sssp_set_param(sssp_graph_t g, sssp_param p, int64_t value);

/* Device time of every persistent-kernel launch (CUDA events recorded around
 * each cooperative launch on the handle's stream): *total_ms = sum since the
 * last reset, *launches = how many. Synchronises on the pending events.
 * reset != 0 zeroes the accumulators after reporting. */
sssp_status sssp_kernel_time(sssp_graph_t g, double* total_ms, int64_t* launches, int reset);

/* Scheduler timeline of the last run: one entry per grid barrier (written by
 * the last CTA to arrive, before it releases the others) plus a kernel-start
 * entry (which = 99). which: 0 end of phase 1, 1 end of phases 2&3, 2/3
 * rescan stages, 4/5 sweep fall-back stages, 6 edge-balanced phase-2
 * compaction, 7 adaptive-Delta slot merge; pad = end of the current bucket in
 * ring-slot units (cur + 1 with a fixed Delta). With SSSP_PARAM_ADAPTIVE_DELTA
 * every closed bucket i also adds which = 8: cur = C_i (settled vertices),
 * tail = T_i (phase-1 queue items), mode = width of the next bucket in slots,
 * far_min = Delta_{i+1} as binary32 bits (in slot units), pad = i + 1.
 * Every entry whose step closed a bucket (moved past it) carries that bucket
 * and its settled-vertex count in closed_b / closed_c (bucket
 * i = distances in [i*Delta, (i+1)*Delta)). Up to 4096 entries. */
typedef struct sssp_trace_entry {
    uint64_t t_ns;   /* %globaltimer */
    uint32_t which;  /* barrier kind (see above) */
    uint32_t cur;    /* current bucket after the scheduler step */
    uint32_t tail;   /* entries in that bucket's queue */
    uint32_t mode;   /* next mode: 0 phase 1, 1 phase 2, 2 done, 3/4 rescan, 5/6 sweep */
    uint32_t far_min, pad;
    uint32_t closed_b; /* bucket (ring-slot units) this scheduler step closed, 0xFFFFFFFF if none */
    uint32_t closed_c; /* C: vertices settled in that bucket (final distance inside it), counted
                          by phases 2&3 (push: entries with d == dist[v]; pull: candidates whose
                          distance lies in the bucket). Exact for u32 graphs; 0xFFFFFFFF
                          (not counted) when the CTA-local chase was on (its in-bucket entries
                          never reach the bucket's queue) */
    uint64_t t_first;  /* %globaltimer of the first CTA's arrival at this barrier */
    uint64_t t_rel;    /* %globaltimer when the scheduler step was done and the grid released */
} sssp_trace_entry;
sssp_status sssp_get_trace(sssp_graph_t g, sssp_trace_entry* out, int64_t max_entries,
                           int64_t* n_entries);

/* Diagnostics of the last run: samples of every 37th CTA, in time order per
 * CTA. which = 100, a phase-1 claim: t_ns = %globaltimer; cur = bucket; tail
 * = queue entries pushed so far; far_min = pending entries; mode = entries
 * claimed (0: the phase ended); pad = first claimed position; closed_b = CTA;
 * closed_c = 1 for a CTA-local batch. which = 101, a processed batch: tail =
 * warp tasks, mode = thread-bin tasks, far_min = range-list entries, t_first
 * / t_rel / pad = SM cycles staging / in warp 0's task loop / waiting for the
 * other warps and flushing, closed_c = 10 * phase + source (batch records only
 * in builds with -DSSSP_BATCH_SAMPLES=1). Up to 16384. */
sssp_status sssp_get_samples(sssp_graph_t g, sssp_trace_entry* out, int64_t max_entries,
                             int64_t* n_entries);

/* Diagnostics of the last run: summed SM cycles of thread 0 of every
 * persistent CTA in [claim, stage, task, tail, grid-barrier], the number of
 * batches and of warp tasks, then (diagnostics builds with SSSP_LAT=1 only,
 * else 0) warp-0 cycles waiting for arcs, dist probes, atomics, staging and
 * the number of tasks measured (12 values). */
sssp_status sssp_get_profile(sssp_graph_t g, uint64_t* out, int n);

/* *out = 1 if the arc multiset is symmetric (every (u,v,w) has its reverse
 * (v,u,w) with the same multiplicity), else 0. Needs weight-sorted
 * adjacencies (sssp_reorder / SSSP_PRO_WEIGHT), else SSSP_ERR_INVALID_STATE:
 * every run of equal arcs is matched by a lower_bound in the other end's
 * sorted segment (one kernel, cached until the next reorder). Synchronises. */
sssp_status sssp_is_symmetric(sssp_graph_t g, int* out);

/* Device-memory allocator hook (process-wide; "the library allocates device
 * memory through an optional allocator hook, so torch's caching allocator can back it").
 * With a hook set, every device buffer a handle owns (graph, queues, distances, staging,
 * reorder temporaries) comes from alloc(bytes, device, stream, ctx), which returns NULL on
 * failure (-> SSSP_ERR_OUT_OF_MEMORY), and goes back through the free_fn of the hook that
 * made it (ptr, bytes, device, stream, ctx) -- also after the hook changes, so set it before
 * creating handles for consistency. The library synchronises its stream before it frees a
 * buffer that work may still use. NULL, NULL restores cudaMalloc / cudaFree; exactly one of
 * the two NULL is SSSP_ERR_INVALID_ARGUMENT. Small per-call scratch words still use
 * stream-ordered cudaMallocAsync. */
typedef void* (*sssp_alloc_fn)(size_t bytes, int device, void* cuda_stream, void* ctx);
typedef void (*sssp_free_fn)(void* ptr, size_t bytes, int device, void* cuda_stream, void* ctx);
sssp_status sssp_set_allocator(sssp_alloc_fn alloc, sssp_free_fn free_fn, void* ctx);

/* Library/device info: number of SMs of the handle's device. */
int sssp_device_sm_count(sssp_graph_t g);

#ifdef __cplusplus
}
#endif
#endif /* SSSP_H */
