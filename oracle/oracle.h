/* oracle.h -- plain, slow, obviously-correct CPU oracle for the SSSP hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may load this library. The product path
 * (paper_conf_icppw_zhangczsdhay23_b200/, libsssp.so) never calls it and shares
 * no code with it.
 *
 * Citations: "P:n" = line n of the paper text PAPER.md (Zhang et al., "A
 * Bucket-aware Asynchronous Single-Source Shortest Path Algorithm on GPU",
 * ICPP-W 2023).
 *
 * What the method computes (plain definition, PAPER §2.1, Alg. 1
 * P:231-240; Delta-stepping is exact for every Delta):
 *   d[s] = 0, d[v] = min over s->v paths of len(path), INF if unreachable,
 * where len is the exact integer sum for u32 weights and the left-to-right
 * float32 round-to-nearest sum fl(fl(w1+w2)+w3)... for f32 weights (that is
 * what every relaxation new_dist = dist[u] + w of Alg. 1 line 1 computes).
 * INF is 0xFFFFFFFF (u32) / +inf (f32).
 *
 * Parity pins (tests/test_oracle_pins.py): Fig. 1 and Fig. 4 worked examples,
 * closed forms (grid Manhattan distance, path prefix sums, star, unit-weight
 * BFS), brute-force path enumeration / Floyd-Warshall / Bellman-Ford on tiny
 * random graphs, the f32 left-to-right path pin, and the
 * certificate checker against corrupted inputs.
 */
#ifndef SSSP_ORACLE_H
#define SSSP_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_OK 0
#define ORACLE_ERR_ARG 1
#define ORACLE_ERR_OVERFLOW 5

/* Dijkstra, PAPER §2.1: indexed binary heap with decrease-key.
 * u32: exact u64 accumulation; returns ORACLE_ERR_OVERFLOW if a finite
 * distance would reach 0xFFFFFFFF. f32: new_dist = dist[u] + w in binary32. */
int oracle_dijkstra_u32(int64_t V, const int64_t* row, const uint32_t* col, const uint32_t* w,
                        int64_t src, uint32_t* dist);
int oracle_dijkstra_f32(int64_t V, const int64_t* row, const uint32_t* col, const float* w,
                        int64_t src, float* dist);

/* Bellman-Ford, PAPER §2.1: relax every arc until no change
 * (at most V rounds). Returns the number of rounds, or -1 on overflow. */
int64_t oracle_bellman_ford_u32(int64_t V, const int64_t* row, const uint32_t* col,
                                const uint32_t* w, int64_t src, uint32_t* dist);
int64_t oracle_bellman_ford_f32(int64_t V, const int64_t* row, const uint32_t* col,
                                const float* w, int64_t src, float* dist);

/* Floyd-Warshall all-pairs (u32 only: its tree-shaped sums are exact for
 * integers but not for float32). D is V*V u64, UINT64_MAX = unreachable. */
int oracle_floyd_warshall_u32(int64_t V, const int64_t* row, const uint32_t* col,
                              const uint32_t* w, uint64_t* D);

/* Certificate: d[s]=0; for every arc with d[u]<INF d[v]<=d[u]+w;
 * every finite d[v], v!=s, tight on an arc with d[u] < d[v]. A complete proof
 * of optimality for integer weights >= 1. Returns -1 if valid, else the first
 * offending vertex id (or V for a bad source entry). */
int64_t oracle_certificate_u32(int64_t V, const int64_t* row, const uint32_t* col,
                               const uint32_t* w, int64_t src, const uint32_t* dist);

/* Property-driven reordering, PAPER §4.1, Fig. 4:
 *  1. relabel vertices by descending degree (ties: ascending original id,
 *     pinned by Fig. 4: degrees 2,4,2,3,3 -> new2old 1,3,4,0,2);
 *  2. sort every adjacency by ascending weight (ties: ascending new id);
 * Outputs new2old[V], old2new[V], new_row[V+1], adj[A] (new ids), val[A]
 * (weight bits; f32 bits order like the values since weights are >= 0). */
int oracle_pro_reorder(int64_t V, const int64_t* row, const uint32_t* col, const uint32_t* wbits,
                       uint32_t* new2old, uint32_t* old2new, int64_t* new_row, uint32_t* adj,
                       uint32_t* val);

/* Heavy-edge offsets added to the row list: the
 * interleaved list start_0, heavy_0, start_1, heavy_1, ..., end (2V+1
 * entries), heavy_v = first arc of v whose weight is not light. Light means
 * w < Delta. wtype 0 = u32 (Delta rounded up to an integer),
 * 1 = f32 (Delta rounded to nearest binary32). */
void oracle_pro_rowlist(int64_t V, const int64_t* new_row, const uint32_t* val, int wtype,
                        double delta, int64_t* rowlist);

/* Bucket index of a distance, B_i = [i*Delta, (i+1)*Delta):
 * u32: d / ceil(Delta); f32: (u32)(d * fl32(1/Delta)). Histogram of final
 * distances per bucket (INF excluded) into counts[0..nb); returns the number
 * of buckets needed (max index + 1), counts only written below nb. */
int64_t oracle_bucket_histogram(int64_t V, const uint32_t* dist_bits, int wtype, double delta,
                                int64_t* counts, int64_t nb);

#ifdef __cplusplus
}
#endif
#endif
