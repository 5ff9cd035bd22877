/* gen.h -- seeded synthetic graph generators (Kronecker / road-like grid).
 *
 * This module is the ONLY code shared by the CPU oracle side (tests, bench's
 * cpu_baseline) and the CUDA path: it produces inputs and holds none of the
 * method's arithmetic (no relaxation, no bucketing, no reordering).
 *
 * Workloads follow PAPER.md §5.1.2: Graph500 Kronecker
 * generator with A=.57 B=.19 C=.19 D=.05, V = 2^SCALE, E = edgefactor*2^SCALE.
 * Per-level quadrant bits use integer thresholds on u32 draws so
 * the graph is bit-reproducible; vertex labels are scrambled with a 4-round
 * Feistel bijection on SCALE bits (Graph500 practice).
 * Weights: u32 U{lo..hi} or f32 ((x>>8)+1)*2^-24 in (0,1] (BASELINE.json).
 *
 * All randomness is counter-based (splitmix64 of seed/stream/counter), so the
 * output does not depend on the number of threads.
 */
#ifndef SSSP_GEN_H
#define SSSP_GEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* 64-bit counter-based draw: stream selects an independent sequence. */
uint64_t gen_rand64(uint64_t seed, uint64_t stream, uint64_t counter);

/* Feistel label scramble on `scale` bits (bijective on [0, 2^scale)). */
uint32_t gen_scramble(uint32_t x, int scale, uint64_t seed);

/* Kronecker edge list: num_edges edges (src[i], dst[i]) in [0, 2^scale). */
void gen_kronecker_edges(int scale, int64_t num_edges, uint64_t seed, int scramble,
                         uint32_t* src, uint32_t* dst, int nthreads);

/* Road-like grid W x H, row-major ids: every horizontal edge, each vertical
 * edge kept with probability p_vertical. Returns the number of edges written
 * (capacity needed: H*(W-1) + (H-1)*W). Edge i keeps counter-id `eid[i]`
 * (horizontal edges first) so weights are independent of the kept set. */
int64_t gen_grid_edges(int64_t W, int64_t H, double p_vertical, uint64_t seed,
                       uint32_t* src, uint32_t* dst, uint64_t* eid);

/* Per-edge weights indexed by edge counter id (eid==NULL means eid[i]=i). */
void gen_weights_u32(int64_t n, const uint64_t* eid, uint64_t seed, uint32_t lo, uint32_t hi,
                     uint32_t* w, int nthreads);
void gen_weights_f32(int64_t n, const uint64_t* eid, uint64_t seed, float* w, int nthreads);

/* CSR build, pass 1: arcs per vertex (self-loops dropped; symmetrize adds the
 * reverse arc). Writes row[0..V] as exclusive prefix sums; returns A = row[V]. */
int64_t gen_csr_rows(int64_t V, int64_t E, const uint32_t* src, const uint32_t* dst,
                     int symmetrize, int64_t* row, int nthreads);

/* CSR build, pass 2: fill col/wout (4-byte weights, u32 or f32 bits). Each
 * adjacency is ordered by (dst, weight bits) ascending -> deterministic. */
void gen_csr_fill(int64_t V, int64_t E, const uint32_t* src, const uint32_t* dst,
                  const uint32_t* w, int symmetrize, const int64_t* row,
                  uint32_t* col, uint32_t* wout, int nthreads);

/* n distinct source vertices with out-degree >= 1 (PAPER P:1229-1230:
 * "64 different starting vertices randomly"). Returns how many were found. */
int64_t gen_sample_sources(int64_t V, const int64_t* row, int64_t n, uint64_t seed, int64_t* out);

#ifdef __cplusplus
}
#endif
#endif
