/* gen.c -- seeded synthetic graph generators; see gen.h for the contract.
 * Holds no SSSP arithmetic: only random draws, edge lists and CSR assembly. */
#include "gen.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- RNG --- */
static inline uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

uint64_t gen_rand64(uint64_t seed, uint64_t stream, uint64_t counter) {
    uint64_t key = mix64(seed * 0x9E3779B97F4A7C15ULL + stream + 0x632BE59BD9B4E019ULL);
    return mix64(key + (counter + 1) * 0x9E3779B97F4A7C15ULL);
}

enum { STREAM_KRON = 1, STREAM_FEISTEL = 2, STREAM_WEIGHT = 3, STREAM_GRID = 4, STREAM_SRC = 5 };

/* ----------------------------------------------------------- threading --- */
typedef void (*range_fn)(void* ctx, int64_t lo, int64_t hi);
typedef struct {
    range_fn fn;
    void* ctx;
    int64_t n, chunk;
    int64_t next; /* atomic work counter */
} pf_state;

static void* pf_worker(void* arg) {
    pf_state* s = (pf_state*)arg;
    for (;;) {
        int64_t lo = __atomic_fetch_add(&s->next, s->chunk, __ATOMIC_RELAXED);
        if (lo >= s->n) break;
        int64_t hi = lo + s->chunk < s->n ? lo + s->chunk : s->n;
        s->fn(s->ctx, lo, hi);
    }
    return NULL;
}

static void parallel_for(int64_t n, int64_t chunk, int nthreads, range_fn fn, void* ctx) {
    if (n <= 0) return;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    pf_state s = {fn, ctx, n, chunk < 1 ? 1 : chunk, 0};
    if (nthreads == 1 || n <= chunk) {
        pf_worker(&s);
        return;
    }
    pthread_t th[256];
    int started = 0;
    for (int t = 1; t < nthreads; ++t)
        if (pthread_create(&th[started], NULL, pf_worker, &s) == 0) ++started;
    pf_worker(&s);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
}

/* ------------------------------------------------------------ Feistel --- */
uint32_t gen_scramble(uint32_t x, int scale, uint64_t seed) {
    int lb = scale / 2, rb = scale - lb;
    uint32_t lmask = lb ? (uint32_t)((1ULL << lb) - 1) : 0u;
    uint32_t rmask = (uint32_t)((1ULL << rb) - 1);
    uint32_t L = (uint32_t)(((uint64_t)x >> rb) & lmask), R = x & rmask;
    for (int k = 0; k < 4; ++k) {
        if ((k & 1) == 0)
            L ^= (uint32_t)gen_rand64(seed, STREAM_FEISTEL, ((uint64_t)k << 32) | R) & lmask;
        else
            R ^= (uint32_t)gen_rand64(seed, STREAM_FEISTEL, ((uint64_t)k << 32) | L) & rmask;
    }
    return (uint32_t)(((uint64_t)L << rb) | R);
}

/* ---------------------------------------------------------- Kronecker --- */
/* P(row bit) = C+D = .24; P(col | row=0) = B/(A+B); P(col | row=1) = D/(C+D).
 * Bit set iff a u32 draw x >= T. */
#define T_AB 3264175145u /* ceil(0.76 * 2^32) */
#define T_A 3221225472u  /* ceil(A/(A+B) * 2^32) = ceil(0.75 * 2^32) */
#define T_C 3400182443u  /* ceil(C/(C+D) * 2^32) */

typedef struct {
    int scale, scramble;
    uint64_t seed;
    uint32_t *src, *dst;
} kron_ctx;

static void kron_range(void* c, int64_t lo, int64_t hi) {
    kron_ctx* k = (kron_ctx*)c;
    for (int64_t i = lo; i < hi; ++i) {
        uint32_t u = 0, v = 0;
        for (int l = 0; l < k->scale; ++l) {
            uint64_t x = gen_rand64(k->seed, STREAM_KRON, (uint64_t)i * 64u + (uint64_t)l);
            uint32_t xr = (uint32_t)x, xc = (uint32_t)(x >> 32);
            uint32_t rb = xr >= T_AB;
            uint32_t cb = rb ? (xc >= T_C) : (xc >= T_A);
            u = (u << 1) | rb;
            v = (v << 1) | cb;
        }
        if (k->scramble) {
            u = gen_scramble(u, k->scale, k->seed);
            v = gen_scramble(v, k->scale, k->seed);
        }
        k->src[i] = u;
        k->dst[i] = v;
    }
}

void gen_kronecker_edges(int scale, int64_t num_edges, uint64_t seed, int scramble,
                         uint32_t* src, uint32_t* dst, int nthreads) {
    kron_ctx k = {scale, scramble, seed, src, dst};
    parallel_for(num_edges, 1 << 16, nthreads, kron_range, &k);
}

/* --------------------------------------------------------------- grid --- */
int64_t gen_grid_edges(int64_t W, int64_t H, double p_vertical, uint64_t seed,
                       uint32_t* src, uint32_t* dst, uint64_t* eid) {
    int64_t n = 0;
    int64_t nh = H * (W - 1);
    double t = p_vertical * 4294967296.0;
    uint64_t thr = t >= 4294967296.0 ? (1ULL << 32) : (uint64_t)t;
    for (int64_t r = 0; r < H; ++r) {
        for (int64_t c = 0; c + 1 < W; ++c) {
            src[n] = (uint32_t)(r * W + c);
            dst[n] = (uint32_t)(r * W + c + 1);
            eid[n] = (uint64_t)(r * (W - 1) + c);
            ++n;
        }
        if (r + 1 < H) {
            for (int64_t c = 0; c < W; ++c) {
                uint64_t id = (uint64_t)(nh + r * W + c);
                if ((gen_rand64(seed, STREAM_GRID, id) & 0xFFFFFFFFULL) < thr) {
                    src[n] = (uint32_t)(r * W + c);
                    dst[n] = (uint32_t)((r + 1) * W + c);
                    eid[n] = id;
                    ++n;
                }
            }
        }
    }
    return n;
}

/* ------------------------------------------------------------ weights --- */
typedef struct {
    const uint64_t* eid;
    uint64_t seed;
    uint32_t lo, hi;
    void* w;
} w_ctx;

static void wu32_range(void* c, int64_t lo, int64_t hi) {
    w_ctx* k = (w_ctx*)c;
    uint64_t span = (uint64_t)k->hi - k->lo + 1;
    uint32_t* w = (uint32_t*)k->w;
    for (int64_t i = lo; i < hi; ++i) {
        uint64_t id = k->eid ? k->eid[i] : (uint64_t)i;
        uint64_t x = gen_rand64(k->seed, STREAM_WEIGHT, id) & 0xFFFFFFFFULL;
        w[i] = k->lo + (uint32_t)((x * span) >> 32);
    }
}

static void wf32_range(void* c, int64_t lo, int64_t hi) {
    w_ctx* k = (w_ctx*)c;
    float* w = (float*)k->w;
    for (int64_t i = lo; i < hi; ++i) {
        uint64_t id = k->eid ? k->eid[i] : (uint64_t)i;
        uint32_t x = (uint32_t)gen_rand64(k->seed, STREAM_WEIGHT, id);
        w[i] = (float)((x >> 8) + 1) * (1.0f / 16777216.0f); /* exact: (u24+1)*2^-24 */
    }
}

void gen_weights_u32(int64_t n, const uint64_t* eid, uint64_t seed, uint32_t lo, uint32_t hi,
                     uint32_t* w, int nthreads) {
    w_ctx k = {eid, seed, lo, hi, w};
    parallel_for(n, 1 << 18, nthreads, wu32_range, &k);
}

void gen_weights_f32(int64_t n, const uint64_t* eid, uint64_t seed, float* w, int nthreads) {
    w_ctx k = {eid, seed, 0, 0, w};
    parallel_for(n, 1 << 18, nthreads, wf32_range, &k);
}

/* ---------------------------------------------------------------- CSR --- */
typedef struct {
    int64_t E;
    const uint32_t *src, *dst, *w;
    int symmetrize;
    int64_t* cnt;          /* pass 1: degree counters (row+1) */
    int64_t* cursor;       /* pass 2 */
    uint64_t* tmp;         /* packed (dst<<32 | w) per arc */
    const int64_t* row;
    uint32_t *col, *wout;
} csr_ctx;

static void deg_range(void* c, int64_t lo, int64_t hi) {
    csr_ctx* k = (csr_ctx*)c;
    for (int64_t i = lo; i < hi; ++i) {
        uint32_t u = k->src[i], v = k->dst[i];
        if (u == v) continue;
        __atomic_fetch_add(&k->cnt[u], 1, __ATOMIC_RELAXED);
        if (k->symmetrize) __atomic_fetch_add(&k->cnt[v], 1, __ATOMIC_RELAXED);
    }
}

int64_t gen_csr_rows(int64_t V, int64_t E, const uint32_t* src, const uint32_t* dst,
                     int symmetrize, int64_t* row, int nthreads) {
    memset(row, 0, sizeof(int64_t) * (size_t)(V + 1));
    csr_ctx k;
    memset(&k, 0, sizeof k);
    k.E = E;
    k.src = src;
    k.dst = dst;
    k.symmetrize = symmetrize;
    k.cnt = row + 1;
    parallel_for(E, 1 << 16, nthreads, deg_range, &k);
    /* row[v+1] holds deg(v); inclusive scan turns it into CSR offsets */
    for (int64_t v = 0; v < V; ++v) row[v + 1] += row[v];
    return row[V];
}

static void scatter_range(void* c, int64_t lo, int64_t hi) {
    csr_ctx* k = (csr_ctx*)c;
    for (int64_t i = lo; i < hi; ++i) {
        uint32_t u = k->src[i], v = k->dst[i];
        if (u == v) continue;
        uint32_t w = k->w[i];
        int64_t p = __atomic_fetch_add(&k->cursor[u], 1, __ATOMIC_RELAXED);
        k->tmp[p] = ((uint64_t)v << 32) | w;
        if (k->symmetrize) {
            p = __atomic_fetch_add(&k->cursor[v], 1, __ATOMIC_RELAXED);
            k->tmp[p] = ((uint64_t)u << 32) | w;
        }
    }
}

static int cmp_u64(const void* a, const void* b) {
    uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
    return x < y ? -1 : x > y;
}

static void sort_rows_range(void* c, int64_t lo, int64_t hi) {
    csr_ctx* k = (csr_ctx*)c;
    for (int64_t v = lo; v < hi; ++v) {
        int64_t b = k->row[v], e = k->row[v + 1], n = e - b;
        uint64_t* a = k->tmp + b;
        if (n <= 48) {
            for (int64_t i = 1; i < n; ++i) {
                uint64_t x = a[i];
                int64_t j = i - 1;
                while (j >= 0 && a[j] > x) {
                    a[j + 1] = a[j];
                    --j;
                }
                a[j + 1] = x;
            }
        } else {
            qsort(a, (size_t)n, sizeof(uint64_t), cmp_u64);
        }
        for (int64_t i = 0; i < n; ++i) {
            k->col[b + i] = (uint32_t)(a[i] >> 32);
            k->wout[b + i] = (uint32_t)a[i];
        }
    }
}

void gen_csr_fill(int64_t V, int64_t E, const uint32_t* src, const uint32_t* dst,
                  const uint32_t* w, int symmetrize, const int64_t* row,
                  uint32_t* col, uint32_t* wout, int nthreads) {
    int64_t A = row[V];
    csr_ctx k;
    memset(&k, 0, sizeof k);
    k.E = E;
    k.src = src;
    k.dst = dst;
    k.w = w;
    k.symmetrize = symmetrize;
    k.row = row;
    k.col = col;
    k.wout = wout;
    k.cursor = (int64_t*)malloc(sizeof(int64_t) * (size_t)(V > 0 ? V : 1));
    k.tmp = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(A > 0 ? A : 1));
    memcpy(k.cursor, row, sizeof(int64_t) * (size_t)V);
    parallel_for(E, 1 << 16, nthreads, scatter_range, &k);
    parallel_for(V, 1 << 12, nthreads, sort_rows_range, &k);
    free(k.cursor);
    free(k.tmp);
}

/* ------------------------------------------------------------ sources --- */
int64_t gen_sample_sources(int64_t V, const int64_t* row, int64_t n, uint64_t seed, int64_t* out) {
    int64_t found = 0;
    for (uint64_t c = 0; found < n && c < (uint64_t)V * 64 + 1024; ++c) {
        int64_t v = (int64_t)(gen_rand64(seed, STREAM_SRC, c) % (uint64_t)V);
        if (row[v + 1] == row[v]) continue;
        int dup = 0;
        for (int64_t j = 0; j < found; ++j)
            if (out[j] == v) dup = 1;
        if (!dup) out[found++] = v;
    }
    return found;
}
