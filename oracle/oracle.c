/* oracle.c -- plain CPU oracle for the SSSP hot path. TEST INFRASTRUCTURE ONLY
 * (see oracle.h). Written for obviousness, not speed. Shares no code with the
 * CUDA path. Compiled with -O2 -ffp-contract=off (no FMA, IEEE binary32 adds).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

#define INF_U32 0xFFFFFFFFu

/* ------------------------------------------------ indexed binary heap --- */
/* Min-heap of vertex ids keyed by an external key array; pos[v] = slot or -1.
 * Two key types (u64 for exact u32 sums, float for f32) -> two small copies
 * of the same textbook code. */
typedef struct {
    int64_t* heap;
    int64_t* pos;
    int64_t n;
} iheap;

static int iheap_init(iheap* h, int64_t V) {
    h->heap = (int64_t*)malloc(sizeof(int64_t) * (size_t)(V > 0 ? V : 1));
    h->pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(V > 0 ? V : 1));
    h->n = 0;
    if (!h->heap || !h->pos) return -1;
    for (int64_t v = 0; v < V; ++v) h->pos[v] = -1;
    return 0;
}
static void iheap_free(iheap* h) {
    free(h->heap);
    free(h->pos);
}
static void iheap_swap(iheap* h, int64_t i, int64_t j) {
    int64_t a = h->heap[i], b = h->heap[j];
    h->heap[i] = b;
    h->heap[j] = a;
    h->pos[b] = i;
    h->pos[a] = j;
}

#define DEFINE_HEAP_OPS(SUF, KT)                                                     \
    static void up_##SUF(iheap* h, const KT* key, int64_t i) {                       \
        while (i > 0) {                                                              \
            int64_t p = (i - 1) / 2;                                                 \
            if (key[h->heap[p]] <= key[h->heap[i]]) break;                           \
            iheap_swap(h, i, p);                                                     \
            i = p;                                                                   \
        }                                                                            \
    }                                                                                \
    static void down_##SUF(iheap* h, const KT* key, int64_t i) {                     \
        for (;;) {                                                                   \
            int64_t l = 2 * i + 1, r = l + 1, m = i;                                 \
            if (l < h->n && key[h->heap[l]] < key[h->heap[m]]) m = l;                \
            if (r < h->n && key[h->heap[r]] < key[h->heap[m]]) m = r;                \
            if (m == i) break;                                                       \
            iheap_swap(h, i, m);                                                     \
            i = m;                                                                   \
        }                                                                            \
    }                                                                                \
    static void push_or_decrease_##SUF(iheap* h, const KT* key, int64_t v) {         \
        if (h->pos[v] < 0) {                                                         \
            h->heap[h->n] = v;                                                       \
            h->pos[v] = h->n;                                                        \
            h->n++;                                                                  \
        }                                                                            \
        up_##SUF(h, key, h->pos[v]);                                                 \
    }                                                                                \
    static int64_t pop_##SUF(iheap* h, const KT* key) {                              \
        int64_t v = h->heap[0];                                                      \
        iheap_swap(h, 0, h->n - 1);                                                  \
        h->n--;                                                                      \
        h->pos[v] = -1;                                                              \
        if (h->n > 0) down_##SUF(h, key, 0);                                         \
        return v;                                                                    \
    }

DEFINE_HEAP_OPS(u64, uint64_t)
DEFINE_HEAP_OPS(f32, float)

/* ------------------------------------------------------------ Dijkstra --- */
int oracle_dijkstra_u32(int64_t V, const int64_t* row, const uint32_t* col, const uint32_t* w,
                        int64_t src, uint32_t* dist) {
    if (V <= 0 || src < 0 || src >= V) return ORACLE_ERR_ARG;
    uint64_t* d = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)V);
    iheap h;
    if (!d || iheap_init(&h, V)) return ORACLE_ERR_ARG;
    for (int64_t v = 0; v < V; ++v) d[v] = UINT64_MAX;
    int rc = ORACLE_OK;
    d[src] = 0;
    push_or_decrease_u64(&h, d, src);
    while (h.n > 0) {
        int64_t u = pop_u64(&h, d); /* greedy: nearest active vertex */
        for (int64_t e = row[u]; e < row[u + 1]; ++e) {
            int64_t v = col[e];
            uint64_t nd = d[u] + (uint64_t)w[e]; /* Alg. 1 line 1 */
            if (nd < d[v]) {                      /* Alg. 1 line 2 */
                d[v] = nd;                        /* Alg. 1 line 3 */
                push_or_decrease_u64(&h, d, v);
            }
        }
    }
    for (int64_t v = 0; v < V; ++v) {
        if (d[v] == UINT64_MAX) {
            dist[v] = INF_U32;
        } else if (d[v] >= (uint64_t)INF_U32) {
            dist[v] = INF_U32;
            rc = ORACLE_ERR_OVERFLOW;
        } else {
            dist[v] = (uint32_t)d[v];
        }
    }
    iheap_free(&h);
    free(d);
    return rc;
}

int oracle_dijkstra_f32(int64_t V, const int64_t* row, const uint32_t* col, const float* w,
                        int64_t src, float* dist) {
    if (V <= 0 || src < 0 || src >= V) return ORACLE_ERR_ARG;
    iheap h;
    if (iheap_init(&h, V)) return ORACLE_ERR_ARG;
    for (int64_t v = 0; v < V; ++v) dist[v] = INFINITY;
    dist[src] = 0.0f;
    push_or_decrease_f32(&h, dist, src);
    while (h.n > 0) {
        int64_t u = pop_f32(&h, dist);
        for (int64_t e = row[u]; e < row[u + 1]; ++e) {
            int64_t v = col[e];
            volatile float nd = dist[u] + w[e]; /* one binary32 RN add, Alg. 1 line 1 */
            if (nd < dist[v]) {
                dist[v] = nd;
                push_or_decrease_f32(&h, dist, v);
            }
        }
    }
    iheap_free(&h);
    return ORACLE_OK;
}

/* -------------------------------------------------------- Bellman-Ford --- */
int64_t oracle_bellman_ford_u32(int64_t V, const int64_t* row, const uint32_t* col,
                                const uint32_t* w, int64_t src, uint32_t* dist) {
    uint64_t* d = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)V);
    for (int64_t v = 0; v < V; ++v) d[v] = UINT64_MAX;
    d[src] = 0;
    int64_t rounds = 0;
    for (int changed = 1; changed && rounds <= V; ++rounds) {
        changed = 0;
        for (int64_t u = 0; u < V; ++u) {
            if (d[u] == UINT64_MAX) continue;
            for (int64_t e = row[u]; e < row[u + 1]; ++e) {
                uint64_t nd = d[u] + w[e];
                if (nd < d[col[e]]) {
                    d[col[e]] = nd;
                    changed = 1;
                }
            }
        }
    }
    int64_t rc = rounds;
    for (int64_t v = 0; v < V; ++v) {
        if (d[v] != UINT64_MAX && d[v] >= INF_U32) rc = -1;
        dist[v] = d[v] >= INF_U32 ? INF_U32 : (uint32_t)d[v];
    }
    free(d);
    return rc;
}

int64_t oracle_bellman_ford_f32(int64_t V, const int64_t* row, const uint32_t* col,
                                const float* w, int64_t src, float* dist) {
    for (int64_t v = 0; v < V; ++v) dist[v] = INFINITY;
    dist[src] = 0.0f;
    int64_t rounds = 0;
    for (int changed = 1; changed && rounds <= V; ++rounds) {
        changed = 0;
        for (int64_t u = 0; u < V; ++u) {
            if (isinf(dist[u])) continue;
            for (int64_t e = row[u]; e < row[u + 1]; ++e) {
                volatile float nd = dist[u] + w[e];
                if (nd < dist[col[e]]) {
                    dist[col[e]] = nd;
                    changed = 1;
                }
            }
        }
    }
    return rounds;
}

/* ------------------------------------------------------ Floyd-Warshall --- */
int oracle_floyd_warshall_u32(int64_t V, const int64_t* row, const uint32_t* col,
                              const uint32_t* w, uint64_t* D) {
    if (V <= 0 || V > 4096) return ORACLE_ERR_ARG;
    for (int64_t i = 0; i < V * V; ++i) D[i] = UINT64_MAX;
    for (int64_t i = 0; i < V; ++i) D[i * V + i] = 0;
    for (int64_t u = 0; u < V; ++u)
        for (int64_t e = row[u]; e < row[u + 1]; ++e)
            if (w[e] < D[u * V + col[e]]) D[u * V + col[e]] = w[e];
    for (int64_t k = 0; k < V; ++k)
        for (int64_t i = 0; i < V; ++i) {
            if (D[i * V + k] == UINT64_MAX) continue;
            for (int64_t j = 0; j < V; ++j) {
                if (D[k * V + j] == UINT64_MAX) continue;
                uint64_t s = D[i * V + k] + D[k * V + j];
                if (s < D[i * V + j]) D[i * V + j] = s;
            }
        }
    return ORACLE_OK;
}

/* --------------------------------------------------------- certificate --- */
int64_t oracle_certificate_u32(int64_t V, const int64_t* row, const uint32_t* col,
                               const uint32_t* w, int64_t src, const uint32_t* dist) {
    if (dist[src] != 0) return V;
    unsigned char* tight = (unsigned char*)calloc((size_t)V, 1);
    int64_t bad = -1;
    for (int64_t u = 0; u < V && bad < 0; ++u) {
        if (dist[u] == INF_U32) continue;
        for (int64_t e = row[u]; e < row[u + 1]; ++e) {
            int64_t v = col[e];
            uint64_t s = (uint64_t)dist[u] + w[e];
            uint64_t dv = dist[v] == INF_U32 ? UINT64_MAX : dist[v];
            if (dv > s) { /* d[v] <= d[u] + w violated */
                bad = v;
                break;
            }
            if (dv == s && dist[u] < dist[v]) tight[v] = 1;
        }
    }
    for (int64_t v = 0; v < V && bad < 0; ++v)
        if (v != src && dist[v] != INF_U32 && !tight[v]) bad = v;
    free(tight);
    return bad;
}

/* --------------------------------------------- property-driven reorder --- */
static const int64_t* g_deg; /* qsort context (single-threaded oracle) */
static int cmp_degree_desc(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    if (g_deg[x] != g_deg[y]) return g_deg[x] > g_deg[y] ? -1 : 1; /* descending degree */
    return x < y ? -1 : (x > y);                                     /* then original id */
}
static int cmp_pair(const void* a, const void* b) {
    const uint32_t* x = (const uint32_t*)a; /* {weight bits, new dst} */
    const uint32_t* y = (const uint32_t*)b;
    if (x[0] != y[0]) return x[0] < y[0] ? -1 : 1; /* ascending weight */
    return x[1] < y[1] ? -1 : (x[1] > y[1]);       /* then ascending new id */
}

int oracle_pro_reorder(int64_t V, const int64_t* row, const uint32_t* col, const uint32_t* wbits,
                       uint32_t* new2old, uint32_t* old2new, int64_t* new_row, uint32_t* adj,
                       uint32_t* val) {
    int64_t* deg = (int64_t*)malloc(sizeof(int64_t) * (size_t)V);
    for (int64_t v = 0; v < V; ++v) {
        deg[v] = row[v + 1] - row[v]; /* degree = arcs out of v */
        new2old[v] = (uint32_t)v;
    }
    g_deg = deg;
    qsort(new2old, (size_t)V, sizeof(uint32_t), cmp_degree_desc);
    for (int64_t i = 0; i < V; ++i) old2new[new2old[i]] = (uint32_t)i;
    new_row[0] = 0;
    for (int64_t i = 0; i < V; ++i) new_row[i + 1] = new_row[i] + deg[new2old[i]];
    int64_t maxd = 0;
    for (int64_t v = 0; v < V; ++v)
        if (deg[v] > maxd) maxd = deg[v];
    uint32_t* pairs = (uint32_t*)malloc(sizeof(uint32_t) * 2 * (size_t)(maxd > 0 ? maxd : 1));
    for (int64_t i = 0; i < V; ++i) {
        int64_t o = new2old[i], n = deg[o];
        for (int64_t k = 0; k < n; ++k) {
            pairs[2 * k] = wbits[row[o] + k];
            pairs[2 * k + 1] = old2new[col[row[o] + k]];
        }
        qsort(pairs, (size_t)n, 2 * sizeof(uint32_t), cmp_pair);
        for (int64_t k = 0; k < n; ++k) {
            val[new_row[i] + k] = pairs[2 * k];
            adj[new_row[i] + k] = pairs[2 * k + 1];
        }
    }
    free(pairs);
    free(deg);
    return ORACLE_OK;
}

static int is_light(uint32_t wb, int wtype, double delta) {
    if (wtype == 0) {
        double dc = ceil(delta);
        return (double)wb < dc; /* light iff w < Delta */
    } else {
        float wf, df = (float)delta;
        memcpy(&wf, &wb, 4);
        return wf < df;
    }
}

void oracle_pro_rowlist(int64_t V, const int64_t* new_row, const uint32_t* val, int wtype,
                        double delta, int64_t* rowlist) {
    for (int64_t i = 0; i < V; ++i) {
        int64_t h = new_row[i];
        while (h < new_row[i + 1] && is_light(val[h], wtype, delta)) ++h;
        rowlist[2 * i] = new_row[i];
        rowlist[2 * i + 1] = h;
    }
    rowlist[2 * V] = new_row[V];
}

/* ------------------------------------------------------------- buckets --- */
int64_t oracle_bucket_histogram(int64_t V, const uint32_t* dist_bits, int wtype, double delta,
                                int64_t* counts, int64_t nb) {
    int64_t maxb = -1;
    for (int64_t i = 0; i < nb; ++i) counts[i] = 0;
    uint32_t dint = (uint32_t)ceil(delta);
    float df = (float)delta;
    volatile float inv = (float)(1.0 / (double)df);
    for (int64_t v = 0; v < V; ++v) {
        int64_t b;
        if (wtype == 0) {
            if (dist_bits[v] == INF_U32) continue;
            b = dist_bits[v] / dint;
        } else {
            float d;
            memcpy(&d, &dist_bits[v], 4);
            if (isinf(d)) continue;
            volatile float p = d * inv;
            b = (int64_t)(uint32_t)p;
        }
        if (b > maxb) maxb = b;
        if (b < nb) counts[b]++;
    }
    return maxb + 1;
}
