/*
 * oracle.c — the parity oracle.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this library.  The product path (paper_conf_icpp_carocc25_b200) never
 * imports, links or calls it, and it shares no code, header, table or helper with the
 * CUDA path.  Plain single-threaded C: textbook sequential algorithms that reach the
 * plain definitions the method (SYgraph, ICPP'25) computes, written for readability
 * rather than speed (DESIGN.md §3 "Oracle").
 *
 *   oracle_bfs   queue BFS            — hop levels      (PAPER.md:163-189 Listing 1; :161 §3.4)
 *   oracle_sssp  binary-heap Dijkstra — shortest dist   (§3.4: Bellman-Ford fixed point)
 *   oracle_cc    union-find           — min-id labels   (§3.4: label propagation fixed point)
 *   oracle_bc    Brandes, long double — pair dependency (§3.4 "Brandes' formulation"; ref [9])
 *
 * Graph input: symmetric CSR, row_ptr int64[n+1], col_idx int32[nnz]; weights uint8[nnz].
 * Unreached vertices: UINT32_MAX (reading C6).  Labels: component minimum id.
 * BC: sum over the given sources of delta_s(v), unnormalised, ordered pairs, no halving,
 * delta_s(s) excluded (reading C14).
 *
 * Every function is pinned by CPU tests (tests/test_oracle_*.py) against brute force,
 * closed forms and invariants that do not use this file.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define OR_EXPORT __attribute__((visibility("default")))
#define INF32 0xFFFFFFFFu

/* ------------------------------------------------------------------ BFS ---- */
/* Queue BFS (Listing 1 semantics: level[src] = 0, neighbours of level-d vertices that are
 * unvisited get d+1).  Returns the number of reached vertices. */
OR_EXPORT int64_t oracle_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                             int32_t src, uint32_t *level) {
    for (int64_t v = 0; v < n; v++) level[v] = INF32;
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int64_t head = 0, tail = 0;
    level[src] = 0;
    queue[tail++] = src;
    while (head < tail) {
        int32_t u = queue[head++];
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int32_t v = col_idx[e];
            if (level[v] == INF32) {
                level[v] = level[u] + 1;
                queue[tail++] = v;
            }
        }
    }
    free(queue);
    return tail;
}

/* ----------------------------------------------------------------- SSSP ---- */
/* Dijkstra with a binary min-heap of (dist, vertex) and lazy deletion; distances
 * accumulate in uint64 and are stored as uint32 (INF32 = unreachable). */
typedef struct { uint64_t d; int32_t v; } heap_item;

static void heap_push(heap_item *h, int64_t *size, heap_item x) {
    int64_t i = (*size)++;
    h[i] = x;
    while (i > 0) {
        int64_t p = (i - 1) / 2;
        if (h[p].d <= h[i].d) break;
        heap_item t = h[p]; h[p] = h[i]; h[i] = t;
        i = p;
    }
}

static heap_item heap_pop(heap_item *h, int64_t *size) {
    heap_item top = h[0];
    h[0] = h[--(*size)];
    int64_t i = 0;
    for (;;) {
        int64_t l = 2 * i + 1, r = l + 1, m = i;
        if (l < *size && h[l].d < h[m].d) m = l;
        if (r < *size && h[r].d < h[m].d) m = r;
        if (m == i) break;
        heap_item t = h[m]; h[m] = h[i]; h[i] = t;
        i = m;
    }
    return top;
}

OR_EXPORT int64_t oracle_sssp(int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                              const uint8_t *weight, int32_t src, uint32_t *dist_out) {
    uint64_t *dist = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n > 0 ? n : 1));
    for (int64_t v = 0; v < n; v++) dist[v] = UINT64_MAX;
    /* each improvement pushes once: at most nnz + 1 entries */
    int64_t cap = row_ptr[n] + 1;
    heap_item *heap = (heap_item *)malloc(sizeof(heap_item) * (size_t)cap);
    int64_t size = 0, reached = 0;
    dist[src] = 0;
    heap_push(heap, &size, (heap_item){0, src});
    while (size > 0) {
        heap_item it = heap_pop(heap, &size);
        if (it.d > dist[it.v]) continue;          /* stale entry */
        reached++;
        int32_t u = it.v;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int32_t v = col_idx[e];
            uint64_t nd = it.d + (uint64_t)weight[e];
            if (nd < dist[v]) {
                dist[v] = nd;
                heap_push(heap, &size, (heap_item){nd, v});
            }
        }
    }
    for (int64_t v = 0; v < n; v++) dist_out[v] = dist[v] == UINT64_MAX ? INF32 : (uint32_t)dist[v];
    free(heap);
    free(dist);
    return reached;
}

/* ------------------------------------------------------------------- CC ---- */
/* Union-find with path halving; the larger root is linked under the smaller, so every
 * root is its component's minimum id and label[v] = find(v) is min-canonical. */
static int32_t uf_find(int32_t *parent, int32_t x) {
    while (parent[x] != x) {
        parent[x] = parent[parent[x]];
        x = parent[x];
    }
    return x;
}

OR_EXPORT int64_t oracle_cc(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int32_t *label) {
    for (int64_t v = 0; v < n; v++) label[v] = (int32_t)v;
    for (int64_t u = 0; u < n; u++)
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int32_t v = col_idx[e];
            if (u >= v) continue;                 /* each undirected edge once */
            int32_t ru = uf_find(label, (int32_t)u), rv = uf_find(label, v);
            if (ru == rv) continue;
            if (ru < rv) label[rv] = ru; else label[ru] = rv;
        }
    int64_t ncomp = 0;
    for (int64_t v = 0; v < n; v++) {
        label[v] = uf_find(label, (int32_t)v);
        if (label[v] == v) ncomp++;
    }
    return ncomp;
}

/* ------------------------------------------------------------------- BC ---- */
/* One Brandes source: BFS recording the visit order S, levels and path counts sigma
 * (long double, 15-bit exponent: no scaling needed, reading C20); then in
 * reverse visit order, delta[v] += sigma[v]/sigma[w] * (1 + delta[w]) for each
 * predecessor v of w (level[v] == level[w] - 1). */
static void brandes_one(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int32_t s,
                        uint32_t *level, long double *sigma, long double *delta, int32_t *order,
                        int64_t *nreached) {
    for (int64_t v = 0; v < n; v++) { level[v] = INF32; sigma[v] = 0.0L; delta[v] = 0.0L; }
    int64_t head = 0, tail = 0;
    level[s] = 0; sigma[s] = 1.0L; order[tail++] = s;
    while (head < tail) {
        int32_t v = order[head++];
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; e++) {
            int32_t w = col_idx[e];
            if (level[w] == INF32) { level[w] = level[v] + 1; order[tail++] = w; }
            if (level[w] == level[v] + 1) sigma[w] += sigma[v];
        }
    }
    for (int64_t i = tail - 1; i >= 0; i--) {
        int32_t w = order[i];
        for (int64_t e = row_ptr[w]; e < row_ptr[w + 1]; e++) {
            int32_t v = col_idx[e];
            if (level[v] != INF32 && level[v] + 1 == level[w])
                delta[v] += sigma[v] / sigma[w] * (1.0L + delta[w]);
        }
    }
    *nreached = tail;
}

/* bc[v] = sum over sources s (duplicates counted again) of delta_s(v), v != s. */
OR_EXPORT int oracle_bc(int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                        const int32_t *sources, int64_t k, double *bc_out) {
    uint32_t *level = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)n);
    long double *sigma = (long double *)malloc(sizeof(long double) * (size_t)n);
    long double *delta = (long double *)malloc(sizeof(long double) * (size_t)n);
    long double *bc = (long double *)calloc((size_t)n, sizeof(long double));
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    if (!level || !sigma || !delta || !bc || !order) return -1;
    for (int64_t i = 0; i < k; i++) {
        int32_t s = sources[i];
        int64_t reached;
        brandes_one(n, row_ptr, col_idx, s, level, sigma, delta, order, &reached);
        for (int64_t j = 0; j < reached; j++) {
            int32_t w = order[j];
            if (w != s) bc[w] += delta[w];
        }
    }
    for (int64_t v = 0; v < n; v++) bc_out[v] = (double)bc[v];
    free(level); free(sigma); free(delta); free(bc); free(order);
    return 0;
}

/* Single-source forward/backward state for pins: level, sigma (as double, and as log2 for
 * sigma beyond the double range) and delta.  Returns the number of reached vertices. */
OR_EXPORT int oracle_bc_single(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int32_t s,
                               uint32_t *level, double *sigma_out, double *log2_sigma_out, double *delta_out) {
    long double *sigma = (long double *)malloc(sizeof(long double) * (size_t)n);
    long double *delta = (long double *)malloc(sizeof(long double) * (size_t)n);
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    if (!sigma || !delta || !order) return -1;
    int64_t reached;
    brandes_one(n, row_ptr, col_idx, s, level, sigma, delta, order, &reached);
    for (int64_t v = 0; v < n; v++) {
        sigma_out[v] = (double)sigma[v];
        if (log2_sigma_out) log2_sigma_out[v] = sigma[v] > 0.0L ? (double)log2l(sigma[v]) : -1.0;
        delta_out[v] = (double)delta[v];
    }
    free(sigma); free(delta); free(order);
    return (int)reached;
}
