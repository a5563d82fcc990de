/*
 * gen.c — seeded synthetic graph generators + CSR builder (input construction only).
 *
 * This module is shared by the oracle side and the CUDA side *as input construction*.
 * It holds none of the method's arithmetic (no traversal, no relaxation, no labels,
 * no bitmap frontier): it draws random endpoints, drops self-loops, canonicalises,
 * sorts, de-duplicates and mirrors edges into a symmetric CSR with ascending rows
 * (SURVEY.md §8(d) "Synthetic inputs", readings C8, C9,
 * C11, C15, C17).
 *
 * RNG (counter based, order independent, so generation is multithreaded and bit
 * reproducible):  mix = splitmix64 finaliser,
 *     rnd(seed, stream, i) = mix(mix(seed ^ (stream << 56)) + i),
 *     unif = (rnd >> 11) * 2^-53.
 * Streams: 0 RMAT quadrants, 1 G(n,m) endpoints, 2 lattice edge keep, 3 weights,
 *          4 Fisher-Yates permutation, 5/6 source lists.
 *
 * Two-phase API: a builder returns a handle holding the sorted, unique arc keys;
 * the caller allocates row_ptr[n+1] / col_idx[nnz] (numpy or pinned torch memory)
 * and calls sgg_fill().  All functions are plain C, no exceptions.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

#define SGG_EXPORT __attribute__((visibility("default")))

static inline uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
static inline uint64_t stream_base(uint64_t seed, uint64_t stream) { return mix64(seed ^ (stream << 56)); }
static inline uint64_t rnd_b(uint64_t base, uint64_t i) { return mix64(base + i); }
static inline double unif_b(uint64_t base, uint64_t i) { return (double)(rnd_b(base, i) >> 11) * 0x1.0p-53; }

SGG_EXPORT uint64_t sgg_rnd(uint64_t seed, uint64_t stream, uint64_t i) { return rnd_b(stream_base(seed, stream), i); }

typedef struct sgg_graph {
    int64_t n;
    int shift;          /* key = (u << shift) | v */
    int64_t nkeys;      /* number of unique arcs (= nnz) */
    uint64_t *keys;     /* sorted unique arc keys (NULL for direct builders) */
    int64_t *row_ptr;   /* direct builders (lattice) fill these immediately */
    int32_t *col_idx;
} sgg_graph;

static int bits_for(int64_t n) {
    int b = 1;
    while (((int64_t)1 << b) < n) b++;
    return b;
}

/* ---- parallel LSD radix sort on u64 keys (stable, deterministic) ---- */
#define RADIX_BITS 11
#define RADIX_SIZE (1 << RADIX_BITS)
static void radix_sort_u64(uint64_t **pa, uint64_t **ptmp, int64_t N, int key_bits) {
    uint64_t *a = *pa, *t = *ptmp;
    int passes = (key_bits + RADIX_BITS - 1) / RADIX_BITS;
    int nt = omp_get_max_threads();
    int64_t *hist = (int64_t *)calloc((size_t)nt * RADIX_SIZE, sizeof(int64_t));
    for (int p = 0; p < passes; p++) {
        int sh = p * RADIX_BITS;
        memset(hist, 0, sizeof(int64_t) * (size_t)nt * RADIX_SIZE);
#pragma omp parallel num_threads(nt)
        {
            int tid = omp_get_thread_num();
            int64_t lo = N * tid / nt, hi = N * (tid + 1) / nt;
            int64_t *h = hist + (size_t)tid * RADIX_SIZE;
            for (int64_t i = lo; i < hi; i++) h[(a[i] >> sh) & (RADIX_SIZE - 1)]++;
#pragma omp barrier
#pragma omp single
            {
                int64_t s = 0;
                for (int d = 0; d < RADIX_SIZE; d++)
                    for (int q = 0; q < nt; q++) {
                        int64_t c = hist[(size_t)q * RADIX_SIZE + d];
                        hist[(size_t)q * RADIX_SIZE + d] = s;
                        s += c;
                    }
            }
            for (int64_t i = lo; i < hi; i++) {
                uint64_t k = a[i];
                t[h[(k >> sh) & (RADIX_SIZE - 1)]++] = k;
            }
        }
        uint64_t *x = a; a = t; t = x;
    }
    free(hist);
    *pa = a; *ptmp = t;
}

/* sort + unique the keys; invalid keys are UINT64_MAX and sort to the end */
static sgg_graph *finish_keys(int64_t n, uint64_t *keys, int64_t N, int shift) {
    uint64_t *tmp = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(N > 0 ? N : 1));
    if (!tmp) { free(keys); return NULL; }
    /* UINT64_MAX sentinels need all 64 bits to sort last: map them to (1<<2*shift) */
    uint64_t sentinel = (uint64_t)1 << (2 * shift);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; i++) if (keys[i] == UINT64_MAX) keys[i] = sentinel;
    radix_sort_u64(&keys, &tmp, N, 2 * shift + 1);
    free(tmp);
    /* parallel unique (compaction) */
    int nt = omp_get_max_threads();
    int64_t *cnt = (int64_t *)calloc((size_t)nt + 1, sizeof(int64_t));
#pragma omp parallel num_threads(nt)
    {
        int tid = omp_get_thread_num();
        int64_t lo = N * tid / nt, hi = N * (tid + 1) / nt, c = 0;
        for (int64_t i = lo; i < hi; i++)
            if (keys[i] != sentinel && (i == 0 || keys[i] != keys[i - 1])) c++;
        cnt[tid + 1] = c;
#pragma omp barrier
#pragma omp single
        for (int q = 0; q < nt; q++) cnt[q + 1] += cnt[q];
        int64_t pos = cnt[tid];
        /* in-place compaction is unsafe across threads: write into a fresh array */
#pragma omp barrier
#pragma omp single
        {
            uint64_t *out = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(cnt[nt] > 0 ? cnt[nt] : 1));
            tmp = out;
        }
        for (int64_t i = lo; i < hi; i++)
            if (keys[i] != sentinel && (i == 0 || keys[i] != keys[i - 1])) tmp[pos++] = keys[i];
    }
    int64_t total = cnt[nt];
    free(cnt);
    free(keys);
    sgg_graph *g = (sgg_graph *)calloc(1, sizeof(sgg_graph));
    g->n = n; g->shift = shift; g->nkeys = total; g->keys = tmp;
    return g;
}

static inline uint64_t arc_key(int64_t u, int64_t v, int shift) { return ((uint64_t)u << shift) | (uint64_t)v; }

/* Fisher-Yates permutation of [0,n), stream 4 (sequential by definition). */
static int32_t *make_perm(int64_t n, uint64_t seed) {
    int32_t *p = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    for (int64_t i = 0; i < n; i++) p[i] = (int32_t)i;
    uint64_t b = stream_base(seed, 4);
    for (int64_t i = n - 1; i > 0; i--) {
        int64_t j = (int64_t)(rnd_b(b, (uint64_t)i) % (uint64_t)(i + 1));
        int32_t x = p[i]; p[i] = p[j]; p[j] = x;
    }
    return p;
}

/* R-MAT / Kronecker (Graph500 A,B,C,D; no noise), edge_factor counts generated
 * undirected edges (reading C17).  Quadrant for edge i, level l from unif(stream 0,
 * i*scale + l); bit l of (u, v).  Optional seeded vertex permutation (stream 4). */
SGG_EXPORT sgg_graph *sgg_rmat(int scale, int64_t edge_factor, double A, double B, double C,
                               uint64_t seed, int permute) {
    int64_t n = (int64_t)1 << scale;
    int64_t m = n * edge_factor;
    int shift = bits_for(n);
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(2 * m));
    if (!keys) return NULL;
    int32_t *perm = permute ? make_perm(n, seed) : NULL;
    uint64_t b = stream_base(seed, 0);
    double ab = A + B, abc = A + B + C;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; i++) {
        int64_t u = 0, v = 0;
        uint64_t base_i = (uint64_t)i * (uint64_t)scale;
        for (int l = 0; l < scale; l++) {
            double r = unif_b(b, base_i + (uint64_t)l);
            int bu, bv;
            if (r < A) { bu = 0; bv = 0; }
            else if (r < ab) { bu = 0; bv = 1; }
            else if (r < abc) { bu = 1; bv = 0; }
            else { bu = 1; bv = 1; }
            u |= (int64_t)bu << l;
            v |= (int64_t)bv << l;
        }
        if (perm) { u = perm[u]; v = perm[v]; }
        if (u == v) { keys[2 * i] = UINT64_MAX; keys[2 * i + 1] = UINT64_MAX; }
        else { keys[2 * i] = arc_key(u, v, shift); keys[2 * i + 1] = arc_key(v, u, shift); }
    }
    free(perm);
    return finish_keys(n, keys, 2 * m, shift);
}

/* Uniform G(n, m): endpoints rnd(stream 1, 2i) mod n, rnd(stream 1, 2i+1) mod n. */
SGG_EXPORT sgg_graph *sgg_gnm(int64_t n, int64_t m, uint64_t seed) {
    int shift = bits_for(n);
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(2 * m > 0 ? 2 * m : 1));
    if (!keys) return NULL;
    uint64_t b = stream_base(seed, 1);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; i++) {
        int64_t u = (int64_t)(rnd_b(b, 2 * (uint64_t)i) % (uint64_t)n);
        int64_t v = (int64_t)(rnd_b(b, 2 * (uint64_t)i + 1) % (uint64_t)n);
        if (u == v) { keys[2 * i] = UINT64_MAX; keys[2 * i + 1] = UINT64_MAX; }
        else { keys[2 * i] = arc_key(u, v, shift); keys[2 * i + 1] = arc_key(v, u, shift); }
    }
    return finish_keys(n, keys, 2 * m, shift);
}

/* Arbitrary undirected edge list (closed-form families, hand-made cases). */
SGG_EXPORT sgg_graph *sgg_from_edges(int64_t n, int64_t m, const int64_t *eu, const int64_t *ev) {
    int shift = bits_for(n);
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(2 * m > 0 ? 2 * m : 1));
    if (!keys) return NULL;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; i++) {
        int64_t u = eu[i], v = ev[i];
        if (u == v || u < 0 || v < 0 || u >= n || v >= n) { keys[2 * i] = UINT64_MAX; keys[2 * i + 1] = UINT64_MAX; }
        else { keys[2 * i] = arc_key(u, v, shift); keys[2 * i + 1] = arc_key(v, u, shift); }
    }
    return finish_keys(n, keys, 2 * m, shift);
}

/* Bond-percolated R x C lattice, row-major ids; edge kept iff unif(stream 2, id) < p.
 * Horizontal (r,c)-(r,c+1): id r(C-1)+c; vertical (r,c)-(r+1,c): id R(C-1)+rC+c.
 * Built directly: neighbours up, left, right, down are already ascending. */
static inline int keep_h(uint64_t b, int64_t R, int64_t C, int64_t r, int64_t c, double p) {
    (void)R; return unif_b(b, (uint64_t)(r * (C - 1) + c)) < p;
}
static inline int keep_v(uint64_t b, int64_t R, int64_t C, int64_t r, int64_t c, double p) {
    return unif_b(b, (uint64_t)(R * (C - 1) + r * C + c)) < p;
}
SGG_EXPORT sgg_graph *sgg_lattice(int64_t R, int64_t C, double p, uint64_t seed) {
    int64_t n = R * C;
    uint64_t b = stream_base(seed, 2);
    sgg_graph *g = (sgg_graph *)calloc(1, sizeof(sgg_graph));
    g->n = n; g->shift = bits_for(n);
    g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    int64_t *rp = g->row_ptr;
    rp[0] = 0;
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; v++) {
        int64_t r = v / C, c = v % C; int d = 0;
        if (r > 0 && keep_v(b, R, C, r - 1, c, p)) d++;
        if (c > 0 && keep_h(b, R, C, r, c - 1, p)) d++;
        if (c + 1 < C && keep_h(b, R, C, r, c, p)) d++;
        if (r + 1 < R && keep_v(b, R, C, r, c, p)) d++;
        rp[v + 1] = d;
    }
    for (int64_t v = 0; v < n; v++) rp[v + 1] += rp[v];
    g->nkeys = rp[n];
    g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(g->nkeys > 0 ? g->nkeys : 1));
    int32_t *ci = g->col_idx;
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; v++) {
        int64_t r = v / C, c = v % C, o = rp[v];
        if (r > 0 && keep_v(b, R, C, r - 1, c, p)) ci[o++] = (int32_t)(v - C);
        if (c > 0 && keep_h(b, R, C, r, c - 1, p)) ci[o++] = (int32_t)(v - 1);
        if (c + 1 < C && keep_h(b, R, C, r, c, p)) ci[o++] = (int32_t)(v + 1);
        if (r + 1 < R && keep_v(b, R, C, r, c, p)) ci[o++] = (int32_t)(v + C);
    }
    return g;
}

SGG_EXPORT int64_t sgg_n(const sgg_graph *g) { return g ? g->n : -1; }
SGG_EXPORT int64_t sgg_nnz(const sgg_graph *g) { return g ? g->nkeys : -1; }

/* Write row_ptr[n+1] and col_idx[nnz] into caller memory. */
SGG_EXPORT int sgg_fill(const sgg_graph *g, int64_t *row_ptr, int32_t *col_idx) {
    if (!g) return -1;
    int64_t n = g->n, N = g->nkeys;
    if (!g->keys) {
        memcpy(row_ptr, g->row_ptr, sizeof(int64_t) * (size_t)(n + 1));
        memcpy(col_idx, g->col_idx, sizeof(int32_t) * (size_t)N);
        return 0;
    }
    int shift = g->shift;
    uint64_t mask = ((uint64_t)1 << shift) - 1;
    const uint64_t *k = g->keys;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; i++) col_idx[i] = (int32_t)(k[i] & mask);
    /* row_ptr: for each row boundary in the sorted keys */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i <= N; i++) {
        int64_t cur = (i < N) ? (int64_t)(k[i] >> shift) : n;
        int64_t prev = (i > 0) ? (int64_t)(k[i - 1] >> shift) : -1;
        for (int64_t r = prev + 1; r <= cur; r++) row_ptr[r] = i;
    }
    return 0;
}

SGG_EXPORT void sgg_free(sgg_graph *g) {
    if (!g) return;
    free(g->keys); free(g->row_ptr); free(g->col_idx); free(g);
}

/* Symmetric integer weights (reading C11): w(u,v) = 1 + rnd(stream 3, min*n+max) mod wmax. */
SGG_EXPORT void sgg_weights(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, uint64_t seed,
                            uint32_t wmax, uint8_t *w_out) {
    uint64_t b = stream_base(seed, 3);
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < n; u++)
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int64_t v = col_idx[e];
            int64_t lo = u < v ? u : v, hi = u < v ? v : u;
            w_out[e] = (uint8_t)(1 + rnd_b(b, (uint64_t)(lo * n + hi)) % wmax);
        }
}

/* First k distinct vertices rnd(stream, i) mod n with degree > 0 (reading C15) and, when
 * `eligible` is non-NULL, eligible[v] != 0 (config 5: the largest component, computed by the
 * caller with a library routine).  Returns the number found (< k only if fewer exist). */
SGG_EXPORT int64_t sgg_sources(int64_t n, const int64_t *row_ptr, uint64_t seed, uint64_t stream,
                               int64_t k, int32_t *out, const uint8_t *eligible) {
    uint64_t b = stream_base(seed, stream);
    int64_t found = 0;
    for (uint64_t i = 0; found < k && i < (uint64_t)(64 * n + 1024); i++) {
        int64_t v = (int64_t)(rnd_b(b, i) % (uint64_t)n);
        if (row_ptr[v + 1] == row_ptr[v]) continue;
        if (eligible && !eligible[v]) continue;
        int dup = 0;
        for (int64_t j = 0; j < found; j++) if (out[j] == v) { dup = 1; break; }
        if (!dup) out[found++] = (int32_t)v;
    }
    return found;
}
