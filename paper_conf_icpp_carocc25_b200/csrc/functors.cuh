// functors.cuh — per-edge advance functors (Table 2: Functor(src, dst, edge,
// weight) -> bool "whether dst should be added to the frontier"; algorithms P:161 §3.4).
//
// Split into ctx(src) (loaded once per source vertex), probe(dst) (the one random load per
// arc; issued for several arcs before any decision so the loads overlap) and act_batch<K>(...)
// (decision + atomics + insertion into the output 2LB for K arcs at once: every atomic of the
// batch is issued before any result is consumed, so a thread has K atomics in flight instead
// of K round trips in series).  The compute step of Listing 1 (dist[v] = iter + 1,
// P:178-181) is fused: the thread whose atomic inserts v writes its value (the paper keeps it
// separate; on B200 the fused store saves a pass).
#pragma once
#include "common.cuh"

namespace sg {

struct OutSink {
    uint64_t *bits;   // nullptr: advance without an output frontier
    uint64_t *summ;
    __device__ __forceinline__ bool insert(int32_t v) const { return bits ? insert_2lb(bits, summ, v) : true; }
};

// Insert the flagged vertices into the output 2LB: all layer-1 atomics first, then the summary
// bits of words that were empty.  flipped[k] = this call set v[k]'s bit.
template <int K>
__device__ __forceinline__ void insert_batch(const OutSink &out, const int32_t (&v)[K], const bool (&f)[K],
                                             bool (&flipped)[K]) {
    if (!out.bits) {
#pragma unroll
        for (int k = 0; k < K; k++) flipped[k] = f[k];
        return;
    }
    unsigned long long old[K];
#pragma unroll
    for (int k = 0; k < K; k++) old[k] = f[k] ? atomic_or_u64(out.bits + (v[k] >> 6), 1ull << (v[k] & 63)) : ~0ull;
#pragma unroll
    for (int k = 0; k < K; k++) {
        flipped[k] = f[k] && !((old[k] >> (v[k] & 63)) & 1ull);
        if (f[k] && old[k] == 0ull) atomic_or_u64(out.summ + (v[k] >> 12), 1ull << ((v[k] >> 6) & 63));
    }
}

// BFS (Listing 1 l.9-13 + l.14-17).  `visited` is updated live: the first thread whose
// atomicOr sets v's visited bit owns v, writes level[v] and inserts v.  A stale probe only
// costs one extra atomic.  Result = {v unvisited before the step with a neighbour in the
// frontier}, identical to the frozen-visited reading (R1).
// diff mode (run_bfs): the arc only ORs v's visited bit, a fire-and-forget RED with no result
// to wait for; k_bfs_diff then derives the output frontier, level[] and the frontier
// statistics from visited & ~visited_before in one pass over the bitmap (same result set).
#ifndef SG_SSSP_NOPROBE
#define SG_SSSP_NOPROBE 0   // SSSP diff mode: 1 skips the dist[v] probe before the RED
#endif
#ifndef SG_WORDS_NOPROBE
#define SG_WORDS_NOPROBE 1
#endif
#ifndef SG_HEAVY_NOPROBE
#define SG_HEAVY_NOPROBE 1
#endif
struct FnBfs {
    static constexpr bool kWeights = false;
    static constexpr bool kSeg = true;      // hubs may take the destination-segmented tier
    using Ctx = uint32_t;
    using Probe = uint64_t;
    uint64_t *visited;
    uint32_t *level;
    uint32_t next;
    const uint32_t *next_ptr;   // device-driven loop: level value read at flip time (else `next`)
    uint32_t *const *level_pp;  // device-driven loop: output buffer pointer read at flip time (else `level`)
    OutSink out;
    uint32_t diff;              // 1: mark visited only (k_bfs_diff builds the output)
    __device__ __forceinline__ Ctx ctx(int32_t) const { return 0u; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return ld_word(visited + (v >> 6)); }
    // CTA tier in diff mode: no probe, every arc issues its RED (no load latency to wait for)
    __device__ __forceinline__ bool skip_probe() const { return SG_HEAVY_NOPROBE && diff; }
    // word-path tiers (warp / thread) in diff mode: SG_WORDS_NOPROBE = 1 skips their probes too
    __device__ __forceinline__ bool skip_probe_words() const { return SG_WORDS_NOPROBE && diff; }
    template <int K>
    __device__ __forceinline__ void act_batch(const Ctx (&)[K], const int32_t (&v)[K], const uint32_t (&)[K],
                                              const Probe (&pr)[K], const bool (&ok)[K]) const {
        bool cand[K], flip[K], done[K];
        unsigned long long old[K];
        bool any = false;
#pragma unroll
        for (int k = 0; k < K; k++) cand[k] = ok[k] && !((pr[k] >> (v[k] & 63)) & 1ull);
        if (diff) {
#pragma unroll
            for (int k = 0; k < K; k++)
                if (cand[k]) atomic_or_u64(visited + (v[k] >> 6), 1ull << (v[k] & 63));   // RED
            return;
        }
#pragma unroll
        for (int k = 0; k < K; k++) old[k] = cand[k] ? atomic_or_u64(visited + (v[k] >> 6), 1ull << (v[k] & 63)) : ~0ull;
#pragma unroll
        for (int k = 0; k < K; k++) {
            flip[k] = cand[k] && !((old[k] >> (v[k] & 63)) & 1ull);
            any |= flip[k];
        }
        if (!any) return;
        uint32_t *lv = level_pp ? *level_pp : level;
        const uint32_t nx = next_ptr ? *next_ptr : next;
#pragma unroll
        for (int k = 0; k < K; k++)
            if (flip[k]) lv[v[k]] = nx;
        insert_batch(out, v, flip, done);
    }
};

// SSSP relax (Bellman-Ford by frontier): nd = dist[u] + w(u,v); v enters the output
// iff its distance decreased.  Updates are visible immediately (reading C12).
struct FnSssp {
    static constexpr bool kWeights = true;
    static constexpr bool kSeg = false;
    using Ctx = uint32_t;
    using Probe = uint32_t;
    uint32_t *dist;
    OutSink out;
    uint32_t diff;   // 1: fire-and-forget REDs (min), k_sssp_diff builds the output frontier
    __device__ __forceinline__ Ctx ctx(int32_t u) const { return *(volatile uint32_t *)(dist + u); }
    __device__ __forceinline__ bool skip_probe_words() const { return SG_SSSP_NOPROBE && diff; }
    __device__ __forceinline__ bool skip_probe() const { return SG_SSSP_NOPROBE && diff; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return dist[v]; }
    template <int K>
    __device__ __forceinline__ void act_batch(const Ctx (&du)[K], const int32_t (&v)[K], const uint32_t (&w)[K],
                                              const Probe (&pr)[K], const bool (&ok)[K]) const {
        uint32_t nd[K], old[K];
        bool cand[K], imp[K], done[K];
        if (diff) {   // relax only: dist[v] = min(dist[v], du + w) with no result to wait for
#pragma unroll
            for (int k = 0; k < K; k++) {
                nd[k] = du[k] + w[k];
                // (a skipped probe reads as INF: every arc of a reached source relaxes)
                const uint32_t p = skip_probe() ? INF32 : pr[k];
                if (ok[k] && du[k] != INF32 && nd[k] < p)
                    asm volatile("red.global.min.u32 [%0], %1;" ::"l"(dist + v[k]), "r"(nd[k]) : "memory");
            }
            return;
        }
#pragma unroll
        for (int k = 0; k < K; k++) {
            nd[k] = du[k] + w[k];
            cand[k] = ok[k] && du[k] != INF32 && nd[k] < pr[k];
        }
#pragma unroll
        for (int k = 0; k < K; k++) old[k] = cand[k] ? atomicMin(dist + v[k], nd[k]) : 0u;
#pragma unroll
        for (int k = 0; k < K; k++) imp[k] = cand[k] && old[k] > nd[k];
        insert_batch(out, v, imp, done);
    }
};

// CC label propagation (Stergiou et al.): push the source's label; v enters iff its
// label decreased.  Fixed point: min id per component (reading C13).
struct FnCc {
    static constexpr bool kWeights = false;
    static constexpr bool kSeg = false;
    using Ctx = int32_t;
    using Probe = int32_t;
    int32_t *label;
    OutSink out;
    __device__ __forceinline__ Ctx ctx(int32_t u) const { return *(volatile int32_t *)(label + u); }
    __device__ __forceinline__ bool skip_probe_words() const { return false; }
    __device__ __forceinline__ bool skip_probe() const { return false; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return label[v]; }
    template <int K>
    __device__ __forceinline__ void act_batch(const Ctx (&lu)[K], const int32_t (&v)[K], const uint32_t (&)[K],
                                              const Probe (&pr)[K], const bool (&ok)[K]) const {
        int32_t old[K];
        bool cand[K], imp[K], done[K];
#pragma unroll
        for (int k = 0; k < K; k++) cand[k] = ok[k] && lu[k] < pr[k];
#pragma unroll
        for (int k = 0; k < K; k++) old[k] = cand[k] ? atomicMin(label + v[k], lu[k]) : 0;
#pragma unroll
        for (int k = 0; k < K; k++) imp[k] = cand[k] && old[k] > lu[k];
        insert_batch(out, v, imp, done);
    }
};

// BC forward sigma (Brandes): `visited` is frozen during the step (levels <= d); every
// predecessor u of an unvisited v adds sigma[u] (level-d scale); the thread that flips v's
// output bit writes level[v] = d + 1.
struct FnBcSigma {
    static constexpr bool kWeights = false;
    static constexpr bool kSeg = false;
    using Ctx = double;
    using Probe = uint64_t;
    const uint64_t *visited;
    double *sigma;
    uint32_t *level;
    uint32_t next;
    OutSink out;
    __device__ __forceinline__ Ctx ctx(int32_t u) const { return sigma[u]; }
    __device__ __forceinline__ bool skip_probe_words() const { return false; }
    __device__ __forceinline__ bool skip_probe() const { return false; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return __ldg(visited + (v >> 6)); }
    template <int K>
    __device__ __forceinline__ void act_batch(const Ctx (&su)[K], const int32_t (&v)[K], const uint32_t (&)[K],
                                              const Probe (&pr)[K], const bool (&ok)[K]) const {
        bool cand[K], flip[K];
#pragma unroll
        for (int k = 0; k < K; k++) cand[k] = ok[k] && !((pr[k] >> (v[k] & 63)) & 1ull);
#pragma unroll
        for (int k = 0; k < K; k++)
            if (cand[k]) atomicAdd(sigma + v[k], su[k]);
        insert_batch(out, v, cand, flip);
#pragma unroll
        for (int k = 0; k < K; k++)
            if (flip[k]) level[v[k]] = next;
    }
};

}  // namespace sg
