// functors.cuh — per-edge advance functors (Table 2: Functor(src, dst, edge,
// weight) -> bool "whether dst should be added to the frontier"; algorithms P:161 §3.4).
//
// Split into ctx(src) (loaded once per source vertex), probe(dst) (the one random load per
// arc; issued for several arcs before any decision so the loads overlap) and act(...)
// (decision + atomics + insertion into the output 2LB).  The compute step of Listing 1
// (dist[v] = iter + 1) is fused into act: the thread whose atomic inserts v
// writes its value (the paper keeps it separate; on B200 the fused store saves a pass).
#pragma once
#include "common.cuh"

namespace sg {

struct OutSink {
    uint64_t *bits;   // nullptr: advance without an output frontier
    uint64_t *summ;
    __device__ __forceinline__ bool insert(int32_t v) const { return bits ? insert_2lb(bits, summ, v) : true; }
};

// BFS (Listing 1 l.9-13 + l.14-17).  `visited` is updated live: the first thread whose
// atomicOr sets v's visited bit owns v, writes level[v] and inserts v.  A stale probe only
// costs one extra atomic.  Result = {v unvisited before the step with a neighbour in the
// frontier}, identical to the frozen-visited reading.
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
    __device__ __forceinline__ Ctx ctx(int32_t) const { return 0u; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return ld_word(visited + (v >> 6)); }
    __device__ __forceinline__ void act(Ctx, int32_t v, uint32_t, Probe pr) const {
        const uint64_t m = 1ull << (v & 63);
        if (pr & m) return;
        if (atomic_or_u64(visited + (v >> 6), m) & m) return;
        (level_pp ? *level_pp : level)[v] = next_ptr ? *next_ptr : next;
        out.insert(v);
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
    __device__ __forceinline__ Ctx ctx(int32_t u) const { return *(volatile uint32_t *)(dist + u); }
    __device__ __forceinline__ Probe probe(int32_t v) const { return dist[v]; }
    __device__ __forceinline__ void act(Ctx du, int32_t v, uint32_t w, Probe pr) const {
        if (du == INF32) return;
        const uint32_t nd = du + w;
        if (nd >= pr) return;
        if (atomicMin(dist + v, nd) > nd) out.insert(v);
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
    __device__ __forceinline__ Probe probe(int32_t v) const { return label[v]; }
    __device__ __forceinline__ void act(Ctx lu, int32_t v, uint32_t, Probe pr) const {
        if (lu >= pr) return;
        if (atomicMin(label + v, lu) > lu) out.insert(v);
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
    __device__ __forceinline__ Probe probe(int32_t v) const { return __ldg(visited + (v >> 6)); }
    __device__ __forceinline__ void act(Ctx su, int32_t v, uint32_t, Probe pr) const {
        if (pr & (1ull << (v & 63))) return;
        atomicAdd(sigma + v, su);
        if (out.insert(v)) level[v] = next;
    }
};

}  // namespace sg
