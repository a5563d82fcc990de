// sparse.cu — one fused kernel per small BFS superstep (the leaf levels of a direction-optimising
// BFS: a few hundred words, a few thousand arcs).
//
// A dense push superstep is k_push_words + k_push_heavy (+ k_push_seg) + k_bfs_diff: four
// launches, the last a full pass over the 2 MB visited bitmap (R8).  For a frontier of a few
// words that is ~25 us of launch latency and bitmap scans around ~1 us of work.  Here the whole
// superstep is one persistent kernel (one CTA per SM):
//   0. (only if the output frontier still holds an old frontier) zero its listed words + layer 2,
//      grid barrier (+ the partition's superstep barrier, so no peer inserts into a replica that
//      is still being cleared);
//   1. a warp per listed input word expands it with the push tiers of push.cuh (thread tier for
//      low degrees, warp tier up to 256 arcs, longer lists queued as 256-arc items), then
//      zeroes the word (so the frontier is all-zero again once consumed);
//   2. grid barrier, then the queued items, a warp each (one round of 8 arcs per lane);
//   3. the output is inserted directly (Table 2 advance into an output frontier):
//      the thread whose atomicOr flips v's visited bit writes level[v] (Listing 1's compute,
//      fused), ORs v into the output layer 1, sets the layer-2 bit and appends the word to the
//      word list on the word's 0 -> non-zero transition; n_f / m_f and the list are
//      staged per CTA in shared memory and published with one global atomic per CTA;
//   4. the last CTA takes the direction decision (bfsstep.cuh), after the partition barrier.
// Results are the push superstep's (same set, same levels); chosen on the device by bfs_decide
// when the frontier has <= SG_SPARSE_WORDS words and m_f <= SG_SPARSE_ARCS; lists longer than
// 256 arcs are queued as 256-arc items so no hub serialises on one warp.
#include "common.cuh"
#include "kernels.h"
#include "push.cuh"
#include "bfsstep.cuh"
#include "xchg.cuh"

namespace sg {

constexpr int SP_THREADS = 256;
constexpr int SP_WARPS = SP_THREADS / 32;
constexpr int SP_LIST = 2048;   // word-list entries staged per CTA (overflow goes straight to global)
constexpr int SP_CHUNK = 256;   // arcs per queued item (one warp_expand round: 8 arcs per lane)

struct SparseAcc {
    unsigned long long nf, mf;
    uint32_t n;
    uint32_t list[SP_LIST];
};

// BFS functor with direct output insertion (no k_bfs_diff pass)
struct FnBfsDirect {
    static constexpr bool kWeights = false;
    static constexpr bool kSeg = false;
    using Ctx = uint32_t;
    using Probe = uint64_t;
    uint64_t *visited, *vis_old;
    uint32_t *const *level_pp;
    const uint32_t *next_ptr;
    uint64_t *out_bits, *out_summ;
    uint32_t *out_offsets;
    DevStats *st;
    const uint8_t *deg8;
    SparseAcc *acc;     // this CTA's shared-memory accumulator
    Xchg x;
    __device__ __forceinline__ Ctx ctx(int32_t) const { return 0u; }
    __device__ __forceinline__ Probe probe(int32_t v) const { return ld_word(visited + (v >> 6)); }
    __device__ __forceinline__ bool skip_probe() const { return false; }
    __device__ __forceinline__ bool skip_probe_words() const { return false; }
    __device__ __forceinline__ void append_word(uint32_t w) const {
        const uint32_t i = atomicAdd(&acc->n, 1u);
        if (i < (uint32_t)SP_LIST) {
            acc->list[i] = w;
            return;
        }
        // staging full: straight to every replica's list
        out_offsets[atomicAdd(&st->count, 1ull)] = w;
        for (int j = 0; j < x.nranks; j++)
            if (j != x.rank) xpeer(x, out_offsets, j)[atomicAdd(&xpeer(x, st, j)->count, 1ull)] = w;
    }
    template <int K>
    __device__ __forceinline__ void act_batch(const Ctx (&)[K], const int32_t (&v)[K], const uint32_t (&)[K],
                                              const Probe (&pr)[K], const bool (&ok)[K]) const {
        bool cand[K], flip[K];
        unsigned long long old[K];
        bool any = false;
#pragma unroll
        for (int k = 0; k < K; k++) cand[k] = ok[k] && !((pr[k] >> (v[k] & 63)) & 1ull);
#pragma unroll
        for (int k = 0; k < K; k++) old[k] = cand[k] ? atomic_or_u64(visited + (v[k] >> 6), 1ull << (v[k] & 63)) : ~0ull;
#pragma unroll
        for (int k = 0; k < K; k++) {
            flip[k] = cand[k] && !((old[k] >> (v[k] & 63)) & 1ull);
            any |= flip[k];
        }
        if (!any) return;
        uint32_t *lv = *level_pp;
        const uint32_t nx = *next_ptr;
        unsigned long long o2[K];
        uint32_t nf = 0;
        unsigned long long mf = 0;
#pragma unroll
        for (int k = 0; k < K; k++) {
            if (!flip[k]) continue;
            const unsigned long long bit = 1ull << (v[k] & 63);
            lv[v[k]] = nx;
            atomicOr(reinterpret_cast<unsigned long long *>(vis_old + (v[k] >> 6)), bit);
            o2[k] = atomic_or_u64(out_bits + (v[k] >> 6), bit);
            for (int j = 0; j < x.nranks; j++)
                if (j != x.rank) atomic_or_u64(xpeer(x, out_bits, j) + (v[k] >> 6), bit);
            nf++;
            mf += deg8_decode(__ldg(deg8 + v[k]));
        }
#pragma unroll
        for (int k = 0; k < K; k++) {
            if (!flip[k] || o2[k] != 0ull) continue;   // the word was already non-zero
            const uint32_t w = (uint32_t)(v[k] >> 6);
            const unsigned long long sb = 1ull << (w & 63);
            atomic_or_u64(out_summ + (w >> 6), sb);
            for (int j = 0; j < x.nranks; j++)
                if (j != x.rank) atomic_or_u64(xpeer(x, out_summ, j) + (w >> 6), sb);
            append_word(w);
        }
        atomicAdd(&acc->nf, (unsigned long long)nf);
        atomicAdd(&acc->mf, mf);
    }
};

// grid-wide barrier of a persistent grid (every CTA resident: one CTA per SM, 1 per SM fits)
__device__ __forceinline__ void grid_sync(unsigned int *gbar) {
    __syncthreads();
    if (threadIdx.x == 0) {
        volatile unsigned int *vgen = gbar + 1;
        const unsigned int gen = *vgen;
        __threadfence();
        if (atomicAdd(gbar, 1u) == gridDim.x - 1) {
            gbar[0] = 0u;
            __threadfence();
            atomicAdd(gbar + 1, 1u);
        } else {
            while (*vgen == gen) __nanosleep(64);
        }
        __threadfence();
    }
    __syncthreads();
}

// one frontier buffer as the loop kernel sees it
struct SpFrontier {
    uint64_t *bits, *summ;
    uint32_t *offsets;
    DevStats *st;
};
struct SpLoop {
    PushParams p;           // graph view, heavy queue, tier thresholds (frontier fields set per superstep)
    SpFrontier F[2];
    FnBfsDirect f;          // visited / vis_old / level / deg8 / peers (output fields set per superstep)
    BfsCtrl *c;
    unsigned int *gbar;
    int start;              // buffer holding the first superstep's input
};

// Consecutive small supersteps in one persistent kernel: superstep, grid barrier, decision by
// CTA 0 (after the partition barrier), grid barrier, and on as long as the decision is another
// sparse superstep — no graph node, launch or kernel tail between them.  The decision sets the
// IF handles of whichever half holds the next input (bfs_decide's next_in).
__global__ void __launch_bounds__(SP_THREADS) k_bfs_sparse_loop(SpLoop L) {
    __shared__ PushWarpSmem<FnBfsDirect> s_warp[SP_WARPS];
    __shared__ SparseAcc acc;
    __shared__ uint32_t s_base[1 + SG_MAX_RANKS];
    const int lane = lane_id(), wid = threadIdx.x >> 5;
    const uint32_t gwarp = blockIdx.x * SP_WARPS + wid, nwarps = gridDim.x * SP_WARPS;
    BfsCtrl *c = L.c;
    const Xchg &x = L.f.x;
    const bool lead = blockIdx.x == 0 && threadIdx.x == 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x, t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int in = L.start;
    unsigned long long t0 = lead ? global_ns() : 0ull;
    auto mark = [&](int k) {
        if (lead) {
            const unsigned long long t1 = global_ns();
            c->dbg[k] += t1 - t0;
            t0 = t1;
        }
    };
    for (;;) {
        const int out = in ^ 1;
        const SpFrontier Fi = L.F[in], Fo = L.F[out];
        if (threadIdx.x == 0) {
            acc.nf = acc.mf = 0ull;
            acc.n = 0u;
        }
        // 0. the output buffer must be all-zero: clear it if it still holds a consumed frontier
        if (*(volatile uint32_t *)&c->dirty[out]) {
            const unsigned long long nc = *(volatile unsigned long long *)&c->saved_count[out];
            if (nc == ~0ull) {
                for (int64_t w = t; w < L.p.g.nw1; w += stride) Fo.bits[w] = 0ull;
            } else {
                for (int64_t i = t; i < (int64_t)nc; i += stride) Fo.bits[Fo.offsets[i]] = 0ull;
            }
            for (int64_t s2 = t; s2 < L.p.g.nw2; s2 += stride) Fo.summ[s2] = 0ull;
            grid_sync(L.gbar);
            if (x.nranks > 1) {   // no peer may insert into this replica before it is clear
                if (lead) xbarrier(x, 0ull, 0ull, 0ull, nullptr);
                grid_sync(L.gbar);
            }
        } else {
            __syncthreads();
        }
        mark(0);
        PushParams p = L.p;
        p.in_bits = Fi.bits;
        p.offsets = Fi.offsets;
        p.st = Fi.st;
        FnBfsDirect fl = L.f;
        fl.out_bits = Fo.bits;
        fl.out_summ = Fo.summ;
        fl.out_offsets = Fo.offsets;
        fl.st = Fo.st;
        fl.acc = &acc;
        // 1. a warp per listed input word; the word is zeroed once expanded
        const uint32_t count = (uint32_t)*(volatile unsigned long long *)&Fi.st->count;
        unsigned long long arcs = 0;
        for (uint32_t i = gwarp; i < count; i += nwarps) {
            const uint32_t w = Fi.offsets[i];
            arcs += push_word(p, fl, (int64_t)w, s_warp[wid], false);
            if (lane == 0) {
                Fi.bits[w] = 0ull;
                Fi.summ[w >> 6] = 0ull;
            }
        }
        // 2. queued long lists: 256-arc items, a warp each
        mark(1);
        grid_sync(L.gbar);
        mark(2);
        const uint32_t hc =
            (uint32_t)min(*(volatile unsigned long long *)&Fi.st->heavy_count, (unsigned long long)p.heavy_cap);
        for (uint32_t i = gwarp; i < hc; i += nwarps) {
            const HeavyItem it = p.heavy[i];
            warp_expand(p.g, fl, it.begin, it.begin + it.len, 0u);
        }
        // 3. publish this CTA's word list (all replicas) and statistics
        mark(3);
        arcs = warp_sum(arcs);
        __syncthreads();
        const uint32_t n = min(acc.n, (uint32_t)SP_LIST);
        if (threadIdx.x == 0) {
            s_base[0] = n ? (uint32_t)atomicAdd(&Fo.st->count, (unsigned long long)n) : 0u;
            for (int j = 0; j < x.nranks; j++)
                if (j != x.rank) s_base[1 + j] = n ? (uint32_t)atomicAdd(&xpeer(x, Fo.st, j)->count, (unsigned long long)n) : 0u;
            if (acc.nf) {
                atomicAdd(&Fo.st->nf, acc.nf);
                atomicAdd(&Fo.st->mf, acc.mf);
            }
        }
        if (lane == 0 && arcs) atomicAdd(&Fi.st->arcs, arcs);
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
            Fo.offsets[s_base[0] + i] = acc.list[i];
            for (int j = 0; j < x.nranks; j++)
                if (j != x.rank) xpeer(x, Fo.offsets, j)[s_base[1 + j] + i] = acc.list[i];
        }
        if (x.nranks > 1) __threadfence_system();   // peer stores before the partition barrier
        mark(4);
        // every CTA arrives; CTA 0 waits for all, decides, and broadcasts through sp_epoch
        __syncthreads();
        uint32_t e0 = 0;
        if (threadIdx.x == 0) {
            e0 = *(volatile uint32_t *)&c->sp_epoch;
            __threadfence();
            atomicAdd(L.gbar + 2, 1u);
        }
        if (lead) {
            while (*(volatile unsigned int *)(L.gbar + 2) < gridDim.x) __nanosleep(32);
            L.gbar[2] = 0u;
            __threadfence();
        }
        mark(5);
        // dead-end lookahead of the output frontier (bfsstep.cuh; single GPU), whole CTA 0
        bool dead = false;
        if (blockIdx.x == 0) {
            __syncthreads();   // (the lead has seen every CTA arrive)
            if (x.nranks <= 1) {
                BfsOut lo{};
                lo.out_bits = Fo.bits;
                lo.out_offsets = Fo.offsets;
                lo.st = Fo.st;
                lo.rp = L.p.g.rp;
                lo.col = L.p.g.col;
                lo.visited = L.f.visited;
                dead = bfs_lookahead(lo);
            }
        }
        // 4. decision (CTA 0): the input is retired as all-zero (cleared word by word above)
        if (lead) {
            DevStats *prev = Fi.st;
            volatile DevStats *vp = prev;
            unsigned long long prev_arcs = vp->arcs;
            c->saved_count[in] = vp->count;
            c->dirty[in] = 0u;
            uint32_t kind;
            if (x.nranks > 1) {
                volatile DevStats *vo = Fo.st;
                const unsigned long long my_nf = vo->nf, my_mf = vo->mf;
                *prev = DevStats{};   // zero before peers may add into it (next output)
                XSlot tot;
                xbarrier(x, my_nf, my_mf, prev_arcs, &tot);
                vo->nf = tot.nf;
                vo->mf = tot.mf;
                vo->pad = tot.arcs;
                kind = bfs_decide(c, Fo.st, tot.arcs, nullptr, out, 0, true);
            } else {
                kind = bfs_decide(c, Fo.st, prev_arcs, prev, out, 0, true, dead);
            }
            c->sp_kind = kind;
            __threadfence();
            *(volatile uint32_t *)&c->sp_epoch = e0 + 1u;
        } else if (threadIdx.x == 0) {
            while (*(volatile uint32_t *)&c->sp_epoch == e0) __nanosleep(32);
            __threadfence();
        }
        mark(6);
        __syncthreads();
        mark(7);
        if (lead) c->dbg[15]++;
        if (*(volatile uint32_t *)&c->sp_kind != SK_SPARSE) break;
        in = out;
    }
}

void launch_bfs_sparse(const PushLaunch &Lp, const BfsArgs &a, const BfsOut &o, uint64_t *in_bits, uint64_t *in_summ,
                       unsigned int *gbar, cudaStream_t s) {
    SpLoop L;
    PushParams &p = L.p;
    p.g = Lp.g;
    p.in_bits = nullptr;
    p.offsets = nullptr;
    p.st = nullptr;
    p.heavy = Lp.heavy;
    p.heavy_cap = Lp.heavy_cap;
    // lists longer than one warp round (256 arcs) are cut into 256-arc items spread over the
    // grid's warps: a sparse superstep has <= SG_SPARSE_ARCS arcs, so a hub must not serialise
    // on one warp (its atomics return values: a round is a chain of dependent round trips)
    p.heavy_deg = SP_CHUNK;
    p.chunk = SP_CHUNK;
    p.small_deg = Lp.small_deg < SP_CHUNK ? Lp.small_deg : SP_CHUNK;
    p.batch = 1;
    p.seg = nullptr;
    p.seg_cap = 0;
    p.seg_mode = 0;
    p.seg_threshold = ~0ull;
    p.skip_mf = ~0ull;
    p.sparse_ok = 0;
    // buffer o.half is the first input, o's output is the other one
    L.start = o.half;
    L.F[o.half] = SpFrontier{in_bits, in_summ, const_cast<uint32_t *>(Lp.offsets), Lp.st};
    L.F[o.half ^ 1] = SpFrontier{o.out_bits, o.out_summ, o.out_offsets, o.st};
    FnBfsDirect &f = L.f;
    f.visited = a.visited;
    f.vis_old = o.vis_old;
    f.level_pp = a.level_pp;
    f.next_ptr = a.next_ptr;
    f.out_bits = nullptr;
    f.out_summ = nullptr;
    f.out_offsets = nullptr;
    f.st = nullptr;
    f.deg8 = Lp.g.deg8;
    f.acc = nullptr;
    f.x = o.x;
    L.c = o.ctrl;
    L.gbar = gbar;
    note_launch();
    k_bfs_sparse_loop<<<num_sms(), SP_THREADS, 0, s>>>(L);
}

}  // namespace sg
