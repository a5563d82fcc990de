// push.cuh — the load-balanced push advance over a Two-Layer-Bitmap frontier
// (PAPER.md:231-233 §4.2 workload mapping, :249-262 §4.3 2LB + offsets buffer).
//
// B200 design:
//   * the offsets buffer (non-zero layer-1 words, from k_compact) is consumed by persistent
//     CTAs that grab batches of PUSH_BATCH words with one atomic per batch (the paper's
//     "set number of workgroups iterating over the offsets buffer", with its
//     coarsening factor);
//   * one warp owns one 64-bit word (2 bits per lane: the paper's MSI for 64-bit words)
//     and splits its active vertices into degree tiers:
//       - thread tier  (deg <= small_deg): the warp packs all such vertices' arcs into one
//         list and gives each lane single arcs (ballot/popc start-mask mapping, no search),
//         so a word with one or two low-degree vertices does not idle 31 lanes (Fig. 5b);
//       - warp tier    (small_deg < deg <= heavy_deg): the warp streams the list with
//         16-byte vectorised col_idx loads, 8 arcs in flight per lane;
//       - CTA/grid tier (deg > heavy_deg): the list is cut into HEAVY_CHUNK-arc chunks queued
//         in global memory and expanded by k_push_heavy, whose CTAs stage each chunk into
//         shared memory with cp.async.bulk (TMA bulk copy, mbarrier completion) in a
//         HEAVY_STAGES-deep ring; a hub's chunks spread across all CTAs (grid tier);
//   * per arc: probe (one random load: visited word / dist / label) issued for all arcs in
//     flight before any decision, then the functor's act (atomics on 64-bit words, summary
//     bit only on the word's 0 -> non-zero transition).
#pragma once
#include <type_traits>
#include "common.cuh"
#include "functors.cuh"

namespace sg {

#ifndef SG_SPARSE_WORDS
#define SG_SPARSE_WORDS 1
#endif
constexpr int PUSH_THREADS = 256;
constexpr int PUSH_WARPS = PUSH_THREADS / 32;
constexpr int HEAVY_THREADS = 256;
constexpr int HEAVY_STAGES = 4;
constexpr int HEAVY_BUF_INTS = HEAVY_CHUNK + 8;   // alignment slack for 16-B bulk copies
constexpr size_t HEAVY_SMEM = (size_t)HEAVY_STAGES * HEAVY_BUF_INTS * 4 + HEAVY_STAGES * 8;

struct PushParams {
    GraphView g;
    const uint64_t *in_bits;
    const uint32_t *offsets;
    DevStats *st;          // count (input), batch / heavy_count / arcs (scratch, zeroed by host)
    HeavyItem *heavy;
    uint32_t heavy_cap;
    int32_t heavy_deg;
    int32_t small_deg;
    int32_t batch;         // words per warp grab (0: derive from the device-side count)
    SegItem *seg;          // destination-segmented hub queue (BFS only)
    uint32_t seg_cap;
    int32_t seg_mode;      // 0 off, 1 auto (when the frontier's m_f >= seg_threshold), 2 always
    unsigned long long seg_threshold;
    unsigned long long skip_mf;   // the segmented (SCSR) advance handles this superstep: m_f >= skip_mf
    int32_t sparse_ok;     // st->nf is exact: words with <= 2 active vertices on average take the
                           // thread-per-word path (push_words_sparse)
    int32_t chunk = HEAVY_CHUNK;   // arcs per queued CTA/grid-tier item (the sparse kernel: a warp round)
};

constexpr int HUBQ = 64;   // hubs a warp buffers before queueing their segment-tier chunks
// segmented hub tier (BFS): hubs found by a warp, queued in bulk (one seg_count atomic per flush
// instead of one per hub: 13-18 K hubs on one counter serialised a level-2 k_push_words at 36 us,
// profiles/r02i)
struct PushHubQ {
    int64_t hq_s[HUBQ], hq_e[HUBQ];
    int32_t hq_u[HUBQ];
    int32_t nhq;
};
struct PushNoHubQ {};
template <class F>
struct PushWarpSmem : std::conditional_t<F::kSeg, PushHubQ, PushNoHubQ> {
    int64_t start[64];
    uint32_t pre[64];
    typename F::Ctx ctx[64];
};

template <class F>
__device__ __forceinline__ uint32_t load_w(const GraphView &g, int64_t i) {
    if constexpr (F::kWeights) return __ldg(g.w + i);
    else return 0u;
}

// ---- warp tier -------------------------------------------------------------------------
template <class F>
__device__ __forceinline__ void warp_expand(const GraphView &g, const F &f, int64_t s, int64_t e,
                                            typename F::Ctx c) {
    const int lane = lane_id();
    int64_t a = (s + 3) & ~3ll;
    if (a > e) a = e;
    const int64_t b = a + ((e - a) & ~3ll);
    {   // ragged head [s, a) on lanes 0..2 and tail [b, e) on lanes 4..6
        int64_t i = -1;
        if (lane < a - s) i = s + lane;
        else if (lane >= 4 && lane - 4 < e - b) i = b + (lane - 4);
        if (i >= 0) {
            const int32_t v[1] = {__ldg(g.col + i)};
            const uint32_t w[1] = {load_w<F>(g, i)};
            const typename F::Probe pr[1] = {f.skip_probe_words() ? typename F::Probe{} : f.probe(v[0])};
            const typename F::Ctx cc[1] = {c};
            const bool ok[1] = {true};
            f.act_batch(cc, v, w, pr, ok);
        }
    }
    for (int64_t i = a + 4 * lane; i < b; i += 256) {
        const bool two = i + 128 < b;
        const int4 v0 = __ldg(reinterpret_cast<const int4 *>(g.col + i));
        int4 v1 = make_int4(0, 0, 0, 0);
        if (two) v1 = __ldg(reinterpret_cast<const int4 *>(g.col + i + 128));
        uint32_t w0 = 0, w1 = 0;
        if constexpr (F::kWeights) {
            w0 = __ldg(reinterpret_cast<const uint32_t *>(g.w + i));
            if (two) w1 = __ldg(reinterpret_cast<const uint32_t *>(g.w + i + 128));
        }
        const int32_t v[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
        const uint32_t w[8] = {w0 & 0xff, (w0 >> 8) & 0xff, (w0 >> 16) & 0xff, w0 >> 24,
                               w1 & 0xff, (w1 >> 8) & 0xff, (w1 >> 16) & 0xff, w1 >> 24};
        const bool ok[8] = {true, true, true, true, two, two, two, two};
        typename F::Probe pr[8];
        typename F::Ctx cc[8];
#pragma unroll
        for (int k = 0; k < 8; k++) {
            pr[k] = ok[k] && !f.skip_probe_words() ? f.probe(v[k]) : typename F::Probe{};
            cc[k] = c;
        }
        f.act_batch(cc, v, w, pr, ok);
    }
}

// ---- CTA/grid tier enqueue -------------------------------------------------------------
__device__ __forceinline__ void enqueue_heavy(const PushParams &p, int32_t u, int64_t s, int64_t e) {
    const int64_t d = e - s;
    const int64_t ch = p.chunk;
    const uint32_t nch = (uint32_t)((d + ch - 1) / ch);
    const unsigned long long pos = atomicAdd(&p.st->heavy_count, (unsigned long long)nch);
    for (uint32_t j = 0; j < nch; j++) {
        if (pos + j >= p.heavy_cap) break;      // cannot happen: capacity bound in DESIGN.md
        HeavyItem it;
        it.begin = s + (int64_t)j * ch;
        it.len = (int32_t)min(ch, e - it.begin);
        it.u = u;
        p.heavy[pos + j] = it;
    }
}

// ---- segmented hub tier enqueue (BFS) ----------------------------------------------------
__device__ __forceinline__ void enqueue_seg(const PushParams &p, int32_t h, int64_t s, int64_t e) {
    const int64_t d = e - s;
    const uint32_t nch = (uint32_t)((d + HEAVY_CHUNK - 1) / HEAVY_CHUNK);
    const unsigned long long pos = atomicAdd(&p.st->seg_count, (unsigned long long)nch);
    for (uint32_t j = 0; j < nch; j++) {
        if (pos + j >= p.seg_cap) break;        // cannot happen: capacity bound in DESIGN.md
        SegItem it;
        it.begin = s + (int64_t)j * HEAVY_CHUNK;
        it.row = s;
        it.len = (int32_t)min((int64_t)HEAVY_CHUNK, e - it.begin);
        it.h = h;
        p.seg[pos + j] = it;
    }
}

// queue the warp's buffered hubs as segment-tier chunks: one atomic for all of them, each
// lane writes the chunks of its entries (whole warp; sm.nhq warp-uniform)
template <class F>
__device__ __forceinline__ void flush_hubs(const PushParams &p, PushWarpSmem<F> &sm) {
    const int lane = lane_id();
    const int n = sm.nhq;
    if (n == 0) return;
    int64_t s[2] = {0, 0}, e[2] = {0, 0};
    int32_t h[2] = {0, 0};
    uint32_t nch[2] = {0u, 0u};
#pragma unroll
    for (int k = 0; k < 2; k++) {
        const int i = lane + 32 * k;
        if (i < n) {
            s[k] = sm.hq_s[i];
            e[k] = sm.hq_e[i];
            h[k] = __ldg(p.g.hub_idx + sm.hq_u[i]);
            nch[k] = (uint32_t)((e[k] - s[k] + HEAVY_CHUNK - 1) / HEAVY_CHUNK);
        }
    }
    const uint32_t mine = nch[0] + nch[1];
    const uint32_t incl = warp_inclusive_scan(mine);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 31);
    unsigned long long base = 0;
    if (lane == 31) base = atomicAdd(&p.st->seg_count, (unsigned long long)tot);
    base = __shfl_sync(0xffffffffu, base, 31) + (incl - mine);
#pragma unroll
    for (int k = 0; k < 2; k++) {
        for (uint32_t j = 0; j < nch[k]; j++, base++) {
            if (base >= p.seg_cap) break;   // cannot happen: capacity bound in DESIGN.md
            SegItem it;
            it.begin = s[k] + (int64_t)j * HEAVY_CHUNK;
            it.row = s[k];
            it.len = (int32_t)min((int64_t)HEAVY_CHUNK, e[k] - it.begin);
            it.h = h[k];
            p.seg[base] = it;
        }
    }
    __syncwarp();
    if (lane == 0) sm.nhq = 0;
    __syncwarp();
}

// ---- one word on one warp ----------------------------------------------------------------
template <class F>
__device__ __forceinline__ unsigned long long push_word(const PushParams &p, const F &f, int64_t w,
                                                        PushWarpSmem<F> &sm, bool seg_on) {
    const int lane = lane_id();
    const uint64_t x = __ldg(p.in_bits + w);
    int64_t sa, ea, sb, eb;
    word_bounds(p.g, w, x, sa, ea, sb, eb);
    const int32_t ua = (int32_t)(w * 64 + lane), ub = ua + 32;
    const int64_t d_total = (ea - sa) + (eb - sb);
    if constexpr (F::kSeg) {
        if (seg_on) {   // hubs go to the destination-segmented tier (visited slice in shared memory),
                        // buffered per warp and queued in bulk (flush_hubs)
            const bool qa = ea - sa >= SEG_MIN, qb = eb - sb >= SEG_MIN;
            const uint32_t ba = __ballot_sync(0xffffffffu, qa), bb = __ballot_sync(0xffffffffu, qb);
            const int nq = __popc(ba) + __popc(bb);
            if (nq) {
                if (sm.nhq + nq > HUBQ) flush_hubs(p, sm);
                const uint32_t lt = (1u << lane) - 1u;
                const int n0 = sm.nhq;
                if (qa) {
                    const int i = n0 + __popc(ba & lt);
                    sm.hq_s[i] = sa;
                    sm.hq_e[i] = ea;
                    sm.hq_u[i] = ua;
                    sa = ea;
                }
                if (qb) {
                    const int i = n0 + __popc(ba) + __popc(bb & lt);
                    sm.hq_s[i] = sb;
                    sm.hq_e[i] = eb;
                    sm.hq_u[i] = ub;
                    sb = eb;
                }
                __syncwarp();
                if (lane == 0) sm.nhq = n0 + nq;
                __syncwarp();
            }
        }
    }
    const int64_t da = ea - sa, db = eb - sb;
    const bool ha = da > p.heavy_deg, hb = db > p.heavy_deg;
    if (ha) enqueue_heavy(p, ua, sa, ea);
    if (hb) enqueue_heavy(p, ub, sb, eb);
    const bool ma = !ha && da > p.small_deg, mb = !hb && db > p.small_deg;
    const bool ta = da > 0 && da <= p.small_deg, tb = db > 0 && db <= p.small_deg;
    typename F::Ctx ca{}, cb{};
    if (ma || ta) ca = f.ctx(ua);
    if (mb || tb) cb = f.ctx(ub);

    // warp tier: one vertex at a time, whole warp
    uint32_t mm = __ballot_sync(0xffffffffu, ma);
    while (mm) {
        const int src = __ffs(mm) - 1;
        mm &= mm - 1;
        warp_expand(p.g, f, __shfl_sync(0xffffffffu, sa, src), __shfl_sync(0xffffffffu, ea, src),
                    __shfl_sync(0xffffffffu, ca, src));
    }
    mm = __ballot_sync(0xffffffffu, mb);
    while (mm) {
        const int src = __ffs(mm) - 1;
        mm &= mm - 1;
        warp_expand(p.g, f, __shfl_sync(0xffffffffu, sb, src), __shfl_sync(0xffffffffu, eb, src),
                    __shfl_sync(0xffffffffu, cb, src));
    }

    // thread tier: pack the low-degree vertices' arcs, one arc per lane per window
    const uint32_t la = ta ? (uint32_t)da : 0u, lb = tb ? (uint32_t)db : 0u;
    const uint32_t mine = la + lb;
    const uint32_t incl = warp_inclusive_scan(mine);
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    if (total) {
        const uint32_t pa = incl - mine, pb = pa + la;
        const uint32_t bal_a = __ballot_sync(0xffffffffu, ta), bal_b = __ballot_sync(0xffffffffu, tb);
        const uint32_t lt = (1u << lane) - 1u;
        const int slot_a = __popc(bal_a & lt) + __popc(bal_b & lt);
        const int slot_b = slot_a + (ta ? 1 : 0);
        if (ta) { sm.start[slot_a] = sa; sm.pre[slot_a] = pa; sm.ctx[slot_a] = ca; }
        if (tb) { sm.start[slot_b] = sb; sm.pre[slot_b] = pb; sm.ctx[slot_b] = cb; }
        __syncwarp();
        int kb = -1;
        for (uint32_t base = 0; base < total; base += 64) {
            // bit (P_k - base) marks vertex k's first arc inside this 64-arc window
            uint64_t m = 0;
            if (ta && pa >= base && pa < base + 64) m |= 1ull << (pa - base);
            if (tb && pb >= base && pb < base + 64) m |= 1ull << (pb - base);
            const uint32_t lo = __reduce_or_sync(0xffffffffu, (uint32_t)m);
            const uint32_t hi = __reduce_or_sync(0xffffffffu, (uint32_t)(m >> 32));
            const uint64_t mask = (uint64_t)lo | ((uint64_t)hi << 32);
            const int k0 = kb + __popcll(mask & ((2ull << lane) - 1ull));
            const int k1 = kb + __popcll(mask & ((2ull << (lane + 32)) - 1ull));
            const uint32_t e0 = base + lane, e1 = base + 32 + lane;
            const bool ok0 = e0 < total, ok1 = e1 < total;
            int32_t v[2] = {0, 0};
            uint32_t w[2] = {0u, 0u};
            typename F::Ctx cc[2] = {};
            const bool ok[2] = {ok0, ok1};
            if (ok0) {
                const int64_t i = sm.start[k0] + (e0 - sm.pre[k0]);
                v[0] = __ldg(p.g.col + i);
                w[0] = load_w<F>(p.g, i);
                cc[0] = sm.ctx[k0];
            }
            if (ok1) {
                const int64_t i = sm.start[k1] + (e1 - sm.pre[k1]);
                v[1] = __ldg(p.g.col + i);
                w[1] = load_w<F>(p.g, i);
                cc[1] = sm.ctx[k1];
            }
            typename F::Probe pr[2] = {};
            if (ok0 && !f.skip_probe_words()) pr[0] = f.probe(v[0]);
            if (ok1 && !f.skip_probe_words()) pr[1] = f.probe(v[1]);
            f.act_batch(cc, v, w, pr, ok);
            kb += __popcll(mask);
        }
        __syncwarp();
    }
    return (unsigned long long)d_total;
}

// ---- sparse frontiers: one thread per word -------------------------------------------------
// When the words hold <= 2 active vertices on average (n_f <= 2 count) of low average degree
// (m_f <= 16 n_f: the leaf levels of a BFS),
// a warp-per-word mapping runs the word's dependent load chain (word -> row_ptr -> col_idx ->
// probe) once per word per warp.  Here each lane takes one word: its vertices' low-degree lists
// are expanded by the lane itself (4 arcs in flight), up to 2 mid-degree vertices per lane are
// expanded afterwards by the whole warp, hubs go to the CTA / segmented tiers as usual.
template <class F>
__device__ __forceinline__ void thread_expand(const GraphView &g, const F &f, int64_t s, int64_t e,
                                              typename F::Ctx c) {
    for (int64_t r = s; r < e; r += 4) {
        int32_t v[4];
        uint32_t w[4];
        bool ok[4];
        typename F::Probe pr[4];
        typename F::Ctx cc[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            ok[k] = r + k < e;
            v[k] = ok[k] ? __ldg(g.col + r + k) : 0;
            w[k] = ok[k] ? load_w<F>(g, r + k) : 0u;
            cc[k] = c;
        }
#pragma unroll
        for (int k = 0; k < 4; k++) pr[k] = ok[k] && !f.skip_probe_words() ? f.probe(v[k]) : typename F::Probe{};
        f.act_batch(cc, v, w, pr, ok);
    }
}
template <class F>
__device__ __forceinline__ unsigned long long push_words_sparse(const PushParams &p, const F &f, uint32_t i,
                                                                uint32_t count, bool seg_on) {
    unsigned long long arcs = 0;
    int64_t ds[2] = {0, 0}, de[2] = {0, 0};
    int32_t du[2] = {-1, -1};
    int nd = 0;
    if (i < count) {
        const int64_t w = p.offsets[i];
        uint64_t x = __ldg(p.in_bits + w);
        while (x) {
            const int b = __ffsll((long long)x) - 1;
            x &= x - 1;
            const int32_t u = (int32_t)(w * 64 + b);
            const int64_t s = __ldg(p.g.rp + u), e = __ldg(p.g.rp + u + 1);
            const int64_t d = e - s;
            arcs += (unsigned long long)d;
            if constexpr (F::kSeg) {
                if (seg_on && d >= SEG_MIN) {
                    enqueue_seg(p, __ldg(p.g.hub_idx + u), s, e);
                    continue;
                }
            }
            if (d > p.heavy_deg) {
                enqueue_heavy(p, u, s, e);
            } else if (d > p.small_deg && nd < 2) {
                ds[nd] = s;
                de[nd] = e;
                du[nd] = u;
                nd++;
            } else if (d > 0) {
                thread_expand(p.g, f, s, e, f.ctx(u));
            }
        }
    }
#pragma unroll
    for (int k = 0; k < 2; k++) {   // mid-degree vertices: the whole warp, one at a time
        uint32_t mm = __ballot_sync(0xffffffffu, du[k] >= 0);
        while (mm) {
            const int src = __ffs(mm) - 1;
            mm &= mm - 1;
            const int32_t u = __shfl_sync(0xffffffffu, du[k], src);
            warp_expand(p.g, f, __shfl_sync(0xffffffffu, ds[k], src), __shfl_sync(0xffffffffu, de[k], src), f.ctx(u));
        }
    }
    return arcs;
}

template <class F>
__global__ void __launch_bounds__(PUSH_THREADS) k_push_words(PushParams p, F f) {
    __shared__ PushWarpSmem<F> s_warp[PUSH_WARPS];
    __shared__ unsigned long long s_arcs[PUSH_WARPS];
    if (p.st->mf >= p.skip_mf) return;
    const uint32_t count = (uint32_t)p.st->count;
    const int wid = threadIdx.x >> 5;
    unsigned long long arcs = 0;
    // each warp grabs `batch` words (the coarsening factor) with one atomic; no CTA barrier in
    // the loop, so a warp never waits for a slower sibling's batch
    uint32_t batch = (uint32_t)p.batch;
    if (batch == 0) {   // device-driven loop: coarsening factor from the device-side count
        batch = count / (gridDim.x * PUSH_WARPS * 4u);
        batch = batch < 1u ? 1u : (batch > 8u ? 8u : batch);
    }
    bool seg_on = false;
    if constexpr (F::kSeg)
        seg_on = p.g.hub_idx != nullptr && p.seg != nullptr &&
                 (p.seg_mode == 2 || (p.seg_mode == 1 && p.st->mf >= p.seg_threshold));
    // sparse: <= 2 active vertices per word on average, of average degree <= 16 (else the
    // warp-tier vertices of 32 words would serialise on one warp)
    const bool sparse = SG_SPARSE_WORDS && p.sparse_ok && p.st->nf <= 2ull * count && p.st->mf <= 16ull * p.st->nf;
    if constexpr (F::kSeg) {
        if (lane_id() == 0) s_warp[wid].nhq = 0;
        __syncwarp();
    }
    const uint32_t grab = sparse ? 32u : batch;
    if constexpr (F::kSeg) {
        // BFS: each CTA takes a contiguous share of the word list; its warps take `grab` words at
        // a time, the first grab static (warp id x grab), later ones from a shared-memory counter.
        // (One global counter for all warps serialised a 13 K-word hub level at ~8 K same-address
        // atomics: 45 % of that k_push_words' stall samples, profiles/r02j_full_l2push.  Its hubs
        // leave the warp as queued chunks, so the per-word work is small and even.)
        __shared__ uint32_t s_next;
        if (threadIdx.x == 0) s_next = 0u;
        __syncthreads();
        const uint32_t per = (count + gridDim.x - 1) / gridDim.x;
        const uint32_t c0 = min(blockIdx.x * per, count), c1 = min(c0 + per, count);
        const uint32_t statics = PUSH_WARPS * grab;
        for (uint32_t r = wid * grab;;) {
            const uint32_t b0 = c0 + r;
            if (b0 >= c1) break;
            if (sparse) {   // 32 words per grab, one per lane
                arcs += push_words_sparse(p, f, b0 + lane_id(), c1, seg_on);
            } else {
                const uint32_t b1 = min(b0 + grab, c1);
                for (uint32_t i = b0; i < b1; i++) arcs += push_word(p, f, p.offsets[i], s_warp[wid], seg_on);
            }
            if (c0 + statics >= c1) break;
            uint32_t nb = 0;
            if (lane_id() == 0) nb = statics + atomicAdd(&s_next, grab);
            r = __shfl_sync(0xffffffffu, nb, 0);
        }
    } else {
        // SSSP / CC / BC: grid-wide dynamic grabs (a warp's first grab static, later ones from one
        // global counter): their words carry uneven warp-tier work that a static CTA share leaves
        // unbalanced (C2 SSSP 0.90 -> 1.51 ms when it shared the BFS scheme)
        const uint32_t gwarp = (blockIdx.x * PUSH_THREADS + threadIdx.x) >> 5;
        const uint32_t nwarps = gridDim.x * PUSH_WARPS;
        const unsigned long long statics = (unsigned long long)nwarps * grab;
        for (unsigned long long b0l = (unsigned long long)gwarp * grab;;) {
            if (b0l >= count) break;
            const uint32_t b0 = (uint32_t)b0l;
            if (sparse) {
                arcs += push_words_sparse(p, f, b0 + lane_id(), count, seg_on);
            } else {
                const uint32_t b1 = min(b0 + grab, count);
                for (uint32_t i = b0; i < b1; i++) arcs += push_word(p, f, p.offsets[i], s_warp[wid], seg_on);
            }
            if (statics >= count) break;
            unsigned long long nb = 0;
            if (lane_id() == 0) nb = statics + atomicAdd(&p.st->batch, (unsigned long long)grab);
            b0l = __shfl_sync(0xffffffffu, nb, 0);
        }
    }
    if constexpr (F::kSeg) flush_hubs(p, s_warp[wid]);
    arcs = warp_sum(arcs);
    if (lane_id() == 0) s_arcs[wid] = arcs;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int i = 0; i < PUSH_WARPS; i++) t += s_arcs[i];
        if (t) atomicAdd(&p.st->arcs, t);
    }
}

// ---- CTA/grid tier: TMA-bulk-staged chunks ---------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *ptr) {
    return (uint32_t)__cvta_generic_to_shared(ptr);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(phase)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk_g2s(void *dst_smem, const void *src_gmem, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst_smem)),
        "l"(src_gmem), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

template <class F>
__global__ void __launch_bounds__(HEAVY_THREADS) k_push_heavy(PushParams p, F f) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    int32_t *buf = reinterpret_cast<int32_t *>(smem_raw);
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem_raw + (size_t)HEAVY_STAGES * HEAVY_BUF_INTS * 4);
    const unsigned long long hc = p.st->heavy_count;
    const uint32_t nitems = (uint32_t)(hc < p.heavy_cap ? hc : p.heavy_cap);
    const uint32_t G = gridDim.x;
    const uint32_t my_n = nitems > blockIdx.x ? (nitems - blockIdx.x + G - 1) / G : 0u;
    if (my_n == 0) return;
    if (threadIdx.x == 0) {
        for (int s = 0; s < HEAVY_STAGES; s++) mbar_init(bar + s, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](uint32_t j) {
        const HeavyItem it = p.heavy[blockIdx.x + (size_t)j * G];
        const int64_t a = it.begin & ~3ll;
        const int64_t b = (it.begin + it.len + 3) & ~3ll;
        const uint32_t bytes = (uint32_t)((b - a) * 4);
        const int s = j % HEAVY_STAGES;
        mbar_expect_tx(bar + s, bytes);
        bulk_g2s(buf + (size_t)s * HEAVY_BUF_INTS, p.g.col + a, bytes, bar + s);
    };
    if (threadIdx.x == 0)
        for (uint32_t j = 0; j < my_n && j < (uint32_t)HEAVY_STAGES; j++) issue(j);
    for (uint32_t j = 0; j < my_n; j++) {
        const int s = j % HEAVY_STAGES;
        const uint32_t phase = (j / HEAVY_STAGES) & 1u;
        const HeavyItem it = p.heavy[blockIdx.x + (size_t)j * G];
        const typename F::Ctx c = f.ctx(it.u);
        mbar_wait(bar + s, phase);
        const int32_t *src = buf + (size_t)s * HEAVY_BUF_INTS + (it.begin & 3);
        // all HEAVY_CHUNK / HEAVY_THREADS arcs of a thread in one batch: their probes and then
        // their atomics are all in flight together
        constexpr int KH = HEAVY_CHUNK / HEAVY_THREADS;
        {
            const int i = threadIdx.x;
            int32_t v[KH];
            uint32_t w[KH];
            bool ok[KH];
            typename F::Probe pr[KH];
            typename F::Ctx cc[KH];
#pragma unroll
            for (int k = 0; k < KH; k++) {
                const int ii = i + k * HEAVY_THREADS;
                ok[k] = ii < it.len;
                v[k] = ok[k] ? src[ii] : 0;
                w[k] = ok[k] ? load_w<F>(p.g, it.begin + ii) : 0u;
                cc[k] = c;
            }
#pragma unroll
            for (int k = 0; k < KH; k++) pr[k] = ok[k] && !f.skip_probe() ? f.probe(v[k]) : typename F::Probe{};
            f.act_batch(cc, v, w, pr, ok);
        }
        __syncthreads();   // buffer s fully consumed
        if (threadIdx.x == 0 && j + HEAVY_STAGES < my_n) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(j + HEAVY_STAGES);
        }
    }
}

}  // namespace sg
