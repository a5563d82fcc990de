// pull.cu — bottom-up (pull) BFS step for direction-optimising BFS (§3.4:
// "it is also possible to use both push and pull techniques as per Beamer et al. [5]").
//
// Every unvisited vertex v looks for a neighbour u in the input frontier (symmetric CSR: N(v)
// = its in-neighbours, reading C8).  An unvisited vertex's visited neighbours are all in the
// frontier (one at an earlier level would have reached v already), so any hit is a parent.
//   1. candidate test: u = fnbr[v], the neighbour of largest degree among v's first arcs
//      (graph load, frontier.cu): one bit test on the 2LB layer 1, no row_ptr / col_idx access.
//      In the large scale-free frontiers where the policy pulls, the hubs are in the frontier
//      and most vertices end here.
//   2. a vertex whose candidate missed scans N(v) until its first frontier neighbour.
// Mapping: one thread per quad of 4 consecutive vertices (16 threads = one 64-bit visited word),
// no loop in the common path: the thread reads the visited word and, if one of its vertices is
// unvisited, their 4 candidates with one 16-B load, then tests them (the only random reads, on
// a 2 MB bitmap that stays in L2).  The 16 threads of a word OR their found bits together
// (half-warp reduction).  The step writes its own output (no k_bfs_diff pass after a pull): the
// thread adds n_f / m_f of the vertices it found (degree codes, one 4-B load) and stores the
// levels of the word's new vertices lane16 + 16 i (64-B runs per store); the half-warp's first
// thread writes the output word (zero or not) and the new bits to visited and vis_old.  A CTA
// takes a whole layer-2 word, so it writes that word and appends its words to the output list
// itself, and the last CTA decides the next superstep (bfsstep.cuh).  The step is a streaming
// pass over the visited bitmap and fnbr with enough independent threads in flight to cover the
// latency of the dependent bit test.  Output identical to a push step from the same state.
// Late pull steps leave a few unvisited vertices per word, and the quad rounds become
// issue-bound (every warp runs the whole round for its one or two unvisited lanes).  So each
// CTA first reads the 64 visited words of its layer-2 word: none unvisited -> 64 zero output
// words; at most SG_PULL_WORD_MAX unvisited in every word -> word mode (a thread per layer-1
// word walks its unvisited vertices, SG_PULL_WORD_BATCH candidate tests in flight); else the
// quad rounds, where a warp whose two words are fully visited skips without loading them.
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"
#include "bfsstep.cuh"
#include "pullw.cuh"

namespace sg {

#ifndef SG_PULL_THREADS
#define SG_PULL_THREADS 256
#endif
constexpr int PULL_THREADS = SG_PULL_THREADS;   // 128, 256, 512 or 1024
constexpr int PULL_ROUNDS = 1024 / PULL_THREADS;
#ifndef SG_PULL_ARCS
#define SG_PULL_ARCS 2
#endif
constexpr int PULL_ARCS = SG_PULL_ARCS;
#ifndef SG_PULL_WAVES
#define SG_PULL_WAVES 16   // CTAs per SM in the grid (x 148)
#endif   // arcs in flight per step of a list scan

#ifndef SG_PULL_PF
#define SG_PULL_PF 0   // 1: load the next round's visited word one round ahead
#endif
#ifndef SG_PULL_WSKIP
#define SG_PULL_WSKIP 1   // 1: per layer-2 word mask of fully visited layer-1 words (skip without loads)
#endif
#ifndef SG_PULL_WORD_MAX
#define SG_PULL_WORD_MAX 16   // word mode when no layer-1 word of the layer-2 word has more unvisited
#endif                       // vertices than this (0: off; needs SG_PULL_WSKIP)
#ifndef SG_PULL_WORD_BATCH
#define SG_PULL_WORD_BATCH 4   // word mode: vertices whose candidate tests are in flight together
#endif
#if SG_PULL_PF && SG_PULL_WSKIP
#error "SG_PULL_PF assumes every round loads its visited word: build it with SG_PULL_WSKIP=0"
#endif
#ifndef SG_PULL_COUNT_SCANS
#define SG_PULL_COUNT_SCANS 1   // count list-scanned vertices (16 B of row_ptr each in the roofline bytes)
#endif
// Miss queue of the quad rounds (SG_PULL_QUEUE=1): a vertex whose candidate missed is not scanned
// by its own thread (a quad's up to 4 misses, 2 arcs per dependent round trip each, serialised on
// one thread: long-scoreboard 13 on the hub-heavy level-2 pulls, profiles/r02h_ncu_full.txt) but
// appended to a CTA queue in shared memory; after the 4 rounds the CTA drains it: stage A gives
// each queued vertex a thread for its first SG_PULLQ_SHORT arcs, all loaded and probed together
// (row bounds -> arcs -> probes: 3 round trips); rows still open go to stage B, a warp per row,
// 64 arcs per round.  Found bits gather in the layer-2 word's 64 output words in shared memory,
// written once at the end.  Same set of new vertices as the per-thread scan (any frontier
// neighbour); only the number of arcs inspected differs (stage A probes a batch past the hit).
#ifndef SG_PULL_QUEUE
#define SG_PULL_QUEUE 1
#endif
#ifndef SG_PULLQ_SHORT
#define SG_PULLQ_SHORT 8
#endif
constexpr int PQ_CAP = 4096;    // a layer-2 word has 4,096 vertices: the queue never overflows
#ifndef SG_PULLQ_RB
#define SG_PULLQ_RB 1   // quad rounds whose loads are issued together (1, 2 or 4 with 256 threads)
#endif
constexpr int PQ_RB = SG_PULLQ_RB;
#ifndef SG_PULLQ2_CAP
#define SG_PULLQ2_CAP 1024
#endif
constexpr int PQ2_CAP = SG_PULLQ2_CAP;   // open rows after stage A (overflow: the thread scans the rest)
#ifndef SG_PULL_MINB   // resident CTAs per SM the registers are sized for (queue: 40 registers, 6 CTAs
#define SG_PULL_MINB (SG_PULL_QUEUE ? 6 : 8)   // measured best: 3.37 vs 3.77 ms pull class at 8)
#endif
#if SG_PULL_QUEUE && !SG_PULL_WSKIP
#error "SG_PULL_QUEUE needs SG_PULL_WSKIP (the prologue's visited words)"
#endif
// list scan of v: true iff some u in N(v) is in the input frontier (stops at the first hit);
// PULL_ARCS arcs in flight per step, `arcs` counts the arcs tested
__device__ __forceinline__ bool pull_scan(const GraphView &g, const uint32_t *__restrict__ in32, int64_t v,
                                          unsigned long long &arcs) {
    int64_t rr = __ldg(g.rp + v);
    const int64_t e = __ldg(g.rp + v + 1);
    bool hit = false;
    while (rr < e && !hit) {
        int32_t u[PULL_ARCS];
        uint32_t y[PULL_ARCS];
#pragma unroll
        for (int j = 0; j < PULL_ARCS; j++) u[j] = rr + j < e ? __ldg(g.col + rr + j) : -1;
#pragma unroll
        for (int j = 0; j < PULL_ARCS; j++) y[j] = u[j] >= 0 ? __ldg(in32 + (u[j] >> 5)) : 0u;
#pragma unroll
        for (int j = 0; j < PULL_ARCS; j++) {
            if (!hit && u[j] >= 0) {
                arcs++;
                hit = (y[j] >> (u[j] & 31)) & 1u;
            }
        }
        rr += PULL_ARCS;
    }
    return hit;
}

#if SG_PULL_QUEUE
// Drain the CTA's miss queue (whole CTA; starts and ends with a barrier).  Found vertices: bit in
// s_found32 (64 output words as 128 u32 halves), level, n_f / m_f.
__device__ __forceinline__ void pullq_drain(const GraphView &g, const uint32_t *__restrict__ in32, const int32_t *s_q,
                                            uint32_t qn, int32_t *s_q2, uint32_t *s_q2n, uint32_t *s_found32,
                                            uint32_t *lvl, uint32_t nx, const uint32_t *s_lut, unsigned long long &nf,
                                            unsigned long long &mf, unsigned long long &arcs) {
    constexpr int S = SG_PULLQ_SHORT;
    auto mark = [&](int32_t v) {
        atomicOr(s_found32 + (((v >> 6) & 63) * 2 + ((v >> 5) & 1)), 1u << (v & 31));
        lvl[v] = nx;
        nf++;
        mf += s_lut[__ldg(g.deg8 + v)];
    };
    // stage A: a thread per queued vertex, its first S arcs in flight together
    for (uint32_t i = threadIdx.x; i < qn; i += blockDim.x) {
        const int32_t v = s_q[i];
        const int64_t r = __ldg(g.rp + v), e = __ldg(g.rp + v + 1);
        int32_t u[S];
        uint32_t y[S];
#pragma unroll
        for (int j = 0; j < S; j++) u[j] = r + j < e ? __ldg(g.col + r + j) : -1;
#pragma unroll
        for (int j = 0; j < S; j++) y[j] = u[j] >= 0 ? __ldg(in32 + (u[j] >> 5)) : 0u;
        int hit = -1;
#pragma unroll
        for (int j = S - 1; j >= 0; j--)
            if (u[j] >= 0 && ((y[j] >> (u[j] & 31)) & 1u)) hit = j;
        if (hit >= 0) {
            arcs += (unsigned long long)(hit + 1);
            mark(v);
        } else {
            arcs += (unsigned long long)min((int64_t)S, e - r);
            if (r + S < e) {
                const uint32_t p = atomicAdd(s_q2n, 1u);
                if (p < (uint32_t)PQ2_CAP) {
                    s_q2[p] = v;
                } else {   // stage-B queue full: scan the rest here
                    bool h = false;
                    for (int64_t k = r + S; k < e && !h; k++) {
                        const int32_t uu = __ldg(g.col + k);
                        arcs++;
                        h = (__ldg(in32 + (uu >> 5)) >> (uu & 31)) & 1u;
                    }
                    if (h) mark(v);
                }
            }
        }
    }
    __syncthreads();
    // stage B: a warp per open row, 64 arcs per round (2 per lane in flight)
    const uint32_t q2n = min(*s_q2n, (uint32_t)PQ2_CAP);
    const int lane = lane_id(), wid = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    for (uint32_t j = wid; j < q2n; j += nwarp) {
        const int32_t v = s_q2[j];
        const int64_t s = __ldg(g.rp + v) + S, e = __ldg(g.rp + v + 1);
        bool hit = false;
        for (int64_t r = s; r < e && !hit; r += 64) {
            const int64_t k0 = r + lane, k1 = r + 32 + lane;
            const int32_t u0 = k0 < e ? __ldg(g.col + k0) : -1, u1 = k1 < e ? __ldg(g.col + k1) : -1;
            const uint32_t y0 = u0 >= 0 ? __ldg(in32 + (u0 >> 5)) : 0u, y1 = u1 >= 0 ? __ldg(in32 + (u1 >> 5)) : 0u;
            const uint32_t b0 = __ballot_sync(0xffffffffu, u0 >= 0 && ((y0 >> (u0 & 31)) & 1u));
            const uint32_t b1 = __ballot_sync(0xffffffffu, u1 >= 0 && ((y1 >> (u1 & 31)) & 1u));
            if (lane == 0)
                arcs += (unsigned long long)(b0 ? __ffs(b0) : b1 ? 32 + __ffs(b1) : (int)min((int64_t)64, e - r));
            hit = (b0 | b1) != 0u;
        }
        if (hit && lane == 0) mark(v);
    }
    __syncthreads();
}
#endif

template <bool P>
__global__ void __launch_bounds__(PULL_THREADS, SG_PULL_MINB)
k_pull_bfs(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *__restrict__ visited, DevStats *st,
           BfsOut o) {
    __shared__ uint64_t s_wm[PULL_THREADS / 32], s_S[1];
    __shared__ uint32_t s_base[1 + SG_MAX_RANKS], s_lut[256];
#if SG_PULL_WSKIP
    __shared__ uint32_t s_full[2][2], s_mx[2][2];   // double-buffered by iteration parity (no barrier at reuse)
    int par = 0;
#endif
#if SG_PULL_QUEUE
    __shared__ uint32_t s_found32[128];   // the layer-2 word's 64 output words (u32 halves)
    __shared__ int32_t s_q[PQ_CAP], s_q2[PQ2_CAP];
    __shared__ uint32_t s_qn, s_q2n;
#endif
    if (o.ctrl ? o.ctrl->pull_warp[o.half] : o.pull_warp) return;   // late pull: k_pull_bfs_w takes it
    deg8_lut_init(s_lut);
    __syncthreads();
    uint32_t *const lvl = o.level_pp ? *o.level_pp : o.level;
    const uint32_t nx = o.next_ptr ? *o.next_ptr : o.next;
    unsigned long long nf = 0, mf = 0, arcs = 0;
    uint32_t scans = 0;
    const int lane = lane_id(), wid = threadIdx.x >> 5;
    const uint32_t *in32 = reinterpret_cast<const uint32_t *>(in_bits);
    const int64_t nq = g.nw1 * 16;
    const uint32_t half = (lane < 16) ? 0x0000ffffu : 0xffff0000u;
    // a CTA takes one layer-2 word (64 layer-1 words = 1,024 quads) in 4 rounds of 256 quads
    // the next round's visited word is loaded one round ahead (it does not depend on this round)
    auto vis_at = [&](int64_t qd) -> uint64_t { return qd < nq ? visited[qd >> 4] : ~0ull; };
#if SG_PULL_PF
    uint64_t vis_next = vis_at((int64_t)blockIdx.x * 1024 + threadIdx.x);
#endif
    // owned layer-2 words only (1-D partition; single GPU: all of them)
    for (int64_t sw = g.w2_lo + blockIdx.x; sw < g.w2_hi; sw += gridDim.x) {
        uint64_t wm = 0;   // the warp's changed words within the layer-2 word
#if SG_PULL_WSKIP
        // bit i of `full`: layer-1 word sw*64+i has no unvisited vertex (or lies past the end).
        // A layer-2 word with no unvisited vertex writes its 64 zero output words and is done;
        // otherwise a warp whose two words are full skips its round without loading them.
        uint64_t my_vis = ~0ull, my_unv = 0ull;   // threads < 64: layer-1 word sw*64+threadIdx.x
#if SG_PULL_QUEUE
        // (the previous layer-2 word's last reads of these ended at bfs_emit_words' barrier)
        if (threadIdx.x < 128) s_found32[threadIdx.x] = 0u;
        if (threadIdx.x == 0) {
            s_qn = 0u;
            s_q2n = 0u;
        }
#endif
        if (threadIdx.x < 64) {
            const int64_t w = sw * 64 + threadIdx.x;
            if (w < g.nw1) {
                const int64_t rem = g.n - w * 64;
                const uint64_t valid = rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
                my_vis = visited[w];
                my_unv = ~my_vis & valid;
            }
            const uint32_t b = __ballot_sync(0xffffffffu, my_unv == 0ull);
            const uint32_t mx = __reduce_max_sync(0xffffffffu, (uint32_t)__popcll(my_unv));
            if (lane == 0) {
                s_full[par][wid] = b;
                s_mx[par][wid] = mx;
            }
        }
        __syncthreads();
        const uint64_t full = (uint64_t)s_full[par][0] | ((uint64_t)s_full[par][1] << 32);
        const uint32_t mxw = max(s_mx[par][0], s_mx[par][1]);
        par ^= 1;
        if (full == ~0ull) {
            if (threadIdx.x < 64 && sw * 64 + threadIdx.x < g.nw1) xstore<P>(o.x, o.out_bits + sw * 64 + threadIdx.x, 0ull);
            if (threadIdx.x == 0) xstore<P>(o.x, o.out_summ + sw, 0ull);
            continue;
        }
#if SG_PULL_WORD_MAX > 0
        if (mxw <= (uint32_t)o.word_max) {
            // word mode (late pull steps: a few unvisited vertices per word): thread t < 64 owns
            // layer-1 word sw*64+t and walks its unvisited vertices one by one (candidate test,
            // then the list scan), so the CTA spends 2 warps instead of 32 quad rounds on it.
            // Same tests in the same order per vertex as the quad mode: identical output / stats.
            if (threadIdx.x < 64) {
                const int64_t w = sw * 64 + threadIdx.x;
                uint64_t nbw = 0;
                // SG_PULL_WORD_BATCH vertices per pass: their candidates and frontier bits are loaded together
                for (uint64_t m = my_unv; m;) {
                    int b[SG_PULL_WORD_BATCH];
                    int32_t c[SG_PULL_WORD_BATCH];
                    uint32_t x[SG_PULL_WORD_BATCH];
#pragma unroll
                    for (int k = 0; k < SG_PULL_WORD_BATCH; k++) {
                        b[k] = m ? __ffsll((long long)m) - 1 : -1;
                        m &= m - 1;
                    }
#pragma unroll
                    for (int k = 0; k < SG_PULL_WORD_BATCH; k++) c[k] = b[k] >= 0 ? __ldg(g.fnbr + w * 64 + b[k]) : -1;
#pragma unroll
                    for (int k = 0; k < SG_PULL_WORD_BATCH; k++) x[k] = c[k] >= 0 ? __ldg(in32 + (c[k] >> 5)) : 0u;
#pragma unroll
                    for (int k = 0; k < SG_PULL_WORD_BATCH; k++) {
                        if (b[k] < 0) continue;
                        bool hit = false;
                        if (c[k] >= 0) {
                            arcs++;
                            hit = (x[k] >> (c[k] & 31)) & 1u;
                        }
                        if (!hit) {
                            if (SG_PULL_COUNT_SCANS) scans++;
                            hit = pull_scan(g, in32, w * 64 + b[k], arcs);
                        }
                        if (hit) nbw |= 1ull << b[k];
                    }
                }
                if (w < g.nw1) {
                    xstore<P>(o.x, o.out_bits + w, nbw);
                    if (nbw) {
                        visited[w] = my_vis | nbw;
                        o.vis_old[w] = my_vis | nbw;
                        nf += __popcll(nbw);
                        for (uint64_t m = nbw; m; m &= m - 1) {
                            const int64_t v = w * 64 + (__ffsll((long long)m) - 1);
                            lvl[v] = nx;
                            mf += s_lut[__ldg(g.deg8 + v)];
                        }
                    }
                }
                const uint32_t b = __ballot_sync(0xffffffffu, nbw != 0ull);
                if (lane == 0) s_wm[wid] = b;
            }
            __syncthreads();
            if (threadIdx.x == 0) s_S[0] = s_wm[0] | (s_wm[1] << 32);
            __syncthreads();
            bfs_emit_words<P>(o, g.w2_hi, sw, s_S, 1, s_base);
            continue;
        }
#endif
#endif
#if SG_PULL_QUEUE
        // quad rounds, SG_PULLQ_RB of them at once (all their candidate loads and probes in
        // flight together: the rounds are independent now that misses are queued); misses
        // queued with one shared atomic per warp and batch
#pragma unroll 1
        for (int rb = 0; rb < PULL_ROUNDS; rb += PQ_RB) {
            uint32_t unv[PQ_RB], codes[PQ_RB], x[PQ_RB][4];
            int4 c4[PQ_RB];
            int64_t w[PQ_RB];
            bool act[PQ_RB];
#pragma unroll
            for (int j = 0; j < PQ_RB; j++) {
                const int r = rb + j;
                const int64_t qd = sw * 1024 + r * PULL_THREADS + threadIdx.x;
                w[j] = qd >> 4;
                const int64_t v0 = w[j] * 64 + (qd & 15) * 4;
                const int64_t rem = g.n - v0;
                const uint32_t valid = qd >= nq ? 0u : rem >= 4 ? 0xfu : (rem > 0 ? (1u << rem) - 1u : 0u);
                const bool skip = ((full >> (r * (PULL_THREADS / 16) + wid * 2)) & 3ull) == 3ull;
                unv[j] = skip ? 0u : (uint32_t)(~vis_at(qd) >> ((qd & 15) * 4)) & valid;
                act[j] = __any_sync(0xffffffffu, unv[j] != 0u);
                c4[j] = make_int4(-1, -1, -1, -1);
                codes[j] = 0u;
                if (unv[j]) {
                    c4[j] = __ldg(reinterpret_cast<const int4 *>(g.fnbr + v0));
                    codes[j] = __ldg(reinterpret_cast<const uint32_t *>(g.deg8 + v0));
                }
            }
#pragma unroll
            for (int j = 0; j < PQ_RB; j++) {
                const int32_t c[4] = {c4[j].x, c4[j].y, c4[j].z, c4[j].w};
#pragma unroll
                for (int k = 0; k < 4; k++) x[j][k] = ((unv[j] >> k) & 1u) && c[k] >= 0 ? __ldg(in32 + (c[k] >> 5)) : 0u;
            }
            uint32_t found[PQ_RB], miss[PQ_RB];
            int cnt = 0;
#pragma unroll
            for (int j = 0; j < PQ_RB; j++) {
                const int32_t c[4] = {c4[j].x, c4[j].y, c4[j].z, c4[j].w};
                found[j] = miss[j] = 0u;
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (!((unv[j] >> k) & 1u)) continue;
                    if (c[k] >= 0) {
                        arcs++;
                        if ((x[j][k] >> (c[k] & 31)) & 1u) {
                            found[j] |= 1u << k;
                            continue;
                        }
                    }
                    miss[j] |= 1u << k;
                }
                cnt += __popc(miss[j]);
            }
            const int incl = warp_inclusive_scan(cnt);
            const int tot = __shfl_sync(0xffffffffu, incl, 31);
            if (tot) {
                uint32_t qb = 0;
                if (lane == 31) qb = atomicAdd(&s_qn, (uint32_t)tot);
                qb = __shfl_sync(0xffffffffu, qb, 31);
                int pos = (int)qb + incl - cnt;
#pragma unroll
                for (int j = 0; j < PQ_RB; j++) {
                    const int32_t v0 = (int32_t)(w[j] * 64 + (lane & 15) * 4);
#pragma unroll
                    for (int k = 0; k < 4; k++)
                        if ((miss[j] >> k) & 1u) s_q[pos++] = v0 + k;
                }
                if (SG_PULL_COUNT_SCANS) scans += (uint32_t)cnt;
            }
#pragma unroll
            for (int j = 0; j < PQ_RB; j++) {
                if (!act[j]) continue;
                const int sh = (lane & 15) * 4;
                const uint64_t mine = (uint64_t)found[j] << sh;
                const uint32_t nlo = __reduce_or_sync(half, (uint32_t)mine), nhi = __reduce_or_sync(half, (uint32_t)(mine >> 32));
                if (found[j]) {
                    nf += __popc(found[j]);
                    mf += quad_mf(s_lut, codes[j], found[j]);
                }
                if (nlo | nhi) {   // candidate hits: level stores strided over the half-warp (64-B runs)
                    const uint64_t t = ((uint64_t)nhi << 32 | nlo) >> (lane & 15);
                    uint32_t *lw = lvl + w[j] * 64 + (lane & 15);
#pragma unroll
                    for (int i = 0; i < 4; i++)
                        if ((t >> (16 * i)) & 1u) lw[16 * i] = nx;
                    if ((lane & 15) == 0) {
                        const int wi = (int)(w[j] & 63);
                        s_found32[2 * wi] = nlo;
                        s_found32[2 * wi + 1] = nhi;
                    }
                }
            }
        }
        __syncthreads();
        if (s_qn) pullq_drain(g, in32, s_q, s_qn, s_q2, &s_q2n, s_found32, lvl, nx, s_lut, nf, mf, arcs);
        // output: the 64 words, visited / vis_old, the warp masks of changed words
        if (threadIdx.x < 64) {
            const int64_t w = sw * 64 + threadIdx.x;
            const uint64_t nb = (uint64_t)s_found32[2 * threadIdx.x] | ((uint64_t)s_found32[2 * threadIdx.x + 1] << 32);
            if (w < g.nw1) {
                xstore<P>(o.x, o.out_bits + w, nb);
                if (nb) {
                    visited[w] = my_vis | nb;
                    o.vis_old[w] = my_vis | nb;
                }
            }
            wm = (uint64_t)__ballot_sync(0xffffffffu, nb != 0ull) << (32 * wid);
        }
#else
#pragma unroll 1
        for (int r = 0; r < PULL_ROUNDS; r++) {
            const int64_t qd = sw * 1024 + r * PULL_THREADS + threadIdx.x;
            const bool ok = qd < nq;
            const int64_t w = qd >> 4;
#if SG_PULL_WSKIP
            if (((full >> (r * (PULL_THREADS / 16) + wid * 2)) & 3ull) == 3ull) {
                if ((lane & 15) == 0 && ok) xstore<P>(o.x, o.out_bits + w, 0ull);
                continue;
            }
#endif
            const int sh = (int)(qd & 15) * 4;
#if SG_PULL_PF
            const uint64_t vis = vis_next;
            vis_next = vis_at(r < PULL_ROUNDS - 1 ? qd + PULL_THREADS : (sw + gridDim.x) * 1024 + threadIdx.x);
#else
            const uint64_t vis = vis_at(qd);
#endif
            const int64_t v0 = w * 64 + sh;
            const int64_t rem = g.n - v0;
            const uint32_t valid = !ok ? 0u : rem >= 4 ? 0xfu : (rem > 0 ? (1u << rem) - 1u : 0u);
            const uint32_t unv = (uint32_t)(~vis >> sh) & valid;
            if (__all_sync(0xffffffffu, unv == 0u)) {   // the warp's two words are fully visited:
                if ((lane & 15) == 0 && ok) xstore<P>(o.x, o.out_bits + w, 0ull);   // no new vertices, no work
                continue;
            }
            uint32_t found = 0, codes = 0;
            if (unv) {
                const int4 c4 = __ldg(reinterpret_cast<const int4 *>(g.fnbr + v0));
                codes = __ldg(reinterpret_cast<const uint32_t *>(g.deg8 + v0));   // in flight with c4
                const int32_t c[4] = {c4.x, c4.y, c4.z, c4.w};
                uint32_t x[4];
#pragma unroll
                for (int k = 0; k < 4; k++) x[k] = ((unv >> k) & 1u) && c[k] >= 0 ? __ldg(in32 + (c[k] >> 5)) : 0u;
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (((unv >> k) & 1u) && c[k] >= 0) {
                        arcs++;
                        if ((x[k] >> (c[k] & 31)) & 1u) found |= 1u << k;
                    }
                }
                // 2. list scans of the vertices whose candidate missed
                for (uint32_t miss = unv & ~found; miss; miss &= miss - 1) {
                    const int k = __ffs(miss) - 1;
                    if (SG_PULL_COUNT_SCANS) scans++;
                    const bool hit = pull_scan(g, in32, v0 + k, arcs);
                    if (hit) found |= 1u << k;
                }
            }
            // the word's found bits: OR over the half-warp
            const uint64_t mine = (uint64_t)found << sh;
            const uint64_t nb = (uint64_t)__reduce_or_sync(half, (uint32_t)mine) |
                                ((uint64_t)__reduce_or_sync(half, (uint32_t)(mine >> 32)) << 32);
            if (found) {   // n_f / m_f of the vertices found here
                nf += __popc(found);
                mf += quad_mf(s_lut, codes, found);
            }
            if (nb) {   // level[] of the word's new vertices, strided over the half-warp (vertex
                        // 16 i + lane16): each store instruction writes 64 contiguous bytes
                const uint64_t t = nb >> (lane & 15);
                uint32_t *lw = lvl + w * 64 + (lane & 15);
#pragma unroll
                for (int i = 0; i < 4; i++)
                    if ((t >> (16 * i)) & 1u) lw[16 * i] = nx;
            }
            if ((lane & 15) == 0 && ok) {
                xstore<P>(o.x, o.out_bits + w, nb);   // every output word is written
                if (nb) {
                    visited[w] = vis | nb;
                    o.vis_old[w] = vis | nb;
                }
            }
            const uint32_t act = __ballot_sync(0xffffffffu, nb != 0ull && (lane & 15) == 0);
            wm |= (uint64_t)((act & 1u) | ((act >> 15) & 2u)) << (r * (PULL_THREADS / 16) + wid * 2);
        }
#endif
        if (lane == 0) s_wm[wid] = wm;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint64_t S = 0;
            for (int i = 0; i < PULL_THREADS / 32; i++) S |= s_wm[i];
            s_S[0] = S;
        }
        __syncthreads();
        bfs_emit_words<P>(o, g.w2_hi, sw, s_S, 1, s_base);
    }
    bfs_finish<P>(o, nf, mf, arcs, st, scans);
}

// Late pull steps (few unvisited vertices left): one warp per layer-2 word (pullw.cuh), no CTA
// barrier, misses drained cooperatively.  Runs iff ctrl->pull_warp (graph mode; both kernels are
// in the pull node and the other one returns at once) or o.pull_warp (host loop).
template <bool P>
__global__ void __launch_bounds__(256, 4)
k_pull_bfs_w(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *__restrict__ visited, DevStats *st,
             BfsOut o) {
    if (!(o.ctrl ? o.ctrl->pull_warp[o.half] : o.pull_warp)) return;
    __shared__ P2Warp s_w[8];
    __shared__ uint32_t s_lut[256];
    deg8_lut_init(s_lut);
    __syncthreads();
    uint32_t *const lvl = o.level_pp ? *o.level_pp : o.level;
    const uint32_t nx = o.next_ptr ? *o.next_ptr : o.next;
    const int wid = threadIdx.x >> 5;
    const uint32_t *in32 = reinterpret_cast<const uint32_t *>(in_bits);
    unsigned long long nf = 0, mf = 0, arcs = 0, scans = 0;
    const int64_t gwarp = (int64_t)blockIdx.x * 8 + wid, nwarps = (int64_t)gridDim.x * 8;
    for (int64_t sw = g.w2_lo + gwarp; sw < g.w2_hi; sw += nwarps)
        pull_l2_warp<P>(g, sw, in32, visited, o, s_w[wid], s_lut, lvl, nx, nf, mf, arcs, scans);
    bfs_finish<P>(o, nf, mf, arcs, st, scans);
}

void launch_pull_bfs(const GraphView &g, const uint64_t *in_bits, uint64_t *visited, DevStats *st, const BfsOut &o_in,
                     cudaStream_t s) {
    BfsOut o = o_in;
    {   // word-mode threshold of the CTA kernel: a runtime parameter (tests force 0 / 64)
        const char *wm = getenv("SG_PULL_WORD_MAX");
        o.word_max = wm ? atoi(wm) : SG_PULL_WORD_MAX;
    }
    // graph mode launches both kernels (the device-side decision picks one; with the late-pull rule
    // off, SG_PULL_WARP_FRAC=0, only the CTA kernel); the host loop launches one
    const char *fr = getenv("SG_PULL_WARP_FRAC");
    const bool both = o.ctrl != nullptr && !(fr && atoi(fr) == 0);
    if (both || !o.pull_warp) {
        // one CTA per layer-2 word in a grid-stride loop over SG_PULL_WAVES CTAs per SM
        int64_t blocks = g.w2_hi - g.w2_lo;
        if (blocks > num_sms() * SG_PULL_WAVES) blocks = num_sms() * SG_PULL_WAVES;
        if (blocks < 1) blocks = 1;
        note_launch();
        if (o.x.nranks > 1) k_pull_bfs<true><<<(int)blocks, PULL_THREADS, 0, s>>>(g, in_bits, visited, st, o);
        else k_pull_bfs<false><<<(int)blocks, PULL_THREADS, 0, s>>>(g, in_bits, visited, st, o);
    }
    if (both || (o.ctrl == nullptr && o.pull_warp)) {
        int64_t blocks = (g.w2_hi - g.w2_lo + 7) / 8;   // one warp per layer-2 word
        if (blocks > num_sms() * 4) blocks = num_sms() * 4;
        if (blocks < 1) blocks = 1;
        note_launch();
        if (o.x.nranks > 1) k_pull_bfs_w<true><<<(int)blocks, 256, 0, s>>>(g, in_bits, visited, st, o);
        else k_pull_bfs_w<false><<<(int)blocks, 256, 0, s>>>(g, in_bits, visited, st, o);
    }
}

}  // namespace sg
