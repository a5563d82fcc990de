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
#include "common.cuh"
#include "kernels.h"
#include "bfsstep.cuh"

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
#ifndef SG_PULL_MINB
#define SG_PULL_MINB 8
#endif
__global__ void __launch_bounds__(PULL_THREADS, SG_PULL_MINB)
k_pull_bfs(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *__restrict__ visited, DevStats *st,
           BfsOut o) {
    __shared__ uint64_t s_wm[PULL_THREADS / 32], s_S[1];
    __shared__ uint32_t s_base, s_lut[256];
    deg8_lut_init(s_lut);
    __syncthreads();
    uint32_t *const lvl = o.level_pp ? *o.level_pp : o.level;
    const uint32_t nx = o.next_ptr ? *o.next_ptr : o.next;
    unsigned long long nf = 0, mf = 0, arcs = 0;
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
    for (int64_t sw = blockIdx.x; sw < g.nw2; sw += gridDim.x) {
        uint64_t wm = 0;   // the warp's changed words within the layer-2 word
#pragma unroll 1
        for (int r = 0; r < PULL_ROUNDS; r++) {
            const int64_t qd = sw * 1024 + r * PULL_THREADS + threadIdx.x;
            const bool ok = qd < nq;
            const int64_t w = qd >> 4;
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
                if ((lane & 15) == 0 && ok) o.out_bits[w] = 0ull;   // no new vertices, no work
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
                    int64_t rr = __ldg(g.rp + v0 + k);
                    const int64_t e = __ldg(g.rp + v0 + k + 1);
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
                o.out_bits[w] = nb;   // every output word is written
                if (nb) {
                    visited[w] = vis | nb;
                    o.vis_old[w] = vis | nb;
                }
            }
            const uint32_t act = __ballot_sync(0xffffffffu, nb != 0ull && (lane & 15) == 0);
            wm |= (uint64_t)((act & 1u) | ((act >> 15) & 2u)) << (r * (PULL_THREADS / 16) + wid * 2);
        }
        if (lane == 0) s_wm[wid] = wm;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint64_t S = 0;
            for (int i = 0; i < PULL_THREADS / 32; i++) S |= s_wm[i];
            s_S[0] = S;
        }
        __syncthreads();
        bfs_emit_words(o, g.nw2, sw, s_S, 1, &s_base);
    }
    bfs_finish(o, nf, mf, arcs, st);
}

void launch_pull_bfs(const GraphView &g, const uint64_t *in_bits, uint64_t *visited, DevStats *st, const BfsOut &o,
                     cudaStream_t s) {
    // one CTA per layer-2 word in a grid-stride loop over SG_PULL_WAVES CTAs per SM
    int64_t blocks = g.nw2;
    if (blocks > 148 * SG_PULL_WAVES) blocks = 148 * SG_PULL_WAVES;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_bfs<<<(int)blocks, PULL_THREADS, 0, s>>>(g, in_bits, visited, st, o);
}

}  // namespace sg
