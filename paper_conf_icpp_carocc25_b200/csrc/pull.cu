// pull.cu — bottom-up (pull) BFS step for direction-optimising BFS (§3.4:
// "it is also possible to use both push and pull techniques as per Beamer et al. [5]").
//
// Every unvisited vertex v scans N(v) (symmetric CSR = its in-neighbours, reading C8) and
// stops at the first u that is in the input frontier (one bit test on the 2LB layer 1).
// One warp owns one 64-bit word of the visited bitmap (lane l: vertices 64w+l and 64w+32+l),
// so the new frontier word, the visited word and level[] are written without atomics; only
// the summary bit is an atomicOr.  The two vertices of a lane are scanned in lock-step (two
// independent load chains in flight per lane): the step is latency-bound, not bandwidth-bound.
// Output identical to a push step from the same state (tested).
#include "common.cuh"
#include "kernels.h"

namespace sg {

constexpr int PULL_THREADS = 256;
#ifndef SG_PULL_ARCS
#define SG_PULL_ARCS 2
#endif
#ifndef SG_PULL_MINB
#define SG_PULL_MINB 6
#endif
constexpr int PULL_ARCS = SG_PULL_ARCS;   // arcs per vertex per iteration

__global__ void __launch_bounds__(PULL_THREADS, SG_PULL_MINB)
k_pull_bfs(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *__restrict__ visited,
           uint64_t *__restrict__ out_bits, uint64_t *__restrict__ out_summ, uint32_t *__restrict__ level,
           uint32_t next, DevStats *st, const uint32_t *next_ptr, uint32_t *const *level_pp) {
    if (next_ptr) next = *next_ptr;
    if (level_pp) level = *level_pp;
    __shared__ unsigned long long s_arcs[PULL_THREADS / 32];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long arcs = 0;
    for (int64_t w = gw; w < g.nw1; w += nwarps) {
        const uint64_t vis = visited[w];
        const int64_t rem = g.n - w * 64;
        const uint64_t valid = rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
        const uint64_t unv = ~vis & valid;
        if (!unv) continue;
        int64_t s[2], e[2];
        word_bounds(g, w, unv, s[0], e[0], s[1], e[1]);
        bool found[2] = {false, false};
        // lock-step scan of both vertices' lists until each hits a frontier neighbour
        while (s[0] < e[0] || s[1] < e[1]) {
            int32_t c[2][PULL_ARCS];
#pragma unroll
            for (int k = 0; k < 2; k++)
#pragma unroll
                for (int j = 0; j < PULL_ARCS; j++) c[k][j] = (s[k] + j < e[k]) ? __ldg(g.col + s[k] + j) : -1;
            uint64_t x[2][PULL_ARCS];
#pragma unroll
            for (int k = 0; k < 2; k++)
#pragma unroll
                for (int j = 0; j < PULL_ARCS; j++) x[k][j] = c[k][j] >= 0 ? __ldg(in_bits + (c[k][j] >> 6)) : 0ull;
#pragma unroll
            for (int k = 0; k < 2; k++) {
                if (s[k] >= e[k]) continue;
                int used = 0;
                bool hit = false;
#pragma unroll
                for (int j = 0; j < PULL_ARCS; j++) {
                    if (!hit && c[k][j] >= 0) {
                        used++;
                        hit = (x[k][j] >> (c[k][j] & 63)) & 1ull;
                    }
                }
                arcs += used;
                if (hit) {
                    found[k] = true;
                    s[k] = e[k];
                } else {
                    s[k] += PULL_ARCS;
                }
            }
        }
        const uint32_t ba = __ballot_sync(0xffffffffu, found[0]), bb = __ballot_sync(0xffffffffu, found[1]);
        const uint64_t nb = (uint64_t)ba | ((uint64_t)bb << 32);
        if (found[0]) level[w * 64 + lane] = next;
        if (found[1]) level[w * 64 + 32 + lane] = next;
        if (nb && lane == 0) {
            out_bits[w] = nb;
            visited[w] = vis | nb;
            atomic_or_u64(out_summ + (w >> 6), 1ull << (w & 63));
        }
    }
    arcs = warp_sum(arcs);
    if (lane == 0) s_arcs[threadIdx.x >> 5] = arcs;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int i = 0; i < PULL_THREADS / 32; i++) t += s_arcs[i];
        if (t) atomicAdd(&st->arcs, t);
    }
}

void launch_pull_bfs(const GraphView &g, const uint64_t *in_bits, uint64_t *visited, uint64_t *out_bits,
                     uint64_t *out_summ, uint32_t *level, uint32_t next, DevStats *st, cudaStream_t s,
                     const uint32_t *next_ptr, uint32_t *const *level_pp) {
    int64_t blocks = (g.nw1 * 32 + PULL_THREADS - 1) / PULL_THREADS;
    if (blocks > 148 * SG_PULL_MINB) blocks = 148 * SG_PULL_MINB;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_bfs<<<(int)blocks, PULL_THREADS, 0, s>>>(g, in_bits, visited, out_bits, out_summ, level, next, st, next_ptr,
                                                    level_pp);
}

}  // namespace sg
