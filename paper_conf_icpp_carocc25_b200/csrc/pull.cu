// pull.cu — bottom-up (pull) BFS step for direction-optimising BFS (§3.4:
// "it is also possible to use both push and pull techniques as per Beamer et al. [5]").
//
// Every unvisited vertex v scans N(v) (symmetric CSR = its in-neighbours, reading C8) and
// stops at the first u that is in the input frontier (one bit test on the 2LB layer 1).
// One warp owns one 64-bit word of the visited bitmap, so the new frontier word, the visited
// word and level[] are written without atomics; only the summary bit is an atomicOr.
// Output identical to a push step from the same state (tested).
#include "common.cuh"
#include "kernels.h"

namespace sg {

constexpr int PULL_THREADS = 256;

// scan N(u) = col[s..e) four arcs at a time (4 independent loads + 4 bit probes in flight)
__device__ __forceinline__ bool pull_scan(const GraphView &g, const uint64_t *__restrict__ in_bits, int64_t s,
                                          int64_t e, unsigned long long &arcs) {
    for (int64_t i = s; i < e; i += 4) {
        int32_t c[4];
#pragma unroll
        for (int k = 0; k < 4; k++) c[k] = (i + k < e) ? __ldg(g.col + i + k) : -1;
        uint64_t x[4];
#pragma unroll
        for (int k = 0; k < 4; k++) x[k] = c[k] >= 0 ? __ldg(in_bits + (c[k] >> 6)) : 0ull;
        bool hit = false;
        int used = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            if (!hit && c[k] >= 0) {
                used++;
                hit = (x[k] >> (c[k] & 63)) & 1ull;
            }
        }
        arcs += used;
        if (hit) return true;
    }
    return false;
}

__global__ void __launch_bounds__(PULL_THREADS)
k_pull_bfs(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *__restrict__ visited,
           uint64_t *__restrict__ out_bits, uint64_t *__restrict__ out_summ, uint32_t *__restrict__ level,
           uint32_t next, DevStats *st) {
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
        int64_t sa, ea, sb, eb;
        word_bounds(g, w, unv, sa, ea, sb, eb);
        const bool fa = (ea > sa) && pull_scan(g, in_bits, sa, ea, arcs);
        const bool fb = (eb > sb) && pull_scan(g, in_bits, sb, eb, arcs);
        const uint32_t ba = __ballot_sync(0xffffffffu, fa), bb = __ballot_sync(0xffffffffu, fb);
        const uint64_t nb = (uint64_t)ba | ((uint64_t)bb << 32);
        if (fa) level[w * 64 + lane] = next;
        if (fb) level[w * 64 + 32 + lane] = next;
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
                     uint64_t *out_summ, uint32_t *level, uint32_t next, DevStats *st, cudaStream_t s) {
    int64_t blocks = (g.nw1 * 32 + PULL_THREADS - 1) / PULL_THREADS;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    k_pull_bfs<<<(int)blocks, PULL_THREADS, 0, s>>>(g, in_bits, visited, out_bits, out_summ, level, next, st);
}

}  // namespace sg
