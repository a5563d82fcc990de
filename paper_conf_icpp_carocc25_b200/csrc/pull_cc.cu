// pull_cc.cu — pull (bottom-up) label-propagation step for connected components.
//
// PAPER.md:161 §3.4: CC by label propagation (Stergiou et al. [29]), stopping when no label
// changes.  When most vertices are active (the first supersteps: every vertex starts in the
// frontier, advance::vertices P:137) the push step performs one atomicMin per improving arc; the
// pull step instead lets each vertex take the minimum over its neighbours' labels and write its
// own label once (no atomics), the direction-optimising idea of Beamer [5] applied to label
// propagation.  One warp owns one word (lane l: vertices 64w+l and 64w+32+l), so the output
// frontier word (vertices whose label decreased) is written without atomics.  The fixed point
// (component minimum, reading C13) is the same; tested bit-exact against union-find.
#include "common.cuh"
#include "kernels.h"

namespace sg {

constexpr int CCP_THREADS = 256;

__global__ void __launch_bounds__(CCP_THREADS)
k_pull_cc(GraphView g, int32_t *__restrict__ label, uint64_t *__restrict__ out_bits, uint64_t *__restrict__ out_summ,
          DevStats *st) {
    __shared__ unsigned long long s_arcs[CCP_THREADS / 32];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long arcs = 0;
    for (int64_t w = gw; w < g.nw1; w += nwarps) {
        const int64_t rem = g.n - w * 64;
        const uint64_t valid = rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
        int64_t sa, ea, sb, eb;
        word_bounds(g, w, valid, sa, ea, sb, eb);
        const int64_t va = w * 64 + lane, vb = va + 32;
        const bool act_a = (valid >> lane) & 1ull, act_b = (valid >> (lane + 32)) & 1ull;
        const int32_t own_a = act_a ? label[va] : 0x7fffffff, own_b = act_b ? label[vb] : 0x7fffffff;
        int32_t ma = own_a, mb = own_b;
        arcs += (unsigned long long)((ea - sa) + (eb - sb));
        // both rows in lock-step, 4 arcs each per step: 8 independent label loads in flight
        for (int64_t ia = sa, ib = sb; ia < ea || ib < eb; ia += 4, ib += 4) {
            int32_t c[8];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                c[k] = (ia + k < ea) ? __ldg(g.col + ia + k) : -1;
                c[4 + k] = (ib + k < eb) ? __ldg(g.col + ib + k) : -1;
            }
            int32_t l[8];
#pragma unroll
            for (int k = 0; k < 8; k++) l[k] = c[k] >= 0 ? label[c[k]] : 0x7fffffff;
#pragma unroll
            for (int k = 0; k < 4; k++) {
                ma = min(ma, l[k]);
                mb = min(mb, l[4 + k]);
            }
        }
        const bool ca = ma < own_a, cb = mb < own_b;
        if (ca) label[va] = ma;
        if (cb) label[vb] = mb;
        const uint64_t nb = (uint64_t)__ballot_sync(0xffffffffu, ca) | ((uint64_t)__ballot_sync(0xffffffffu, cb) << 32);
        if (nb && lane == 0) {
            out_bits[w] = nb;
            atomic_or_u64(out_summ + (w >> 6), 1ull << (w & 63));
        }
    }
    arcs = warp_sum(arcs);
    if (lane == 0) s_arcs[threadIdx.x >> 5] = arcs;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int i = 0; i < CCP_THREADS / 32; i++) t += s_arcs[i];
        if (t) atomicAdd(&st->arcs, t);
    }
}

void launch_pull_cc(const GraphView &g, int32_t *label, uint64_t *out_bits, uint64_t *out_summ, DevStats *st,
                    cudaStream_t s) {
    int64_t blocks = (g.nw1 * 32 + CCP_THREADS - 1) / CCP_THREADS;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_cc<<<(int)blocks, CCP_THREADS, 0, s>>>(g, label, out_bits, out_summ, st);
}

}  // namespace sg
