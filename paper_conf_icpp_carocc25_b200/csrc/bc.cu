// bc.cu — Brandes betweenness centrality helpers (§3.4 "Brandes' formulation
// ... traversing the graph first forward, then backward, from a source vertex"; ref [9]).
//
// Forward sigma runs through the push advance (FnBcSigma).  Path counts overflow fp64 on
// high-diameter graphs (reading C20), so each BFS level d carries a power-of-two exponent
// E[d]: true sigma(v) = sigma[v] * 2^E[level(v)].  After level d+1 is complete its values are
// multiplied by 2^-k (exact) with k = floor(log2 max sigma over the level), E[d+1] = E[d] + k.
// The backward sweep is pull-style and atomic-free: for each v at level d (BFS stack order),
//   delta[v] = 2^(E[d]-E[d+1]) * sigma[v] * sum_{w in N(v), level[w] = d+1} (1 + delta[w]) / sigma[w]
// and bc[v] += delta[v] for v != s.
#include "common.cuh"
#include "kernels.h"

namespace sg {

__global__ void k_bc_level_max(const double *__restrict__ sigma, const uint64_t *__restrict__ bits,
                               const uint32_t *__restrict__ offsets, const DevStats *st,
                               unsigned long long *max_bits) {
    const uint32_t count = (uint32_t)st->count;
    unsigned long long mx = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += stride) {
        const uint32_t w = offsets[i];
        uint64_t x = bits[w];
        while (x) {
            const int b = __ffsll((long long)x) - 1;
            x &= x - 1;
            const unsigned long long vb = (unsigned long long)__double_as_longlong(sigma[(int64_t)w * 64 + b]);
            mx = vb > mx ? vb : mx;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long y = __shfl_xor_sync(0xffffffffu, mx, o);
        mx = y > mx ? y : mx;
    }
    if (lane_id() == 0 && mx) atomicMax(max_bits, mx);
}

// Scale level (level_idx) by 2^-k, record E[level_idx] and append the level to the BFS stack
// (stack == NULL: no stack, the user-driven advance(SG_FN_BC_SIGMA) path).
__global__ void k_bc_scale_stack(double *__restrict__ sigma, const uint64_t *__restrict__ bits,
                                 const uint32_t *__restrict__ offsets, const DevStats *st,
                                 const unsigned long long *max_bits, int32_t *exp_of_level, uint32_t level_idx,
                                 int32_t *__restrict__ stack, unsigned long long *stack_top,
                                 unsigned long long *underflow) {
    const uint32_t count = (uint32_t)st->count;
    const unsigned long long mb = *max_bits;
    const int k = mb ? (int)((mb >> 52) & 0x7ff) - 1023 : 0;      // max is a normal number >= 2^-1022
    if (blockIdx.x == 0 && threadIdx.x == 0) exp_of_level[level_idx] = exp_of_level[level_idx - 1] + k;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += stride) {
        const uint32_t w = offsets[i];
        uint64_t x = bits[w];
        unsigned long long pos = stack ? atomicAdd(stack_top, (unsigned long long)__popcll(x)) : 0ull;
        while (x) {
            const int b = __ffsll((long long)x) - 1;
            x &= x - 1;
            const int64_t v = (int64_t)w * 64 + b;
            const double sv = ldexp(sigma[v], -k);
            if (sv < 2.2250738585072014e-308) atomicAdd(underflow, 1ull);   // subnormal: precision lost
            sigma[v] = sv;
            if (stack) stack[pos++] = (int32_t)v;
        }
    }
}

__global__ void k_bc_backward(GraphView g, const int32_t *__restrict__ stack, int64_t lo, int64_t hi,
                              const uint32_t *__restrict__ level, const double *__restrict__ sigma,
                              double *__restrict__ delta, const int32_t *__restrict__ exp_of_level, uint32_t d,
                              double *__restrict__ bc, int32_t src) {
    const int ediff = exp_of_level[d] - exp_of_level[d + 1];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hi; i += stride) {
        const int32_t v = stack[i];
        double acc = 0.0;
        const int64_t e1 = __ldg(g.rp + v + 1);
        for (int64_t e = __ldg(g.rp + v); e < e1; e++) {
            const int32_t w = __ldg(g.col + e);
            if (level[w] == d + 1) acc += (1.0 + delta[w]) / sigma[w];
        }
        const double dv = ldexp(sigma[v] * acc, ediff);
        delta[v] = dv;
        if (v != src) bc[v] += dv;
    }
}

static int grid_for(int64_t items, int threads, int max_blocks) {
    int64_t b = (items + threads - 1) / threads;
    if (b < 1) b = 1;
    if (b > max_blocks) b = max_blocks;
    return (int)b;
}

void launch_bc_level_max(const double *sigma, const uint64_t *bits, const uint32_t *offsets, const DevStats *st,
                         int64_t max_words, unsigned long long *max_bits, cudaStream_t s) {
    note_launch();
    k_bc_level_max<<<grid_for(max_words, 256, num_sms() * 4), 256, 0, s>>>(sigma, bits, offsets, st, max_bits);
}
void launch_bc_level_scale_and_stack(double *sigma, const uint64_t *bits, const uint32_t *offsets,
                                     const DevStats *st, int64_t max_words, const unsigned long long *max_bits,
                                     int32_t *exp_of_level, uint32_t level_idx, int32_t *stack,
                                     unsigned long long *stack_top, unsigned long long *underflow, cudaStream_t s) {
    note_launch();
    k_bc_scale_stack<<<grid_for(max_words, 256, num_sms() * 4), 256, 0, s>>>(sigma, bits, offsets, st, max_bits,
                                                                        exp_of_level, level_idx, stack, stack_top,
                                                                        underflow);
}
void launch_bc_backward_level(const GraphView &g, const int32_t *stack, int64_t lo, int64_t hi, const uint32_t *level,
                              const double *sigma, double *delta, const int32_t *exp_of_level, uint32_t d,
                              double *bc, int32_t src, cudaStream_t s) {
    if (hi <= lo) return;
    note_launch();
    k_bc_backward<<<grid_for(hi - lo, 256, num_sms() * 8), 256, 0, s>>>(g, stack, lo, hi, level, sigma, delta,
                                                                   exp_of_level, d, bc, src);
}

}  // namespace sg
