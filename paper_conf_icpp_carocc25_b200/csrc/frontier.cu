// frontier.cu — Two-Layer-Bitmap frontier kernels (PAPER.md:139 §3.1, :145 §3.2, :211-262 §4).
//   fill_all / insert / set-ops / summary rebuild, the summary-layer compaction that runs
//   before every advance ("GPU threads map to integers in the second layer to find
//   nonzero integers in the first bitmap layer and store their offsets in a global buffer"),
//   and the per-frontier statistics (n_f, m_f) the direction policy needs.
#include "common.cuh"
#include "kernels.h"

namespace sg {

// ---------------------------------------------------------------------------------------
// fill_all: every vertex active (advance::vertices); tail bits >= n stay 0.
__global__ void k_fill_all(uint64_t *bits, uint64_t *summ, int64_t n, int64_t nw1, int64_t nw2) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) {
        const int64_t lo = w * 64, rem = n - lo;
        bits[w] = rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
    }
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < nw2; s += stride) {
        const int64_t rem = nw1 - s * 64;
        summ[s] = rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
    }
}

__global__ void k_insert(uint64_t *bits, uint64_t *summ, const int32_t *v, int64_t k, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k; i += stride) {
        const int32_t x = v[i];
        if (x >= 0 && x < n) insert_2lb(bits, summ, x);
    }
}

// dst = dst OP src word-wise (§4.1); summary rebuilt by k_rebuild_summary.
__global__ void k_setop(uint64_t *dst, const uint64_t *src, int64_t nw1, int op) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) {
        const uint64_t a = dst[w], b = src[w];
        uint64_t r;
        switch (op) {
            case 0: r = a | b; break;
            case 1: r = a & b; break;
            case 2: r = a & ~b; break;
            default: r = a ^ b; break;
        }
        dst[w] = r;
    }
}

// One warp per summary word: bit l of summ[s] = (bits[64 s + l] != 0).
__global__ void k_rebuild_summary(const uint64_t *bits, uint64_t *summ, int64_t nw1, int64_t nw2) {
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = lane_id();
    for (int64_t s = gw; s < nw2; s += nwarps) {
        const int64_t w0 = s * 64 + lane, w1 = w0 + 32;
        const bool a = w0 < nw1 && bits[w0] != 0ull;
        const bool b = w1 < nw1 && bits[w1] != 0ull;
        const uint32_t ma = __ballot_sync(0xffffffffu, a), mb = __ballot_sync(0xffffffffu, b);
        if (lane == 0) summ[s] = (uint64_t)ma | ((uint64_t)mb << 32);
    }
}

// ---------------------------------------------------------------------------------------
// Summary compaction: one thread per summary word, block-wide exclusive scan of the
// popcounts, one atomicAdd per block to reserve output space; each thread then writes its
// word indices in ascending order (ascending within a block, arbitrary across blocks:
// reading C4).  st->count receives the number of non-zero layer-1 words.
constexpr int COMPACT_THREADS = 512;
__global__ void __launch_bounds__(COMPACT_THREADS)
k_compact(const uint64_t *__restrict__ summ, int64_t nw2, uint32_t *__restrict__ offsets, DevStats *st) {
    __shared__ uint32_t s_warp[COMPACT_THREADS / 32];
    __shared__ uint32_t s_base;
    const int64_t stride = (int64_t)gridDim.x * COMPACT_THREADS;
    for (int64_t s0 = blockIdx.x * (int64_t)COMPACT_THREADS; s0 < nw2; s0 += stride) {
        const int64_t s = s0 + threadIdx.x;
        const uint64_t x = s < nw2 ? summ[s] : 0ull;
        const uint32_t c = __popcll(x);
        const uint32_t incl = warp_inclusive_scan(c);
        const int wid = threadIdx.x >> 5;
        if (lane_id() == 31) s_warp[wid] = incl;
        __syncthreads();
        if (wid == 0) {
            uint32_t t = lane_id() < COMPACT_THREADS / 32 ? s_warp[lane_id()] : 0u;
            const uint32_t ti = warp_inclusive_scan(t);
            if (lane_id() < COMPACT_THREADS / 32) s_warp[lane_id()] = ti - t;
            if (lane_id() == 31) s_base = ti ? (uint32_t)atomicAdd(&st->count, (unsigned long long)ti) : 0u;
        }
        __syncthreads();
        uint32_t pos = s_base + s_warp[wid] + (incl - c);
        uint64_t y = x;
        while (y) {
            const int b = __ffsll((long long)y) - 1;
            offsets[pos++] = (uint32_t)(s * 64 + b);
            y &= y - 1;
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// n_f and m_f of a compacted frontier (Beamer's direction policy inputs): warp per word.
__global__ void __launch_bounds__(256) k_frontier_stats(GraphView g, const uint64_t *__restrict__ bits,
                                                        const uint32_t *__restrict__ offsets, DevStats *st) {
    const uint32_t count = (uint32_t)st->count;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long nf = 0, mf = 0;
    for (int64_t i = gw; i < count; i += nwarps) {
        const int64_t w = offsets[i];
        const uint64_t x = bits[w];
        int64_t sa, ea, sb, eb;
        word_bounds(g, w, x, sa, ea, sb, eb);
        mf += (unsigned long long)((ea - sa) + (eb - sb));
        if (lane_id() == 0) nf += __popcll(x);
    }
    mf = warp_sum(mf);
    nf = warp_sum(nf);
    if (lane_id() == 0 && (mf | nf)) {
        atomicAdd(&st->mf, mf);
        atomicAdd(&st->nf, nf);
    }
}

// popcount of a whole bitmap (frontier_count)
__global__ void k_popcount(const uint64_t *bits, int64_t nw1, unsigned long long *out) {
    unsigned long long c = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) c += __popcll(bits[w]);
    c = warp_sum(c);
    if (lane_id() == 0 && c) atomicAdd(out, c);
}

// dst |= bits over the listed words only (visited |= out after a step).
__global__ void k_or_listed(const uint64_t *__restrict__ bits, const uint32_t *__restrict__ offsets,
                            const DevStats *st, uint64_t *__restrict__ dst) {
    const uint32_t count = (uint32_t)st->count;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += stride) {
        const uint32_t w = offsets[i];
        dst[w] |= bits[w];
    }
}

__global__ void k_or_all(const uint64_t *__restrict__ bits, int64_t nw1, uint64_t *__restrict__ dst) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) dst[w] |= bits[w];
}


__global__ void k_iota_i32(int32_t *p, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride) p[i] = (int32_t)i;
}

// SG_F_VALIDATE: row_ptr[0] = 0, monotone, row_ptr[n] = nnz, 0 <= col < n.
__global__ void k_validate_csr(GraphView g, unsigned long long *bad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    unsigned long long b = 0;
    if (t == 0 && (g.rp[0] != 0 || g.rp[g.n] != g.nnz)) b++;
    for (int64_t v = t; v < g.n; v += stride)
        if (g.rp[v + 1] < g.rp[v]) b++;
    for (int64_t e = t; e < g.nnz; e += stride) {
        const int32_t c = g.col[e];
        if (c < 0 || c >= g.n) b++;
    }
    if (b) atomicAdd(bad, b);
}

__global__ void k_max_u8(const uint8_t *w, int64_t nnz, unsigned int *out) {
    unsigned int m = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += stride) m = max(m, (unsigned)w[e]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
    if (lane_id() == 0 && m) atomicMax(out, m);
}

// in = {src} (both layers) and optionally visited = {src}; buffers were just cleared
__global__ void k_seed(uint64_t *bits, uint64_t *summ, uint64_t *visited, int32_t src) {
    bits[src >> 6] = 1ull << (src & 63);
    summ[src >> 12] = 1ull << ((src >> 6) & 63);
    if (visited) visited[src >> 6] = 1ull << (src & 63);
}

template <typename T>
__global__ void k_set_one(T *p, int64_t i, T v) { p[i] = v; }

// ---------------------------------------------------------------------------------------
// host launchers
static int grid_for(int64_t items, int threads, int max_blocks) {
    int64_t b = (items + threads - 1) / threads;
    if (b < 1) b = 1;
    if (b > max_blocks) b = max_blocks;
    return (int)b;
}

void launch_fill_all(uint64_t *bits, uint64_t *summ, int64_t n, int64_t nw1, int64_t nw2, cudaStream_t s) {
    k_fill_all<<<grid_for(nw1, 256, 148 * 8), 256, 0, s>>>(bits, summ, n, nw1, nw2);
}
void launch_insert(uint64_t *bits, uint64_t *summ, const int32_t *v, int64_t k, int64_t n, cudaStream_t s) {
    if (k > 0) k_insert<<<grid_for(k, 256, 148 * 8), 256, 0, s>>>(bits, summ, v, k, n);
}
void launch_setop(uint64_t *dst, const uint64_t *src, int64_t nw1, int op, cudaStream_t s) {
    k_setop<<<grid_for(nw1, 256, 148 * 8), 256, 0, s>>>(dst, src, nw1, op);
}
void launch_rebuild_summary(const uint64_t *bits, uint64_t *summ, int64_t nw1, int64_t nw2, cudaStream_t s) {
    k_rebuild_summary<<<grid_for(nw2 * 32, 256, 148 * 8), 256, 0, s>>>(bits, summ, nw1, nw2);
}
void launch_compact(const uint64_t *summ, int64_t nw2, uint32_t *offsets, DevStats *st, cudaStream_t s) {
    k_compact<<<grid_for(nw2, COMPACT_THREADS, 148 * 2), COMPACT_THREADS, 0, s>>>(summ, nw2, offsets, st);
}
void launch_frontier_stats(const GraphView &g, const uint64_t *bits, const uint32_t *offsets, DevStats *st,
                           int64_t max_words, cudaStream_t s) {
    k_frontier_stats<<<grid_for(max_words * 32, 256, 148 * 8), 256, 0, s>>>(g, bits, offsets, st);
}
void launch_popcount(const uint64_t *bits, int64_t nw1, unsigned long long *out, cudaStream_t s) {
    k_popcount<<<grid_for(nw1, 256, 148 * 4), 256, 0, s>>>(bits, nw1, out);
}
void launch_or_listed(const uint64_t *bits, const uint32_t *offsets, const DevStats *st, uint64_t *dst,
                      int64_t max_words, cudaStream_t s) {
    k_or_listed<<<grid_for(max_words, 256, 148 * 8), 256, 0, s>>>(bits, offsets, st, dst);
}
void launch_or_all(const uint64_t *bits, int64_t nw1, uint64_t *dst, cudaStream_t s) {
    k_or_all<<<grid_for(nw1, 256, 148 * 8), 256, 0, s>>>(bits, nw1, dst);
}
void launch_set_u32(uint32_t *p, int64_t i, uint32_t v, cudaStream_t s) { k_set_one<uint32_t><<<1, 1, 0, s>>>(p, i, v); }
void launch_set_i32(int32_t *p, int64_t i, int32_t v, cudaStream_t s) { k_set_one<int32_t><<<1, 1, 0, s>>>(p, i, v); }
void launch_set_f64(double *p, int64_t i, double v, cudaStream_t s) { k_set_one<double><<<1, 1, 0, s>>>(p, i, v); }

void launch_seed(uint64_t *bits, uint64_t *summ, uint64_t *visited, int32_t src, cudaStream_t s) {
    k_seed<<<1, 1, 0, s>>>(bits, summ, visited, src);
}
void launch_iota_i32(int32_t *p, int64_t n, cudaStream_t s) { k_iota_i32<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(p, n); }
void launch_validate_csr(const GraphView &g, unsigned long long *bad, cudaStream_t s) {
    k_validate_csr<<<grid_for(g.nnz > g.n ? g.nnz : g.n, 256, 148 * 8), 256, 0, s>>>(g, bad);
}
void launch_max_weight(const uint8_t *w, int64_t nnz, unsigned int *out, cudaStream_t s) {
    if (nnz > 0) k_max_u8<<<grid_for(nnz, 256, 148 * 8), 256, 0, s>>>(w, nnz, out);
}

}  // namespace sg
