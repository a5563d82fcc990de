// frontier.cu — Two-Layer-Bitmap frontier kernels (PAPER.md:139 §3.1, :145 §3.2, :211-262 §4).
//   fill_all / insert / set-ops / summary rebuild, the summary-layer compaction that runs
//   before every advance ("GPU threads map to integers in the second layer to find
//   nonzero integers in the first bitmap layer and store their offsets in a global buffer"),
//   and the per-frontier statistics (n_f, m_f) the direction policy needs.
#include "common.cuh"
#include "kernels.h"
#include "bfsstep.cuh"

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
// Summary compaction: one warp per summary word (lane l owns bits l and l+32), a
// block-wide exclusive scan of the 32 warps' popcounts and one atomicAdd per block to reserve
// output space.  Offsets come out ascending within a block, blocks in arbitrary order
// (reading C4).  st->count receives the number of non-zero layer-1 words.
constexpr int COMPACT_THREADS = 1024;
constexpr int COMPACT_WARPS = COMPACT_THREADS / 32;
__global__ void __launch_bounds__(COMPACT_THREADS)
k_compact(const uint64_t *__restrict__ summ, int64_t nw2, uint32_t *__restrict__ offsets, DevStats *st) {
    __shared__ uint32_t s_cnt[COMPACT_WARPS];
    __shared__ uint32_t s_base;
    const int wid = threadIdx.x >> 5, lane = lane_id();
    for (int64_t s0 = blockIdx.x * (int64_t)COMPACT_WARPS; s0 < nw2; s0 += (int64_t)gridDim.x * COMPACT_WARPS) {
        const int64_t s = s0 + wid;
        const uint64_t x = s < nw2 ? summ[s] : 0ull;
        if (lane == 0) s_cnt[wid] = __popcll(x);
        __syncthreads();
        if (wid == 0) {
            const uint32_t t = s_cnt[lane];
            const uint32_t ti = warp_inclusive_scan(t);
            s_cnt[lane] = ti - t;
            if (lane == 31) s_base = ti ? (uint32_t)atomicAdd(&st->count, (unsigned long long)ti) : 0u;
        }
        __syncthreads();
        const uint32_t base = s_base + s_cnt[wid];
        if ((x >> lane) & 1ull) offsets[base + __popcll(x & ((1ull << lane) - 1ull))] = (uint32_t)(s * 64 + lane);
        if ((x >> (lane + 32)) & 1ull)
            offsets[base + __popcll(x & ((1ull << (lane + 32)) - 1ull))] = (uint32_t)(s * 64 + lane + 32);
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// Direction-policy inputs n_f (popcount) and m_f (sum of frontier degrees).  m_f only steers
// the Beamer heuristic, so it is read from the graph's 8-bit log-coded degree array (16 MB for
// 2^24 vertices, L2 resident; <= 1/16 relative error per vertex) instead of row_ptr (134 MB).
// One thread per layer-1 word, no offsets indirection: bits + 64 code bytes per non-zero word.
// deg8_decode: common.cuh

__global__ void __launch_bounds__(256) k_frontier_stats(const uint64_t *__restrict__ bits, int64_t nw1,
                                                        const uint8_t *__restrict__ deg8, DevStats *st) {
    unsigned long long nf = 0, mf = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) {
        const uint64_t x = bits[w];
        if (!x) continue;
        nf += __popcll(x);
        const uint64_t *q = reinterpret_cast<const uint64_t *>(deg8 + w * 64);
        uint64_t c[8];
#pragma unroll
        for (int k = 0; k < 8; k++) c[k] = ((x >> (8 * k)) & 0xffull) ? __ldg(q + k) : 0ull;
#pragma unroll
        for (int k = 0; k < 8; k++) {
            uint32_t bm = (uint32_t)((x >> (8 * k)) & 0xffull);
            while (bm) {
                const int j = __ffs(bm) - 1;
                bm &= bm - 1;
                mf += deg8_decode((uint32_t)((c[k] >> (8 * j)) & 0xffull));
            }
        }
    }
    // block reduction first: one pair of atomics per CTA (a per-warp atomic on one address
    // serialises ~10^4 operations in L2 on a dense frontier)
    __shared__ unsigned long long s_mf[8], s_nf[8];
    mf = warp_sum(mf);
    nf = warp_sum(nf);
    if (lane_id() == 0) {
        s_mf[threadIdx.x >> 5] = mf;
        s_nf[threadIdx.x >> 5] = nf;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long a = 0, b = 0;
        for (int i = 0; i < (int)(blockDim.x >> 5); i++) {
            a += s_mf[i];
            b += s_nf[i];
        }
        if (a | b) {
            atomicAdd(&st->mf, a);
            atomicAdd(&st->nf, b);
        }
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

// Row structure (reading C9: rows strictly ascending, no self-loops), warp per row:
// bad[0] += pairs col[e] >= col[e+1] inside a row (unsorted or duplicate), bad[1] += self-loops.
// Runs at every load (the segmented tier and the label-blocked CC pull need sorted rows).
__global__ void k_row_check(GraphView g, unsigned long long *bad) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long unsorted = 0, loops = 0;
    for (int64_t v = gw; v < g.n; v += nwarps) {
        const int64_t s = g.rp[v], e = g.rp[v + 1];
        if (e < s || s < 0 || e > g.nnz) continue;   // malformed row_ptr: reported by k_validate_csr
        for (int64_t i = s + lane; i < e; i += 32) {
            const int32_t c = g.col[i];
            if (c == (int32_t)v) loops++;
            if (i + 1 < e && c >= g.col[i + 1]) unsorted++;
        }
    }
    unsorted = warp_sum(unsorted);
    loops = warp_sum(loops);
    if (lane == 0) {
        if (unsorted) atomicAdd(bad, unsorted);
        if (loops) atomicAdd(bad + 1, loops);
    }
}
// Symmetry (reading C8), warp per row: every arc (v, u) needs v in row u (binary search; rows
// sorted).  bad += arcs without their reverse.  SG_F_VALIDATE only (O(nnz log deg)).
__global__ void k_symmetry(GraphView g, unsigned long long *bad) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long miss = 0;
    for (int64_t v = gw; v < g.n; v += nwarps) {
        const int64_t s = g.rp[v], e = g.rp[v + 1];
        if (e < s || s < 0 || e > g.nnz) continue;
        for (int64_t i = s + lane; i < e; i += 32) {
            const int32_t u = g.col[i];
            if (u < 0 || u >= g.n) continue;
            int64_t lo = g.rp[u], hi = g.rp[u + 1];
            if (hi < lo || lo < 0 || hi > g.nnz) { miss++; continue; }
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                if (g.col[mid] < (int32_t)v) lo = mid + 1;
                else hi = mid;
            }
            if (lo >= g.rp[u + 1] || g.col[lo] != (int32_t)v) miss++;
        }
    }
    miss = warp_sum(miss);
    if (lane == 0 && miss) atomicAdd(bad, miss);
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
__global__ void k_seed(uint64_t *bits, uint64_t *summ, uint64_t *visited, int32_t src, uint64_t *vis_old) {
    bits[src >> 6] = 1ull << (src & 63);
    summ[src >> 12] = 1ull << ((src >> 6) & 63);
    if (visited) visited[src >> 6] |= 1ull << (src & 63);
    if (vis_old) vis_old[src >> 6] |= 1ull << (src & 63);
}

// bit v set iff deg(v) == 0: isolated vertices can never be reached, so BFS starts with them
// marked visited and the pull step never scans them (1/3 of a Kronecker graph's ids).
__global__ void k_isolated(const uint8_t *__restrict__ deg8, int64_t n, int64_t nw1, uint64_t *__restrict__ iso) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw1; w += stride) {
        const uint64_t *q = reinterpret_cast<const uint64_t *>(deg8 + w * 64);
        uint64_t m = 0;
        for (int k = 0; k < 8; k++) {
            const uint64_t c = q[k];
            for (int j = 0; j < 8; j++)
                if (((c >> (8 * j)) & 0xffull) == 0ull) m |= 1ull << (8 * k + j);
        }
        const int64_t rem = n - w * 64;
        if (rem < 64) m &= (1ull << rem) - 1ull;
        iso[w] = m;
    }
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
    note_launch();
    k_fill_all<<<grid_for(nw1, 256, num_sms() * 8), 256, 0, s>>>(bits, summ, n, nw1, nw2);
}
void launch_insert(uint64_t *bits, uint64_t *summ, const int32_t *v, int64_t k, int64_t n, cudaStream_t s) {
    if (k > 0) { note_launch(); k_insert<<<grid_for(k, 256, num_sms() * 8), 256, 0, s>>>(bits, summ, v, k, n); }
}
void launch_setop(uint64_t *dst, const uint64_t *src, int64_t nw1, int op, cudaStream_t s) {
    note_launch();
    k_setop<<<grid_for(nw1, 256, num_sms() * 8), 256, 0, s>>>(dst, src, nw1, op);
}
void launch_rebuild_summary(const uint64_t *bits, uint64_t *summ, int64_t nw1, int64_t nw2, cudaStream_t s) {
    note_launch();
    k_rebuild_summary<<<grid_for(nw2 * 32, 256, num_sms() * 8), 256, 0, s>>>(bits, summ, nw1, nw2);
}
void launch_compact(const uint64_t *summ, int64_t nw2, uint32_t *offsets, DevStats *st, cudaStream_t s) {
    note_launch();
    k_compact<<<grid_for(nw2, COMPACT_WARPS, num_sms() * 2), COMPACT_THREADS, 0, s>>>(summ, nw2, offsets, st);
}
void launch_frontier_stats(const GraphView &g, const uint64_t *bits, DevStats *st, cudaStream_t s) {
    note_launch();
    k_frontier_stats<<<grid_for(g.nw1, 256, num_sms() * 8), 256, 0, s>>>(bits, g.nw1, g.deg8, st);
}
// 8-bit log code of each vertex degree (exact below 32, 3 mantissa bits above); padded to 64 B
// per layer-1 word so k_frontier_stats can read whole words.
__global__ void k_deg8(const int64_t *__restrict__ rp, int64_t n, int64_t npad, uint8_t *__restrict__ deg8) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < npad; v += stride) {
        uint32_t c = 0;
        if (v < n) {
            const int64_t d = rp[v + 1] - rp[v];
            if (d < 32) {
                c = (uint32_t)d;
            } else {
                const uint32_t e = 63u - (uint32_t)__clzll((unsigned long long)d);
                c = 32u + (e - 5u) * 8u + (uint32_t)((d >> (e - 3u)) & 7);
                if (c > 255u) c = 255u;
            }
        }
        deg8[v] = (uint8_t)c;
    }
}
// Pull candidate of every vertex (graph load): the neighbour with the largest log-coded degree
// among its first FNBR_SCAN arcs (first such in list order), -1 for an isolated vertex.  A
// bottom-up BFS step tests it before the adjacency list: in a scale-free graph the large
// frontiers that make pull steps worthwhile hold the hubs, so one dense 4-B read usually
// replaces a row_ptr read plus a random col_idx sector.  Any choice is correct.
constexpr int FNBR_SCAN = 64;
__global__ void k_first_nbr(const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                            const uint8_t *__restrict__ deg8, int64_t n, int64_t npad, int32_t *__restrict__ fn) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < npad; v += stride) {
        if (v >= n) {
            fn[v] = -1;
            continue;
        }
        const int64_t s = rp[v];
        int64_t e = rp[v + 1];
        if (e > s + FNBR_SCAN) e = s + FNBR_SCAN;
        int32_t best = -1;
        int bd = -1;
        for (int64_t r = s; r < e; r++) {
            const int32_t u = __ldg(col + r);
            if (u < 0 || (int64_t)u >= n) continue;   // unvalidated input: never index out of range
            const int du = __ldg(deg8 + u);
            if (du > bd) {
                bd = du;
                best = u;
            }
        }
        fn[v] = best;
    }
}
void launch_first_nbr(const int64_t *rp, const int32_t *col, const uint8_t *deg8, int64_t n, int64_t npad,
                      int32_t *fn, cudaStream_t s) {
    if (npad <= 0) return;
    note_launch();
    k_first_nbr<<<grid_for(npad, 256, num_sms() * 8), 256, 0, s>>>(rp, col, deg8, n, npad, fn);
}
void launch_isolated(const uint8_t *deg8, int64_t n, int64_t nw1, uint64_t *iso, cudaStream_t s) {
    note_launch();
    k_isolated<<<grid_for(nw1, 256, num_sms() * 8), 256, 0, s>>>(deg8, n, nw1, iso);
}
void launch_deg8(const int64_t *rp, int64_t n, int64_t npad, uint8_t *deg8, cudaStream_t s) {
    note_launch();
    k_deg8<<<grid_for(npad, 256, num_sms() * 8), 256, 0, s>>>(rp, n, npad, deg8);
}
void launch_popcount(const uint64_t *bits, int64_t nw1, unsigned long long *out, cudaStream_t s) {
    note_launch();
    k_popcount<<<grid_for(nw1, 256, num_sms() * 4), 256, 0, s>>>(bits, nw1, out);
}
void launch_or_listed(const uint64_t *bits, const uint32_t *offsets, const DevStats *st, uint64_t *dst,
                      int64_t max_words, cudaStream_t s) {
    note_launch();
    k_or_listed<<<grid_for(max_words, 256, num_sms() * 8), 256, 0, s>>>(bits, offsets, st, dst);
}
void launch_or_all(const uint64_t *bits, int64_t nw1, uint64_t *dst, cudaStream_t s) {
    note_launch();
    k_or_all<<<grid_for(nw1, 256, num_sms() * 8), 256, 0, s>>>(bits, nw1, dst);
}
void launch_set_u32(uint32_t *p, int64_t i, uint32_t v, cudaStream_t s) { note_launch(); k_set_one<uint32_t><<<1, 1, 0, s>>>(p, i, v); }
void launch_set_i32(int32_t *p, int64_t i, int32_t v, cudaStream_t s) { note_launch(); k_set_one<int32_t><<<1, 1, 0, s>>>(p, i, v); }
void launch_set_f64(double *p, int64_t i, double v, cudaStream_t s) { note_launch(); k_set_one<double><<<1, 1, 0, s>>>(p, i, v); }

void launch_seed(uint64_t *bits, uint64_t *summ, uint64_t *visited, int32_t src, cudaStream_t s,
                 uint64_t *vis_old) {
    note_launch();
    k_seed<<<1, 1, 0, s>>>(bits, summ, visited, src, vis_old);
}

// Output of a diff-mode BFS superstep (FnBfs::diff, the sweep): the vertices first visited by
// the step are new = visited & ~vis_old.  A CTA of 8 warps takes 256 layer-1 words (4 layer-2
// words) per iteration, a warp 32 of them: it reads the word pairs coalesced (one per lane) and
// writes every output word (zero or not) and the changed words' vis_old; the CTA then writes its
// 4 layer-2 words and appends the changed words to the word list (bfs_emit_words).  The changed
// words' vertices are handled 8 words per round, one half-warp per word: a thread reads the
// degree codes of a quad of 4 vertices (m_f; the 4 loads of a round issued together, so a round
// costs one memory latency) and stores the levels of vertices lane16 + 16 i (whole 64-B runs of
// level[] per store instruction).  The last CTA decides the next superstep (graph mode).
#ifndef SG_DIFF_BLOCKS
#define SG_DIFF_BLOCKS (num_sms() * 4)   // grid cap (CTAs)
#endif
#ifndef SG_DIFF_WPR
#define SG_DIFF_WPR 8
#endif
constexpr int DIFF_WORDS_PER_ROUND = SG_DIFF_WPR;
constexpr int DIFF_THREADS = 256;
template <bool P>
__global__ void __launch_bounds__(DIFF_THREADS) k_bfs_diff(GraphView g, const uint64_t *__restrict__ visited, BfsOut o) {
    __shared__ uint64_t s_S[DIFF_THREADS / 64];
    __shared__ uint32_t s_ch[DIFF_THREADS / 32];
    __shared__ uint32_t s_base[1 + SG_MAX_RANKS], s_lut[256];
    deg8_lut_init(s_lut);   // visible after the loop's first __syncthreads
    const int lane = lane_id(), wid = threadIdx.x >> 5;
    const int half = lane >> 4;
    const int sh = (lane & 15) * 4;
    unsigned long long nf = 0, mf = 0;
    uint32_t *lvl = nullptr;
    uint32_t nx = 0;
    // owned layer-1 words only (partitioned: w1_lo is a multiple of 64, so CTA slices start on
    // layer-2 word boundaries); every output word is also stored into the peers' replicas
    for (int64_t base = g.w1_lo + blockIdx.x * (int64_t)DIFF_THREADS; base < g.w1_hi;
         base += (int64_t)gridDim.x * DIFF_THREADS) {
        const int64_t w0 = base + wid * 32;
        const int64_t wa = w0 + lane;
        uint64_t na = 0, oa = 0;
        if (wa < g.w1_hi) {
            na = visited[wa];
            oa = o.vis_old[wa];
        }
        const uint64_t da = na & ~oa;
        uint32_t ch = __ballot_sync(0xffffffffu, da != 0);
        if (lane == 0) s_ch[wid] = ch;
        if (wa < g.w1_hi) xstore<P>(o.x, o.out_bits + wa, da);
        if (da) o.vis_old[wa] = na;
        __syncthreads();
        if (threadIdx.x < DIFF_THREADS / 64)
            s_S[threadIdx.x] = (uint64_t)s_ch[2 * threadIdx.x] | ((uint64_t)s_ch[2 * threadIdx.x + 1] << 32);
        __syncthreads();
        bfs_emit_words<P>(o, g.w2_hi, base >> 6, s_S, DIFF_THREADS / 64, s_base);
        if (ch && !lvl) {
            lvl = o.level_pp ? *o.level_pp : o.level;
            nx = o.next_ptr ? *o.next_ptr : o.next;
        }
        while (ch) {
            int wi[DIFF_WORDS_PER_ROUND / 2];   // this half-warp's words of the round (-1: none)
#pragma unroll
            for (int j = 0; j < DIFF_WORDS_PER_ROUND / 2; j++) {
                const int i0 = ch ? __ffs(ch) - 1 : -1;
                ch &= ch - 1;
                const int i1 = ch ? __ffs(ch) - 1 : -1;
                ch &= ch - 1;
                wi[j] = half ? i1 : i0;
            }
            uint32_t mine[DIFF_WORDS_PER_ROUND / 2], codes[DIFF_WORDS_PER_ROUND / 2], spread[DIFF_WORDS_PER_ROUND / 2];
#pragma unroll
            for (int j = 0; j < DIFF_WORDS_PER_ROUND / 2; j++) {
                const uint64_t x = __shfl_sync(0xffffffffu, da, wi[j] < 0 ? 0 : wi[j]);
                const uint64_t d = wi[j] < 0 ? 0ull : x;
                mine[j] = (uint32_t)(d >> sh) & 0xfu;
                const uint64_t t = d >> (lane & 15);   // bits lane16, 16 + lane16, 32 + .., 48 + ..
                spread[j] = (uint32_t)(t & 1u) | (uint32_t)((t >> 15) & 2u) | (uint32_t)((t >> 30) & 4u) |
                            (uint32_t)((t >> 45) & 8u);
            }
#pragma unroll
            for (int j = 0; j < DIFF_WORDS_PER_ROUND / 2; j++)
                codes[j] = mine[j] ? __ldg(reinterpret_cast<const uint32_t *>(g.deg8 + (w0 + wi[j]) * 64 + sh)) : 0u;
#pragma unroll
            for (int j = 0; j < DIFF_WORDS_PER_ROUND / 2; j++) {
                nf += __popc(mine[j]);
                mf += quad_mf(s_lut, codes[j], mine[j]);
                // level stores strided over the half-warp (vertex 16 i + lane16): each store
                // instruction writes 64 contiguous bytes of level[] instead of 16 scattered quads
                const uint32_t sp = spread[j];
                if (sp) {
                    uint32_t *lw = lvl + (w0 + wi[j]) * 64 + (lane & 15);
#pragma unroll
                    for (int i = 0; i < 4; i++)
                        if ((sp >> i) & 1u) lw[16 * i] = nx;
                }
            }
        }
    }
    bfs_finish<P>(o, nf, mf, 0ull, nullptr);
}
void launch_bfs_diff(const GraphView &g, const uint64_t *visited, const BfsOut &o, cudaStream_t s) {
    int64_t blocks = (g.w1_hi - g.w1_lo + DIFF_THREADS - 1) / DIFF_THREADS;   // 256 layer-1 words per CTA
    if (blocks > SG_DIFF_BLOCKS) blocks = SG_DIFF_BLOCKS;
    if (blocks < 1) blocks = 1;
    note_launch();
    if (o.x.nranks > 1) k_bfs_diff<true><<<(int)blocks, DIFF_THREADS, 0, s>>>(g, visited, o);
    else k_bfs_diff<false><<<(int)blocks, DIFF_THREADS, 0, s>>>(g, visited, o);
}
// Output of a diff-mode SSSP / CC superstep (FnSssp::diff; CC pulls and pushes in place): the
// vertices whose value decreased (value < old, unsigned; CC labels are >= 0).  A CTA of 256
// threads takes 64 layer-1 words (4,096 vertices, one layer-2 word): a thread compares 4 x 4
// values (16-B loads of value and old), the half-warp ORs the word's bits, every output word is
// written, and the CTA emits its layer-2 word and word list; n_f (and m_f from the degree codes
// when want_mf, CC's direction policy) go to o.st.  Partitioned (xchg.cuh): owned layer-2 words
// only; the changed quads' new values and the output words are stored into every peer's replica
// (a value that did not change needs no exchange: peers already hold it), and the last CTA runs
// the superstep barrier.
template <bool P>
__global__ void __launch_bounds__(256) k_value_diff(GraphView g, uint32_t *__restrict__ dist,
                                                    uint32_t *__restrict__ dist_old, BfsOut o, int want_mf) {
    __shared__ uint64_t s_S[1];
    __shared__ uint32_t s_base[1 + SG_MAX_RANKS], s_lut[256];
    deg8_lut_init(s_lut);
    const int lane = lane_id();
    const uint32_t half = (lane < 16) ? 0x0000ffffu : 0xffff0000u;
    const bool vec = (((uintptr_t)dist | (uintptr_t)dist_old) & 15) == 0;
    unsigned long long nf = 0, mf = 0;
    for (int64_t sw = g.w2_lo + blockIdx.x; sw < g.w2_hi; sw += gridDim.x) {
        if (threadIdx.x == 0) s_S[0] = 0ull;
        __syncthreads();
#pragma unroll 1
        for (int r = 0; r < 4; r++) {
            const int64_t qd = sw * 1024 + r * 256 + threadIdx.x;   // quad of 4 vertices
            const int64_t w = qd >> 4;
            const int sh = (int)(qd & 15) * 4;
            uint32_t m = 0;
            if (w < g.w1_hi) {
                const int64_t v0 = w * 64 + sh;
                if (vec && v0 + 4 <= g.n) {
                    const uint4 a = *reinterpret_cast<const uint4 *>(dist + v0);
                    const uint4 b = *reinterpret_cast<const uint4 *>(dist_old + v0);
                    m = (a.x < b.x ? 1u : 0u) | (a.y < b.y ? 2u : 0u) | (a.z < b.z ? 4u : 0u) | (a.w < b.w ? 8u : 0u);
                    if (m) {
                        *reinterpret_cast<uint4 *>(dist_old + v0) = a;
                        if (P && o.x.nranks > 1)
                            for (int j = 0; j < o.x.nranks; j++)
                                if (j != o.x.rank) *reinterpret_cast<uint4 *>(xpeer(o.x, dist + v0, j)) = a;
                    }
                } else {
                    for (int k = 0; k < 4; k++) {
                        if (v0 + k >= g.n) break;
                        const uint32_t a = dist[v0 + k];
                        if (a < dist_old[v0 + k]) {
                            m |= 1u << k;
                            dist_old[v0 + k] = a;
                            if (P && o.x.nranks > 1)
                                for (int j = 0; j < o.x.nranks; j++)
                                    if (j != o.x.rank) *xpeer(o.x, dist + v0 + k, j) = a;
                        }
                    }
                }
                if (m) {
                    nf += __popc(m);
                    if (want_mf) mf += quad_mf(s_lut, __ldg(reinterpret_cast<const uint32_t *>(g.deg8 + v0)), m);
                }
            }
            const uint64_t mine = (uint64_t)m << sh;
            const uint64_t nb = (uint64_t)__reduce_or_sync(half, (uint32_t)mine) |
                                ((uint64_t)__reduce_or_sync(half, (uint32_t)(mine >> 32)) << 32);
            if ((lane & 15) == 0 && w < g.w1_hi) {
                xstore<P>(o.x, o.out_bits + w, nb);
                if (nb) atomicOr(reinterpret_cast<unsigned long long *>(s_S), 1ull << (w & 63));
            }
        }
        __syncthreads();
        bfs_emit_words<P>(o, g.w2_hi, sw, s_S, 1, s_base);
    }
    bfs_finish<P>(o, nf, mf, 0ull, nullptr);
}
void launch_value_diff(const GraphView &g, uint32_t *value, uint32_t *old, const BfsOut &o, int want_mf,
                       cudaStream_t s) {
    int64_t blocks = g.w2_hi - g.w2_lo;
    if (blocks > num_sms() * 16) blocks = num_sms() * 16;
    if (blocks < 1) blocks = 1;
    note_launch();
    if (o.x.nranks > 1) k_value_diff<true><<<(int)blocks, 256, 0, s>>>(g, value, old, o, want_mf);
    else k_value_diff<false><<<(int)blocks, 256, 0, s>>>(g, value, old, o, want_mf);
}
void launch_sssp_diff(const GraphView &g, const uint32_t *dist, uint32_t *dist_old, uint64_t *out_bits,
                      uint64_t *out_summ, uint32_t *out_offsets, DevStats *st, cudaStream_t s) {
    BfsOut o{};
    o.out_bits = out_bits;
    o.out_summ = out_summ;
    o.out_offsets = out_offsets;
    o.st = st;
    launch_value_diff(g, const_cast<uint32_t *>(dist), dist_old, o, 0, s);
}
void launch_iota_i32(int32_t *p, int64_t n, cudaStream_t s) { note_launch(); k_iota_i32<<<grid_for(n, 256, num_sms() * 8), 256, 0, s>>>(p, n); }
void launch_validate_csr(const GraphView &g, unsigned long long *bad, cudaStream_t s) {
    note_launch();
    k_validate_csr<<<grid_for(g.nnz > g.n ? g.nnz : g.n, 256, num_sms() * 8), 256, 0, s>>>(g, bad);
}
void launch_row_check(const GraphView &g, unsigned long long *bad, cudaStream_t s) {
    note_launch();
    k_row_check<<<grid_for(g.n * 32, 256, num_sms() * 8), 256, 0, s>>>(g, bad);
}
void launch_symmetry(const GraphView &g, unsigned long long *bad, cudaStream_t s) {
    note_launch();
    k_symmetry<<<grid_for(g.n * 32, 256, num_sms() * 8), 256, 0, s>>>(g, bad);
}
void launch_max_weight(const uint8_t *w, int64_t nnz, unsigned int *out, cudaStream_t s) {
    if (nnz > 0) { note_launch(); k_max_u8<<<grid_for(nnz, 256, num_sms() * 8), 256, 0, s>>>(w, nnz, out); }
}

}  // namespace sg
