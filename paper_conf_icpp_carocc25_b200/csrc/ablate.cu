// ablate.cu — word-width ablation of the Two-Layer Bitmap push (§4.3
// "we use a 32-bit integer to match a warp on NVIDIA", Fig. 7).
//
// The product path uses 64-bit words with two bits per lane (reading C1).  To measure what the
// width itself costs, this file is one self-contained push-only BFS written once as a template
// over the word type W (uint32_t: one bit per lane, uint64_t: two bits per lane), everything else
// equal: the summary layer has W bits per word (W layer-1 words), a warp per summary word
// compacts its non-zero layer-1 words into the offsets buffer (ballot / popc), a warp per listed
// word expands the word's active vertices one at a time with its lanes striding the adjacency list
// (the paper's subgroup mapping), the visited test-and-set is an atomicOr on a W word,
// the output insert sets the layer-1 bit and, on the word's 0 -> non-zero transition, the summary
// bit.  Host-driven loop (swap, clear, stop on empty).  Results equal the oracle's BFS
// (tested); only the time differs.
#include <vector>

#include "common.cuh"
#include "kernels.h"

namespace sg {

template <class W>
struct WordTraits {
    static constexpr int bits = sizeof(W) * 8;
    static constexpr int shift = sizeof(W) == 4 ? 5 : 6;
};

template <class W>
__device__ __forceinline__ W atomic_or_w(W *p, W m) {
    if constexpr (sizeof(W) == 4) return atomicOr(reinterpret_cast<unsigned int *>(p), (unsigned int)m);
    else return atomicOr(reinterpret_cast<unsigned long long *>(p), (unsigned long long)m);
}

// warp per summary word: list the non-zero layer-1 words (ascending within the summary word)
template <class W>
__global__ void k_ab_compact(const W *__restrict__ bits, const W *__restrict__ summ, int64_t nw1, int64_t nw2,
                             uint32_t *__restrict__ offsets, unsigned long long *count) {
    constexpr int B = WordTraits<W>::bits;
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t s = gw; s < nw2; s += nwarps) {
        const W x = summ[s];
        if (!x) continue;
        // lane l covers summary bits l (and l + 32 for 64-bit words)
        for (int h = 0; h < B; h += 32) {
            const bool on = (x >> (h + lane)) & 1;
            const uint32_t m = __ballot_sync(0xffffffffu, on);
            if (!m) continue;
            unsigned long long base = 0;
            if (lane == 0) base = atomicAdd(count, (unsigned long long)__popc(m));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (on) offsets[base + __popc(m & ((1u << lane) - 1u))] = (uint32_t)(s * B + h + lane);
        }
    }
}

// warp per listed word: its active vertices one at a time, lanes striding the list
template <class W>
__global__ void k_ab_push(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, const W *__restrict__ in_bits,
                          const uint32_t *__restrict__ offsets, const unsigned long long *count, W *visited,
                          W *out_bits, W *out_summ, uint32_t *level, uint32_t next) {
    constexpr int B = WordTraits<W>::bits, S = WordTraits<W>::shift;
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t cnt = (int64_t)*count;
    for (int64_t i = gw; i < cnt; i += nwarps) {
        const int64_t w = offsets[i];
        W x = in_bits[w];
        while (x) {
            const int b = sizeof(W) == 4 ? __ffs((int)x) - 1 : __ffsll((long long)x) - 1;
            x &= x - 1;
            const int64_t u = w * B + b;
            const int64_t s = __ldg(rp + u), e = __ldg(rp + u + 1);
            for (int64_t r = s + lane; r < e; r += 32) {
                const int32_t v = __ldg(col + r);
                const W m = (W)1 << (v & (B - 1));
                if (visited[v >> S] & m) continue;
                const W old = atomic_or_w(visited + (v >> S), m);
                if (old & m) continue;
                level[v] = next;
                const W o2 = atomic_or_w(out_bits + (v >> S), m);
                if (!o2) atomic_or_w(out_summ + ((v >> S) >> S), (W)1 << ((v >> S) & (B - 1)));
            }
        }
    }
}

template <class W>
static int ab_bfs(const GraphView &g, int32_t src, uint32_t *level, cudaStream_t s, int64_t *iters, float *ms) {
    constexpr int B = WordTraits<W>::bits;
    const int64_t nw1 = (g.n + B - 1) / B, nw2 = (nw1 + B - 1) / B;
    W *fb[2] = {}, *fs[2] = {}, *vis = nullptr;
    uint32_t *off = nullptr;
    unsigned long long *cnt = nullptr;
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < 2 && e == cudaSuccess; i++) {
        e = cudaMallocAsync(&fb[i], sizeof(W) * nw1, s);
        if (e == cudaSuccess) e = cudaMallocAsync(&fs[i], sizeof(W) * nw2, s);
    }
    if (e == cudaSuccess) e = cudaMallocAsync(&vis, sizeof(W) * nw1, s);
    if (e == cudaSuccess) e = cudaMallocAsync(&off, sizeof(uint32_t) * (nw1 + 1), s);
    if (e == cudaSuccess) e = cudaMallocAsync(&cnt, sizeof(unsigned long long), s);
    cudaEvent_t a = nullptr, b = nullptr;
    int64_t it = 0;
    if (e == cudaSuccess) {
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int i = 0; i < 2; i++) {
            cudaMemsetAsync(fb[i], 0, sizeof(W) * nw1, s);
            cudaMemsetAsync(fs[i], 0, sizeof(W) * nw2, s);
        }
        cudaMemsetAsync(vis, 0, sizeof(W) * nw1, s);
        cudaMemsetAsync(level, 0xFF, sizeof(uint32_t) * (size_t)g.n, s);
        // seed: the host writes the source's bits (one word each)
        const W sb = (W)1 << (src & (B - 1));
        const int64_t sw = src / B;
        const W ss = (W)1 << (sw & (B - 1));
        cudaMemcpyAsync(fb[0] + sw, &sb, sizeof(W), cudaMemcpyHostToDevice, s);
        cudaMemcpyAsync(vis + sw, &sb, sizeof(W), cudaMemcpyHostToDevice, s);
        cudaMemcpyAsync(fs[0] + sw / B, &ss, sizeof(W), cudaMemcpyHostToDevice, s);
        const uint32_t zero = 0;
        cudaMemcpyAsync(level + src, &zero, sizeof(uint32_t), cudaMemcpyHostToDevice, s);
        cudaStreamSynchronize(s);
        cudaEventRecord(a, s);
        int in = 0;
        const int gridc = num_sms() * 8, gridp = num_sms() * 8;
        for (;;) {
            unsigned long long h = 0;
            cudaMemsetAsync(cnt, 0, sizeof h, s);
            note_launch();
            k_ab_compact<W><<<gridc, 256, 0, s>>>(fb[in], fs[in], nw1, nw2, off, cnt);
            cudaMemcpyAsync(&h, cnt, sizeof h, cudaMemcpyDeviceToHost, s);
            cudaStreamSynchronize(s);
            if (h == 0 || it > g.n) break;
            cudaMemsetAsync(fb[in ^ 1], 0, sizeof(W) * nw1, s);
            cudaMemsetAsync(fs[in ^ 1], 0, sizeof(W) * nw2, s);
            note_launch();
            k_ab_push<W><<<gridp, 256, 0, s>>>(g.rp, g.col, fb[in], off, cnt, vis, fb[in ^ 1], fs[in ^ 1], level,
                                               (uint32_t)(it + 1));
            in ^= 1;
            it++;
        }
        cudaEventRecord(b, s);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(ms, a, b);
        e = cudaGetLastError();
        cudaEventDestroy(a);
        cudaEventDestroy(b);
    }
    for (int i = 0; i < 2; i++) {
        cudaFreeAsync(fb[i], s);
        cudaFreeAsync(fs[i], s);
    }
    cudaFreeAsync(vis, s);
    cudaFreeAsync(off, s);
    cudaFreeAsync(cnt, s);
    cudaStreamSynchronize(s);
    *iters = it;
    return e == cudaSuccess ? 0 : -1;
}

int ablation_bfs_words(const GraphView &g, int32_t src, uint32_t *level, int word_bits, cudaStream_t s, int64_t *iters,
                       float *ms) {
    if (word_bits == 32) return ab_bfs<uint32_t>(g, src, level, s, iters, ms);
    return ab_bfs<uint64_t>(g, src, level, s, iters, ms);
}

}  // namespace sg
