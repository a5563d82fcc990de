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
#include <cub/device/device_scan.cuh>
#include <vector>

#include "common.cuh"
#include "kernels.h"

namespace sg {

constexpr int CCP_THREADS = 256;
#ifndef SG_CC_HINTS
#define SG_CC_HINTS 0   // bit 0: col_idx loads evict-first, bit 1: label loads evict-last (measured: no gain / slower)
#endif
// L2 residency hints: the 2.1 GB col_idx stream must not evict the 84 MB label array, whose
// random probes otherwise cost a DRAM sector each (ncu: 23 GB of DRAM traffic per pull step for
// 4.2 GB of algorithmic bytes)
__device__ __forceinline__ int32_t ld_col(const int32_t *p, uint64_t pol) {
#if SG_CC_HINTS & 1
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
#else
    (void)pol;
    return __ldg(p);
#endif
}
__device__ __forceinline__ int32_t ld_label(const int32_t *p, uint64_t pol) {
#if SG_CC_HINTS & 2
    int32_t v;
    asm volatile("ld.global.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
#else
    (void)pol;
    return *p;
#endif
}

__global__ void __launch_bounds__(CCP_THREADS)
k_pull_cc(GraphView g, int32_t *__restrict__ label, uint64_t *__restrict__ out_bits, uint64_t *__restrict__ out_summ,
          DevStats *st) {
    __shared__ unsigned long long s_arcs[CCP_THREADS / 32];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long arcs = 0;
    uint64_t pol_last = 0, pol_first = 0;
#if SG_CC_HINTS & 1
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_first));
#endif
#if SG_CC_HINTS & 2
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_last));
#endif
    for (int64_t w = g.w1_lo + gw; w < g.w1_hi; w += nwarps) {   // owned words (1-D partition)
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
                c[k] = (ia + k < ea) ? ld_col(g.col + ia + k, pol_first) : -1;
                c[4 + k] = (ib + k < eb) ? ld_col(g.col + ib + k, pol_first) : -1;
            }
            int32_t l[8];
#pragma unroll
            for (int k = 0; k < 8; k++) l[k] = c[k] >= 0 ? ld_label(label + c[k], pol_last) : 0x7fffffff;
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

// ---- label-blocked pull (graphs whose label array does not stay in L2) --------------------
// A pull step probes one random label per arc; at config 3 (84 MB of labels, 2.1 GB of col_idx
// streamed past them) nearly every probe misses L2 and moves a 32-B DRAM sector (ncu: 23 GB per
// step for 4.2 GB of algorithmic bytes).  Rows are sorted, so the arcs of row v into label block
// b (vertices [b*S, (b+1)*S)) are contiguous: the step runs one pass per block, each reading only
// that block's labels (S*4 B <= ~32 MB, L2-resident) and the row parts that point into it.
// cbo[v*(nb-1) + b-1] = first arc of row v into block b (b = 1..nb-1), built once per graph.
__global__ void k_cc_block_offsets(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                                   int nb, int64_t S, uint32_t *__restrict__ cbo) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        const int64_t s0 = rp[v], e0 = rp[v + 1];
        for (int b = 1; b < nb; b++) {   // lower_bound(col[s0..e0), b*S)
            int64_t lo = s0, hi = e0;
            const int64_t key = (int64_t)b * S;
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                if ((int64_t)col[mid] < key) lo = mid + 1;
                else hi = mid;
            }
            cbo[v * (nb - 1) + (b - 1)] = (uint32_t)(lo - s0);
        }
    }
}
void launch_cc_block_offsets(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, uint32_t *cbo,
                             cudaStream_t s) {
    int64_t blocks = (n + 255) / 256;
    if (blocks > num_sms() * 16) blocks = num_sms() * 16;
    note_launch();
    k_cc_block_offsets<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, col, n, nb, S, cbo);
}

// one pass of the blocked pull: vertices take the min over their arcs into block b; the warp
// owning word w writes (b == 0) or ORs (b > 0) the word's changed bits into the output frontier
__global__ void __launch_bounds__(CCP_THREADS)
k_pull_cc_block(GraphView g, int32_t *__restrict__ label, uint64_t *__restrict__ out_bits, DevStats *st,
                const uint32_t *__restrict__ cbo, int nb, int b) {
    __shared__ unsigned long long s_arcs[CCP_THREADS / 32];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long arcs = 0;
    uint64_t pol_last = 0, pol_first = 0;
#if SG_CC_HINTS & 1
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_first));
#endif
#if SG_CC_HINTS & 2
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_last));
#endif
    auto part = [&](int64_t v, int64_t &s0, int64_t &e0) {
        const int64_t r0 = __ldg(g.rp + v), r1 = __ldg(g.rp + v + 1);
        s0 = b == 0 ? r0 : r0 + __ldg(cbo + v * (nb - 1) + (b - 1));
        e0 = b == nb - 1 ? r1 : r0 + __ldg(cbo + v * (nb - 1) + b);
    };
    for (int64_t w = g.w1_lo + gw; w < g.w1_hi; w += nwarps) {   // owned words (1-D partition)
        const int64_t va = w * 64 + lane, vb = va + 32;
        const bool act_a = va < g.n, act_b = vb < g.n;
        int64_t sa = 0, ea = 0, sb = 0, eb = 0;
        if (act_a) part(va, sa, ea);
        if (act_b) part(vb, sb, eb);
        const int32_t own_a = act_a ? label[va] : 0x7fffffff, own_b = act_b ? label[vb] : 0x7fffffff;
        int32_t ma = own_a, mb = own_b;
        arcs += (unsigned long long)((ea - sa) + (eb - sb));
        for (int64_t ia = sa, ib = sb; ia < ea || ib < eb; ia += 4, ib += 4) {
            int32_t c[8];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                c[k] = (ia + k < ea) ? ld_col(g.col + ia + k, pol_first) : -1;
                c[4 + k] = (ib + k < eb) ? ld_col(g.col + ib + k, pol_first) : -1;
            }
            int32_t l[8];
#pragma unroll
            for (int k = 0; k < 8; k++) l[k] = c[k] >= 0 ? ld_label(label + c[k], pol_last) : 0x7fffffff;
#pragma unroll
            for (int k = 0; k < 4; k++) {
                ma = min(ma, l[k]);
                mb = min(mb, l[4 + k]);
            }
        }
        const bool ca = ma < own_a, cb = mb < own_b;
        if (ca) label[va] = ma;
        if (cb) label[vb] = mb;
        const uint64_t nbits = (uint64_t)__ballot_sync(0xffffffffu, ca) | ((uint64_t)__ballot_sync(0xffffffffu, cb) << 32);
        if (lane == 0) {
            if (b == 0) out_bits[w] = nbits;
            else if (nbits) out_bits[w] |= nbits;
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
void launch_pull_cc_block(const GraphView &g, int32_t *label, uint64_t *out_bits, DevStats *st, const uint32_t *cbo,
                          int nb, int b, cudaStream_t s) {
    int64_t blocks = ((g.w1_hi - g.w1_lo) * 32 + CCP_THREADS - 1) / CCP_THREADS;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_cc_block<<<(int)blocks, CCP_THREADS, 0, s>>>(g, label, out_bits, st, cbo, nb, b);
}

void launch_pull_cc(const GraphView &g, int32_t *label, uint64_t *out_bits, uint64_t *out_summ, DevStats *st,
                    cudaStream_t s) {
    int64_t blocks = ((g.w1_hi - g.w1_lo) * 32 + CCP_THREADS - 1) / CCP_THREADS;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_cc<<<(int)blocks, CCP_THREADS, 0, s>>>(g, label, out_bits, out_summ, st);
}


// ---- block-major arc copy for the label-blocked pull (CcBlocks) ----------------------------
// The cbo form above reads, per pass, each row's part into block b from the row-major col_idx:
// ~8 arcs of a 25-arc row, so most parts straddle two 32-B sectors and a pass moves ~2x its
// arcs' bytes (ncu at config 3: 2.8 GB per pass, 8.4 GB per pull step for 2.1 GB of col_idx).
// Here the arcs are copied once per graph into block-major order: block b = for every v the
// neighbours of v inside [b*S, (b+1)*S), contiguous, with u32 offsets off[b][v] (relative to the
// block's base).  A pass then streams exactly its block's arcs.
__global__ void k_ccb_count(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n, int nb,
                            int64_t S, uint32_t *__restrict__ cnt) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        const int64_t s0 = rp[v], e0 = rp[v + 1];
        int64_t prev = s0;
        for (int b = 0; b < nb; b++) {
            int64_t lo = prev, hi = e0;
            const int64_t key = (int64_t)(b + 1) * S;   // lower_bound of the next block's first id
            if (b == nb - 1) {
                lo = e0;
            } else {
                while (lo < hi) {
                    const int64_t mid = (lo + hi) >> 1;
                    if ((int64_t)col[mid] < key) lo = mid + 1;
                    else hi = mid;
                }
            }
            cnt[(size_t)b * (n + 1) + v] = (uint32_t)(lo - prev);
            prev = lo;
        }
    }
}
// warp per row: arc i of row v (sorted) goes to block b = col / S at off[b][v] + its rank in the part
__global__ void k_ccb_fill(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n, int nb,
                           int64_t S, const uint32_t *__restrict__ off, const int64_t *__restrict__ base,
                           int32_t *__restrict__ out) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = gw; v < n; v += nwarps) {
        const int64_t s0 = rp[v], e0 = rp[v + 1];
        for (int64_t i = s0 + lane; i < e0; i += 32) {
            const int32_t c = col[i];
            const int b = (int)((int64_t)c / S);
            // rank of arc i inside its part = i - (first arc of the part); parts are in block order
            int64_t first = s0;
            for (int bb = 0; bb < b; bb++)
                first += off[(size_t)bb * (n + 1) + v + 1] - off[(size_t)bb * (n + 1) + v];
            out[base[b] + off[(size_t)b * (n + 1) + v] + (i - first)] = c;
        }
    }
}
void launch_ccb_count(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, uint32_t *cnt,
                      cudaStream_t s) {
    int64_t blocks = (n + 255) / 256;
    if (blocks > num_sms() * 16) blocks = num_sms() * 16;
    note_launch();
    k_ccb_count<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, col, n, nb, S, cnt);
}
void launch_ccb_fill(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, const uint32_t *off,
                     const int64_t *base, int32_t *out, cudaStream_t s) {
    int64_t blocks = (n * 32 + 255) / 256;
    if (blocks > num_sms() * 16) blocks = num_sms() * 16;
    note_launch();
    k_ccb_fill<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, col, n, nb, S, off, base, out);
}

// one pass of the blocked pull over the block-major copy (same mapping as k_pull_cc_block)
__global__ void __launch_bounds__(CCP_THREADS)
k_pull_ccb(GraphView g, int32_t *__restrict__ label, uint64_t *__restrict__ out_bits, DevStats *st,
           const uint32_t *__restrict__ off, const int32_t *__restrict__ bcol, int b) {
    __shared__ unsigned long long s_arcs[CCP_THREADS / 32];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long arcs = 0;
    for (int64_t w = g.w1_lo + gw; w < g.w1_hi; w += nwarps) {
        const int64_t va = w * 64 + lane, vb = va + 32;
        const bool act_a = va < g.n, act_b = vb < g.n;
        const int64_t sa = act_a ? __ldg(off + va) : 0, ea = act_a ? __ldg(off + va + 1) : 0;
        const int64_t sb = act_b ? __ldg(off + vb) : 0, eb = act_b ? __ldg(off + vb + 1) : 0;
        const int32_t own_a = act_a ? label[va] : 0x7fffffff, own_b = act_b ? label[vb] : 0x7fffffff;
        int32_t ma = own_a, mb = own_b;
        arcs += (unsigned long long)((ea - sa) + (eb - sb));
        for (int64_t ia = sa, ib = sb; ia < ea || ib < eb; ia += 4, ib += 4) {
            int32_t c[8];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                c[k] = (ia + k < ea) ? __ldg(bcol + ia + k) : -1;
                c[4 + k] = (ib + k < eb) ? __ldg(bcol + ib + k) : -1;
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
        const uint64_t nbits = (uint64_t)__ballot_sync(0xffffffffu, ca) | ((uint64_t)__ballot_sync(0xffffffffu, cb) << 32);
        if (lane == 0) {
            if (b == 0) out_bits[w] = nbits;
            else if (nbits) out_bits[w] |= nbits;
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
cudaError_t ccb_build(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, CcBlocks *out,
                      cudaStream_t s) {
    CcBlocks B;
    B.nb = nb;
    B.S = S;
    uint32_t *cnt = nullptr;
    void *tmp = nullptr;
    size_t tb = 0;
    const size_t per = (size_t)(n + 1);
    cudaError_t e = dev_alloc(&cnt, sizeof(uint32_t) * per * nb, s);
    if (e == cudaSuccess) e = dev_alloc(&B.off, sizeof(uint32_t) * per * nb, s);
    if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, sizeof(uint32_t) * per * nb, s);
    if (e == cudaSuccess) {
        launch_ccb_count(rp, col, n, nb, S, cnt, s);
        e = cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, B.off, (int64_t)per, s);
    }
    if (e == cudaSuccess) e = dev_alloc(&tmp, tb, s);
    for (int b = 0; b < nb && e == cudaSuccess; b++) {
        note_launch();
        e = cub::DeviceScan::ExclusiveSum(tmp, tb, cnt + (size_t)b * per, B.off + (size_t)b * per, (int64_t)per, s);
    }
    std::vector<uint32_t> tot(nb, 0);
    for (int b = 0; b < nb && e == cudaSuccess; b++)
        e = cudaMemcpyAsync(&tot[b], B.off + (size_t)b * per + n, sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    std::vector<int64_t> base(nb + 1, 0);
    for (int b = 0; b < nb; b++) base[b + 1] = base[b] + tot[b];
    B.total = base[nb];
    if (e == cudaSuccess) e = dev_alloc(&B.base, sizeof(int64_t) * (size_t)(nb + 1), s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(B.base, base.data(), sizeof(int64_t) * (size_t)(nb + 1), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = dev_alloc(&B.col, sizeof(int32_t) * (size_t)B.total + 64, s);
    if (e == cudaSuccess) {
        launch_ccb_fill(rp, col, n, nb, S, B.off, B.base, B.col, s);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (cnt) cudaFreeAsync(cnt, s);
    if (tmp) cudaFreeAsync(tmp, s);
    B.h_base = base;
    if (e != cudaSuccess) {
        ccb_free(&B);
        return e;
    }
    *out = B;
    return cudaSuccess;
}
void ccb_free(CcBlocks *B) {
    dev_free(B->off);
    dev_free(B->base);
    dev_free(B->col);
    B->off = nullptr;
    B->base = nullptr;
    B->col = nullptr;
    B->nb = 0;
}

void launch_pull_ccb(const GraphView &g, int32_t *label, uint64_t *out_bits, DevStats *st, const uint32_t *off,
                     const int32_t *bcol, int b, cudaStream_t s) {
    int64_t blocks = ((g.w1_hi - g.w1_lo) * 32 + CCP_THREADS - 1) / CCP_THREADS;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_pull_ccb<<<(int)blocks, CCP_THREADS, 0, s>>>(g, label, out_bits, st, off, bcol, b);
}

}  // namespace sg
