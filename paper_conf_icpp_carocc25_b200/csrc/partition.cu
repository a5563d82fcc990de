// partition.cu — graph-load side of the 1-D destination partition (PAPER.md:386
// §6 "static graph partitioning ... each GPU handles a local subgraph").
//
// Rank r owns destinations [lo_r, hi_r): bounds at the arc quantiles nnz*r/P (first vertex whose
// row starts at or after the quantile), rounded to the nearest multiple of 4,096 vertices (one
// layer-2 word, so every rank owns whole layer-1 and layer-2 words), monotone, clamped to n —
// the same rule as partition.py's partition_ranges (tested equal).  A rank keeps
//   push block: for every source u the arcs (u, v) with v owned — a CSR over all n rows; rows are
//               sorted, so each is one contiguous sub-range of u's row (two binary searches);
//   pull block: the owned rows themselves (symmetric graph: in-neighbours), as a CSR over all n
//               rows whose rows outside [lo, hi) are empty.
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>

#include "common.cuh"
#include "kernels.h"

namespace sg {

// first index i in [0, n] with rp[i] >= nnz * r / P, for r = 1..P-1 (out[r-1])
__global__ void k_part_quantiles(const int64_t *__restrict__ rp, int64_t n, int64_t nnz, int P, int64_t *out) {
    const int r = 1 + blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= P) return;
    const int64_t target = (int64_t)((__int128)nnz * r / P);
    int64_t lo = 0, hi = n + 1;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (rp[mid] < target) lo = mid + 1;
        else hi = mid;
    }
    out[r - 1] = lo;
}

__device__ __forceinline__ int64_t lower_bound_row(const int32_t *__restrict__ col, int64_t s, int64_t e, int64_t key) {
    while (s < e) {
        const int64_t mid = (s + e) >> 1;
        if ((int64_t)col[mid] < key) s = mid + 1;
        else e = mid;
    }
    return s;
}

// cnt[u] = arcs of row u into [lo, hi); beg[u] = the first of them
__global__ void k_push_count(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n, int64_t lo,
                             int64_t hi, int64_t *__restrict__ cnt, int64_t *__restrict__ beg) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += stride) {
        const int64_t s = rp[u], e = rp[u + 1];
        const int64_t a = lower_bound_row(col, s, e, lo);
        const int64_t b = lower_bound_row(col, a, e, hi);
        cnt[u] = b - a;
        beg[u] = a;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) cnt[n] = 0;
}

// warp per row: copy the row's owned part (and its weights) to the push block
__global__ void k_push_fill(const int32_t *__restrict__ col, const uint8_t *__restrict__ w, int64_t n,
                            const int64_t *__restrict__ beg, const int64_t *__restrict__ rpp, int32_t *__restrict__ colp,
                            uint8_t *__restrict__ wp) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < n; u += nwarps) {
        const int64_t d = rpp[u + 1] - rpp[u], b = beg[u], o = rpp[u];
        for (int64_t i = lane; i < d; i += 32) {
            colp[o + i] = col[b + i];
            if (w) wp[o + i] = w[b + i];
        }
    }
}

// pull block row pointers: rp_l[v] = rp[clamp(v, lo, hi)] - rp[lo]
__global__ void k_pull_rowptr(const int64_t *__restrict__ rp, int64_t n, int64_t lo, int64_t hi,
                              int64_t *__restrict__ rpl) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t base = rp[lo];
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n; v += stride) {
        const int64_t c = v < lo ? lo : (v > hi ? hi : v);
        rpl[v] = rp[c] - base;
    }
}

static int grid_of(int64_t items, int per) {
    int64_t b = (items + per - 1) / per;
    if (b < 1) b = 1;
    if (b > num_sms() * 16) b = num_sms() * 16;
    return (int)b;
}

cudaError_t part_quantiles(const int64_t *rp, int64_t n, int64_t nnz, int P, int64_t *h_out, cudaStream_t s) {
    if (P <= 1) return cudaSuccess;
    int64_t *d = nullptr;
    cudaError_t e = cudaMallocAsync(&d, sizeof(int64_t) * P, s);
    if (e != cudaSuccess) return e;
    note_launch();
    k_part_quantiles<<<1, 64, 0, s>>>(rp, n, nnz, P, d);
    e = cudaMemcpyAsync(h_out, d, sizeof(int64_t) * (P - 1), cudaMemcpyDeviceToHost, s);
    cudaFreeAsync(d, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    return e;
}

cudaError_t part_push_block(const int64_t *rp, const int32_t *col, const uint8_t *w, int64_t n, int64_t lo, int64_t hi,
                            int64_t **rpp_out, int32_t **colp_out, uint8_t **wp_out, int64_t *nnz_out, cudaStream_t s) {
    int64_t *cnt = nullptr, *beg = nullptr, *rpp = nullptr;
    int32_t *colp = nullptr;
    uint8_t *wp = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    int64_t nnzp = 0;
    cudaError_t e = dev_alloc(&cnt, sizeof(int64_t) * (size_t)(n + 1), s);
    if (e == cudaSuccess) e = dev_alloc(&beg, sizeof(int64_t) * (size_t)n, s);
    if (e == cudaSuccess) e = dev_alloc(&rpp, sizeof(int64_t) * (size_t)(n + 1), s);
    if (e == cudaSuccess) {
        note_launch();
        k_push_count<<<grid_of(n, 256), 256, 0, s>>>(rp, col, n, lo, hi, cnt, beg);
        e = cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, cnt, rpp, n + 1, s);
    }
    if (e == cudaSuccess) e = dev_alloc(&tmp, tmp_bytes, s);
    if (e == cudaSuccess) {
        note_launch();
        e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cnt, rpp, n + 1, s);
    }
    if (e == cudaSuccess) e = cudaMemcpyAsync(&nnzp, rpp + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = dev_alloc(&colp, sizeof(int32_t) * (size_t)nnzp + 64, s);
    if (e == cudaSuccess) e = cudaMemsetAsync((char *)colp + sizeof(int32_t) * (size_t)nnzp, 0, 64, s);
    if (e == cudaSuccess && w) e = dev_alloc(&wp, (size_t)nnzp + 64, s);
    if (e == cudaSuccess && w) e = cudaMemsetAsync(wp + nnzp, 0, 64, s);
    if (e == cudaSuccess) {
        note_launch();
        k_push_fill<<<grid_of(n * 32, 256), 256, 0, s>>>(col, w, n, beg, rpp, colp, wp);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (cnt) cudaFreeAsync(cnt, s);
    if (beg) cudaFreeAsync(beg, s);
    if (tmp) cudaFreeAsync(tmp, s);
    if (e != cudaSuccess) {
        if (rpp) cudaFreeAsync(rpp, s);
        if (colp) cudaFreeAsync(colp, s);
        if (wp) cudaFreeAsync(wp, s);
        return e;
    }
    *rpp_out = rpp;
    *colp_out = colp;
    *wp_out = wp;
    *nnz_out = nnzp;
    return cudaSuccess;
}

cudaError_t part_pull_block(const int64_t *rp, const int32_t *col, int64_t n, int64_t lo, int64_t hi,
                            int64_t **rpl_out, int32_t **coll_out, int64_t *nnz_out, cudaStream_t s) {
    int64_t r[2] = {0, 0};
    cudaError_t e = cudaMemcpyAsync(&r[0], rp + lo, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&r[1], rp + hi, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return e;
    const int64_t m = r[1] - r[0];
    int64_t *rpl = nullptr;
    int32_t *coll = nullptr;
    e = dev_alloc(&rpl, sizeof(int64_t) * (size_t)(n + 1), s);
    if (e == cudaSuccess) e = dev_alloc(&coll, sizeof(int32_t) * (size_t)m + 64, s);
    if (e == cudaSuccess) e = cudaMemsetAsync((char *)coll + sizeof(int32_t) * (size_t)m, 0, 64, s);
    if (e == cudaSuccess && m) e = cudaMemcpyAsync(coll, col + r[0], sizeof(int32_t) * (size_t)m, cudaMemcpyDeviceToDevice, s);
    if (e == cudaSuccess) {
        note_launch();
        k_pull_rowptr<<<grid_of(n + 1, 256), 256, 0, s>>>(rp, n, lo, hi, rpl);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
        if (rpl) cudaFreeAsync(rpl, s);
        if (coll) cudaFreeAsync(coll, s);
        return e;
    }
    *rpl_out = rpl;
    *coll_out = coll;
    *nnz_out = m;
    return cudaSuccess;
}


// ---- transpose (CSC) of a directed CSR for pull steps (§3.1 "CSR and CSC") --
// in-degree histogram -> exclusive scan -> scatter with per-row cursors -> per-row sort (the pull
// candidate heuristic scans a row's first arcs; sorted rows keep it deterministic)
__global__ void k_indeg(const int32_t *__restrict__ col, int64_t nnz, unsigned long long *__restrict__ indeg) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += stride)
        atomicAdd(indeg + col[e], 1ull);
}
__global__ void k_csc_fill(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                           const int64_t *__restrict__ rpt, unsigned long long *__restrict__ cursor,
                           int32_t *__restrict__ colt) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < n; u += nwarps)
        for (int64_t e = rp[u] + lane; e < rp[u + 1]; e += 32) {
            const int32_t v = col[e];
            colt[rpt[v] + (int64_t)atomicAdd(cursor + v, 1ull)] = (int32_t)u;
        }
}

cudaError_t build_csc(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int64_t **rpt_out,
                      int32_t **colt_out, cudaStream_t s) {
    unsigned long long *cnt = nullptr;
    int64_t *rpt = nullptr;
    int32_t *colt = nullptr, *sorted = nullptr;
    void *tmp = nullptr;
    size_t tb = 0, tb2 = 0;
    cudaError_t e = dev_alloc(&cnt, sizeof(unsigned long long) * (size_t)(n + 1), s);
    if (e == cudaSuccess) e = dev_alloc(&rpt, sizeof(int64_t) * (size_t)(n + 1), s);
    if (e == cudaSuccess) e = dev_alloc(&colt, sizeof(int32_t) * (size_t)nnz + 64, s);
    if (e == cudaSuccess) e = dev_alloc(&sorted, sizeof(int32_t) * (size_t)nnz + 64, s);
    if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * (size_t)(n + 1), s);
    if (e == cudaSuccess && nnz) {
        note_launch();
        k_indeg<<<grid_of(nnz, 256), 256, 0, s>>>(col, nnz, cnt);
    }
    if (e == cudaSuccess)
        e = cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, reinterpret_cast<unsigned long long *>(rpt), n + 1, s);
    if (e == cudaSuccess)
        e = cub::DeviceSegmentedSort::SortKeys(nullptr, tb2, colt, sorted, nnz, n, rpt, rpt + 1, s);
    if (e == cudaSuccess) e = dev_alloc(&tmp, tb > tb2 ? tb : tb2, s);
    if (e == cudaSuccess) {
        note_launch();
        e = cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, reinterpret_cast<unsigned long long *>(rpt), n + 1, s);
    }
    if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * (size_t)(n + 1), s);
    if (e == cudaSuccess && nnz) {
        note_launch();
        k_csc_fill<<<grid_of(n * 32, 256), 256, 0, s>>>(rp, col, n, rpt, cnt, colt);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess && nnz) {
        note_launch();
        e = cub::DeviceSegmentedSort::SortKeys(tmp, tb2, colt, sorted, nnz, n, rpt, rpt + 1, s);
    }
    if (e == cudaSuccess) e = cudaMemsetAsync((char *)sorted + sizeof(int32_t) * (size_t)nnz, 0, 64, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (cnt) cudaFreeAsync(cnt, s);
    if (tmp) cudaFreeAsync(tmp, s);
    if (colt) cudaFreeAsync(colt, s);
    if (e != cudaSuccess) {
        if (rpt) cudaFreeAsync(rpt, s);
        if (sorted) cudaFreeAsync(sorted, s);
        return e;
    }
    *rpt_out = rpt;
    *colt_out = sorted;
    return cudaSuccess;
}

}  // namespace sg
