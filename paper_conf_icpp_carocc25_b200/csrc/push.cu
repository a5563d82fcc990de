// push.cu — instantiations + launchers of the push advance for the four functors
// (§3.4: BFS, SSSP, CC, BC).  Design: push.cuh / seg.cuh header comments, DESIGN.md §6.
#include "kernels.h"
#include "push.cuh"
#include "seg.cuh"

namespace sg {

static PushParams make_params(const PushLaunch &L) {
    PushParams p;
    p.g = L.g;
    p.in_bits = L.in_bits;
    p.offsets = L.offsets;
    p.st = L.st;
    p.heavy = L.heavy;
    p.heavy_cap = L.heavy_cap;
    p.heavy_deg = L.heavy_deg;
    p.small_deg = L.small_deg;
    p.batch = L.batch;
    p.seg = L.seg;
    p.seg_cap = L.seg_cap;
    p.seg_mode = L.seg_mode;
    p.seg_threshold = L.seg_threshold;
    p.skip_mf = L.skip_mf;
    p.sparse_ok = L.sparse_ok;
    p.chunk = HEAVY_CHUNK;
    return p;
}

template <class F>
static void launch_push(const PushLaunch &L, const F &f, cudaStream_t s) {
    static bool attr_done = false;
    if (!attr_done) {
        cudaFuncSetAttribute(k_push_heavy<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)HEAVY_SMEM);
        if constexpr (F::kSeg)
            cudaFuncSetAttribute(k_push_seg, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SEG_SMEM);
        attr_done = true;
    }
    const PushParams p = make_params(L);
    note_launch();
    k_push_words<F><<<L.grid_words, PUSH_THREADS, 0, s>>>(p, f);
    note_launch();
    k_push_heavy<F><<<L.grid_heavy, HEAVY_THREADS, HEAVY_SMEM, s>>>(p, f);
    if constexpr (F::kSeg) {
        if (p.seg && p.seg_mode && L.g.hub_idx) {
            note_launch();
            // one CTA per SM (192 KB slice); at least one per destination segment (SG_SEG_OWNER)
            k_push_seg<<<L.g.nseg > num_sms() ? L.g.nseg : num_sms(), SEG_THREADS, SEG_SMEM, s>>>(p, f);
        }
    }
}

int push_max_grid_words() { return num_sms() * 4; }   // 64 regs x 256 threads: 4 CTAs per SM resident
int push_max_grid_heavy() { return num_sms() * 3; }

void launch_push_bfs(const PushLaunch &L, const BfsArgs &a, cudaStream_t s) {
    FnBfs f;
    f.visited = a.visited;
    f.level = a.level;
    f.next = a.next;
    f.next_ptr = a.next_ptr;
    f.level_pp = a.level_pp;
    f.out = OutSink{a.out_bits, a.out_summ};
    f.diff = a.diff;
    launch_push(L, f, s);
}
void launch_push_sssp(const PushLaunch &L, const SsspArgs &a, cudaStream_t s) {
    FnSssp f;
    f.dist = a.dist;
    f.out = OutSink{a.out_bits, a.out_summ};
    f.diff = a.diff;
    launch_push(L, f, s);
}
void launch_push_cc(const PushLaunch &L, const CcArgs &a, cudaStream_t s) {
    FnCc f;
    f.label = a.label;
    f.out = OutSink{a.out_bits, a.out_summ};
    launch_push(L, f, s);
}
void launch_push_bc(const PushLaunch &L, const BcArgs &a, cudaStream_t s) {
    FnBcSigma f;
    f.visited = a.visited;
    f.sigma = a.sigma;
    f.level = a.level;
    f.next = a.next;
    f.out = OutSink{a.out_bits, a.out_summ};
    launch_push(L, f, s);
}

// ---- hub segment offsets (graph load) ----------------------------------------------------
__global__ void k_hub_mark(const int64_t *__restrict__ rp, int64_t n, int32_t *__restrict__ hub_idx,
                           int32_t *__restrict__ hub_vertex, unsigned int *count) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += stride) {
        int32_t h = -1;
        if (rp[u + 1] - rp[u] >= SEG_MIN) {
            h = (int32_t)atomicAdd(count, 1u);
            hub_vertex[h] = (int32_t)u;
        }
        hub_idx[u] = h;
    }
}

// hub_off[h][b] = number of neighbours of hub h with id < b * SEG_V (lower bound in the sorted row)
__global__ void k_hub_off(const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                          const int32_t *__restrict__ hub_vertex, int64_t nh, int nseg, uint32_t *__restrict__ off) {
    const int64_t S1 = nseg + 1;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nh * S1; t += stride) {
        const int64_t h = t / S1;
        const int b = (int)(t % S1);
        const int32_t u = hub_vertex[h];
        const int64_t r0 = rp[u], d = rp[u + 1] - r0;
        int64_t lo = 0, hi = d;
        const int64_t key = (int64_t)b * SEG_V;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if ((int64_t)col[r0 + mid] < key) lo = mid + 1;
            else hi = mid;
        }
        off[t] = (uint32_t)lo;
    }
}

void launch_hub_mark(const int64_t *rp, int64_t n, int32_t *hub_idx, int32_t *hub_vertex, unsigned int *count,
                     cudaStream_t s) {
    int64_t blocks = (n + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    note_launch();
    k_hub_mark<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, n, hub_idx, hub_vertex, count);
}
void launch_hub_off(const int64_t *rp, const int32_t *col, const int32_t *hub_vertex, int64_t nh, int nseg,
                    uint32_t *off, cudaStream_t s) {
    const int64_t items = nh * (nseg + 1);
    int64_t blocks = (items + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    note_launch();
    k_hub_off<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, col, hub_vertex, nh, nseg, off);
}

}  // namespace sg
