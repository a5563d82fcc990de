// ctrl.cu — device-side superstep control for the CUDA-graph driven loops.
//
// Listing 1's host loop (P:172 `while (!in_frontier.empty())`, swap + clear at P:182-184) costs
// one device->host round trip per superstep.  Here the whole BFS is one CUDA graph: a WHILE node
// whose body runs two supersteps (A->B, B->A, so kernel arguments stay static), each superstep
// IF(push) / IF(sweep) / IF(pull) nodes whose last kernel (k_bfs_diff, or the pull step itself)
// writes the whole output frontier with its word list and statistics, and whose last CTA applies
// the direction policy and sets the conditional handles (cudaGraphSetConditional, bfsstep.cuh).
// Results are identical to the host loop (tested).
#include "common.cuh"
#include "kernels.h"
#include "bfsstep.cuh"
#include "xchg.cuh"

namespace sg {

// Clear a frontier after it was advanced (only its listed non-zero words + its summary) and
// zero the control block of the frontier about to be compacted.
__global__ void k_clear_listed(uint64_t *__restrict__ bits, uint64_t *__restrict__ summ,
                               const uint32_t *__restrict__ offsets, const DevStats *st, int64_t nw2,
                               DevStats *zero_st) {
    const uint32_t count = (uint32_t)st->count;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = t; i < count; i += stride) bits[offsets[i]] = 0ull;
    for (int64_t s = t; s < nw2; s += stride) summ[s] = 0ull;
    if (zero_st && t < (int64_t)(sizeof(DevStats) / 8)) reinterpret_cast<unsigned long long *>(zero_st)[t] = 0ull;
}

// One-layer ablation: the offsets list names every layer-1 word (count = nw1), the control
// block's other fields are reset and m_f is copied from the compacted frontier.
__global__ void k_list_all(uint32_t *offsets, DevStats *st_all, const DevStats *st_src, int64_t nw1) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    for (int64_t w = t; w < nw1; w += stride) offsets[w] = (uint32_t)w;
    if (t == 0) {
        st_all->count = (unsigned long long)nw1;
        st_all->nf = st_src->nf;
        st_all->mf = st_src->mf;
        st_all->arcs = st_all->batch = st_all->heavy_count = st_all->seg_count = st_all->pad = 0ull;
    }
}
void launch_list_all(uint32_t *offsets, DevStats *st_all, const DevStats *st_src, int64_t nw1, cudaStream_t s) {
    int64_t blocks = (nw1 + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    note_launch();
    k_list_all<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(offsets, st_all, st_src, nw1);
}

__global__ void k_zero_u64(unsigned long long *p, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride) p[i] = 0ull;
}

// The whole BFS prologue in one kernel (graph mode): level[] = INF except level[src] = 0
// (16-B stores, buffer pointer from ctrl), and on one thread: in = {src} (layer 1 / 2 bits, word
// list, n_f = 1, m_f = src's coded degree, as the compaction + statistics kernels would give),
// visited |= {src}, then the first direction decision.  The frontier's words were zeroed before.
__global__ void k_bfs_prologue(BfsCtrl *c, int64_t n, const uint8_t *deg8, uint64_t *bits, uint64_t *summ,
                               uint32_t *offsets, DevStats *st, uint64_t *visited, uint64_t *vis_old, Xchg x) {
    uint32_t *level = c->level;
    const int32_t src = c->src;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (((uintptr_t)level & 15) == 0) {
        uint4 *l4 = reinterpret_cast<uint4 *>(level);
        for (int64_t i = t; i < n / 4; i += stride) {
            uint4 q = make_uint4(INF32, INF32, INF32, INF32);
            if (i == (src >> 2)) (&q.x)[src & 3] = 0u;
            l4[i] = q;
        }
        for (int64_t i = (n / 4) * 4 + t; i < n; i += stride) level[i] = i == src ? 0u : INF32;
    } else {
        for (int64_t i = t; i < n; i += stride) level[i] = i == src ? 0u : INF32;
    }
    if (t == 0) {
        c->src_iso = (long long)((visited[src >> 6] >> (src & 63)) & 1ull);   // visited = isolated (copied before)
        bits[src >> 6] = 1ull << (src & 63);
        summ[src >> 12] = 1ull << ((src >> 6) & 63);
        visited[src >> 6] |= 1ull << (src & 63);
        vis_old[src >> 6] |= 1ull << (src & 63);
        offsets[0] = (uint32_t)(src >> 6);
        st->count = 1ull;
        st->nf = 1ull;
        st->mf = deg8_decode(deg8[src]);
        if (x.nranks > 1) xbarrier(x, 0ull, 0ull, 0ull, nullptr);   // every rank's prologue memsets done
        c->dirty[0] = 0u;            // buffer 0: zeroed by the prologue, holds {src}
        c->dirty[1] = 1u;            // buffer 1: a previous run's frontier; contents unknown
        c->saved_count[1] = ~0ull;
        bfs_decide(c, st, 0ull, nullptr, 0, 1);
    }
}
// Single-GPU graph prologue with the frontier / bitmap initialisation folded in (one kernel
// instead of 5 memset / copy nodes + the prologue, ~1 us each in the graph): per layer-1 word w,
// visited[w] = vis_old[w] = isolated[w] (| src's bit), the input frontier's word = src's bit or 0;
// layer 2 likewise; both control blocks written whole by thread 0; then the level pass and the
// first decision as k_bfs_prologue.  Every store lands in a distinct word, so no ordering is needed
// inside the kernel (the supersteps read them after the kernel boundary).  The run's control-block
// initialisation arrives as a kernel parameter (set on the graph node before each launch): no
// host->device copy before the graph.
__global__ void k_bfs_prologue1(const BfsProArgs a) {
    const BfsCtrl *h = reinterpret_cast<const BfsCtrl *>(a.hot);   // the control block's leading part
    uint32_t *level = h->level;
    const int32_t src = h->src;
    const int64_t n = a.n;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t ws = src >> 6;
    const uint64_t sb = 1ull << (src & 63);
    for (int64_t w = t; w < a.nw1; w += stride) {
        const uint64_t v = a.isolated[w] | (w == ws ? sb : 0ull);
        a.visited[w] = v;
        a.vis_old[w] = v;
        a.bits[w] = w == ws ? sb : 0ull;
    }
    for (int64_t w = t; w < a.nw2; w += stride) a.summ[w] = w == (src >> 12) ? 1ull << ((src >> 6) & 63) : 0ull;
    if (((uintptr_t)level & 15) == 0) {
        uint4 *l4 = reinterpret_cast<uint4 *>(level);
        for (int64_t i = t; i < n / 4; i += stride) {
            uint4 q = make_uint4(INF32, INF32, INF32, INF32);
            if (i == (src >> 2)) (&q.x)[src & 3] = 0u;
            l4[i] = q;
        }
        for (int64_t i = (n / 4) * 4 + t; i < n; i += stride) level[i] = i == src ? 0u : INF32;
    } else {
        for (int64_t i = t; i < n; i += stride) level[i] = i == src ? 0u : INF32;
    }
    if (t == 0) {
        BfsCtrl *c = a.c;
        unsigned long long *cw = reinterpret_cast<unsigned long long *>(c);
        for (int i = 0; i < BFS_CTRL_HOT_WORDS; i++) cw[i] = a.hot[i];
        a.offsets[0] = (uint32_t)ws;
        c->src_iso = (long long)((a.isolated[ws] >> (src & 63)) & 1ull);
        DevStats d{};
        d.count = 1ull;
        d.nf = 1ull;
        d.mf = deg8_decode(a.deg8[src]);
        *a.st = d;
        *a.st_out = DevStats{};
        c->dirty[0] = 0u;
        c->dirty[1] = 1u;
        c->saved_count[1] = ~0ull;
        bfs_decide(c, a.st, 0ull, nullptr, 0, 1);
    }
}
// kernel-node parameters of k_bfs_prologue1 for `a` (its address must stay valid while the node
// parameters are set: kernelParams points at it)
void bfs_prologue1_node(BfsProArgs *a, void **arg_slot, cudaKernelNodeParams *kp) {
    int64_t blocks = (a->n / 4 + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    arg_slot[0] = a;
    *kp = cudaKernelNodeParams{};
    kp->func = (void *)k_bfs_prologue1;
    kp->gridDim = dim3((unsigned)blocks);
    kp->blockDim = dim3(256);
    kp->sharedMemBytes = 0;
    kp->kernelParams = arg_slot;
    kp->extra = nullptr;
}
void launch_bfs_prologue(BfsCtrl *c, int64_t n, const uint8_t *deg8, uint64_t *bits, uint64_t *summ,
                         uint32_t *offsets, DevStats *st, uint64_t *visited, uint64_t *vis_old, const Xchg &x,
                         cudaStream_t s) {
    int64_t blocks = (n / 4 + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_bfs_prologue<<<(int)blocks, 256, 0, s>>>(c, n, deg8, bits, summ, offsets, st, visited, vis_old, x);
}

__global__ void k_val_first(ValCtrl *c, const DevStats *st) { val_decide(c, st, 0ull, nullptr, 0, 1); }
void launch_val_first(ValCtrl *c, const DevStats *st, cudaStream_t s) {
    note_launch();
    k_val_first<<<1, 1, 0, s>>>(c, st);
}
// SSSP prologue of the graph-driven loop (dist and dist_old were set to INF): source from the
// control block, dist[src] = dist_old[src] = 0, input frontier {src} with its word list, decision
__global__ void k_val_seed(ValCtrl *c, uint32_t *dist, uint32_t *dist_old, uint64_t *bits, uint64_t *summ,
                           uint32_t *offsets, DevStats *st) {
    const int32_t src = c->src;
    dist[src] = 0u;
    dist_old[src] = 0u;
    bits[src >> 6] = 1ull << (src & 63);
    summ[src >> 12] = 1ull << ((src >> 6) & 63);
    offsets[0] = (uint32_t)(src >> 6);
    st->count = 1ull;
    st->nf = 1ull;
    val_decide(c, st, 0ull, nullptr, 0, 1);
}
void launch_val_seed(ValCtrl *c, uint32_t *dist, uint32_t *dist_old, uint64_t *bits, uint64_t *summ,
                     uint32_t *offsets, DevStats *st, cudaStream_t s) {
    note_launch();
    k_val_seed<<<1, 1, 0, s>>>(c, dist, dist_old, bits, summ, offsets, st);
}

// Barrier across the ranks of a partition (one thread; xchg.cuh)
__global__ void k_xbarrier(Xchg x) { xbarrier(x, 0ull, 0ull, 0ull, nullptr); }
void launch_xbarrier(const Xchg &x, cudaStream_t s) {
    if (x.nranks <= 1) return;
    note_launch();
    k_xbarrier<<<1, 1, 0, s>>>(x);
}
// The owned slice [lo, hi) of `src` into every rank's replica `vals` (own included): the result
// gather of a partitioned BFS (level), 16-B stores when aligned
__global__ void k_publish_owned(const uint32_t *__restrict__ src, uint32_t *vals, int64_t lo, int64_t hi, Xchg x) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < hi; v += stride) {
        const uint32_t a = src[v];
        for (int j = 0; j < x.nranks; j++) *xpeer(x, vals + v, j) = a;
    }
}
void launch_publish_owned(const uint32_t *src, uint32_t *vals, int64_t lo, int64_t hi, const Xchg &x, cudaStream_t s) {
    int64_t blocks = (hi - lo + 255) / 256;
    if (blocks > num_sms() * 8) blocks = num_sms() * 8;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_publish_owned<<<(int)blocks, 256, 0, s>>>(src, vals, lo, hi, x);
}

void launch_clear_listed(uint64_t *bits, uint64_t *summ, const uint32_t *offsets, const DevStats *st, int64_t nw1,
                         int64_t nw2, DevStats *zero_st, cudaStream_t s) {
    int64_t blocks = (nw1 + 255) / 256;
    if (blocks > num_sms() * 4) blocks = num_sms() * 4;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_clear_listed<<<(int)blocks, 256, 0, s>>>(bits, summ, offsets, st, nw2, zero_st);
}
void launch_zero_u64(unsigned long long *p, int64_t n, cudaStream_t s) {
    int64_t blocks = (n + 255) / 256;
    if (blocks > num_sms() * 4) blocks = num_sms() * 4;
    if (blocks < 1) blocks = 1;
    note_launch();
    k_zero_u64<<<(int)blocks, 256, 0, s>>>(p, n);
}

}  // namespace sg
