// capi.cu — the C ABI (include/sygraph.h) and the superstep drivers of BFS / SSSP / CC / BC.
//
// Execution model (§3 BSP; Listing 1): one advance per superstep,
// the output frontier consistent at the end of the step, swap + clear, stop when the frontier
// is empty.  Per superstep the host reads back one 128-byte control block (frontier sizes for
// empty() and the direction policy); everything else stays on the device stream.
#include <atomic>
#include <cstddef>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>
#include <mutex>

#include <cuda.h>   // CUdeviceptr / CUresult types for the driver entry point below (no -lcuda)

#include "sygraph.h"
#include "kernels.h"
#include "comm.h"

using namespace sg;

namespace sg {
static std::atomic<long long> g_launches{0};
void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
}  // namespace sg

// ------------------------------------------------------------------------------------------
// errors
static thread_local std::string t_err;
static int fail(int code, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    t_err = buf;
    return code;
}
#define CK(x)                                                                                          \
    do {                                                                                               \
        cudaError_t e_ = (x);                                                                          \
        if (e_ != cudaSuccess) {                                                                       \
            return fail(e_ == cudaErrorMemoryAllocation ? SG_ERR_OOM : SG_ERR_CUDA, "%s: %s (%s:%d)", #x, \
                        cudaGetErrorString(e_), __FILE__, __LINE__);                                   \
        }                                                                                              \
    } while (0)
#define TRY(x)                 \
    do {                       \
        int r_ = (x);          \
        if (r_ != SG_OK) return r_; \
    } while (0)

// ------------------------------------------------------------------------------------------
// handles
struct sg_frontier {
    const sg_graph *g;
    uint64_t *bits = nullptr;      // nw1 words
    uint64_t *summ = nullptr;      // nw2 words
    uint32_t *offsets = nullptr;   // nw1 entries
    DevStats *st = nullptr;        // control block (device)
    bool owns_st = true;
    bool in_arena = false;         // buffers carved from a partitioned graph's exchange arena
};

struct sg_comm {
    Comm c;
};

// IPC-shared exchange memory of a partitioned graph (xchg.cuh): same layout on every rank, so a
// local pointer p has the peer replica p + x.delta[j].
struct Arena {
    void *base = nullptr;
    size_t bytes = 0;
    XCtl *ctl = nullptr;
    uint64_t *bits[2] = {}, *summ[2] = {};
    uint32_t *offsets[2] = {};
    DevStats *st = nullptr;        // 3 control blocks (fr[0], fr[1], spare)
    uint32_t *vals = nullptr;      // n (+ pad) u32: SSSP dist / CC labels / BFS level gather, replicated
    void *peer[SG_MAX_RANKS] = {};
    Xchg x;
};

// Optional per-kernel-class timing (CUDA events on the launching stream) + algorithmic bytes
// (DESIGN.md §6 "Measurement").  Off by default; bench.py turns it on for the roofline.
struct ProfRec {
    int cls;
    cudaEvent_t a, b;
    double bytes;
};
struct Prof {
    bool on = false;
    std::vector<cudaEvent_t> pool;
    size_t used = 0;
    std::vector<ProfRec> recs;
    double ms[SG_K_COUNT] = {0};
    double bytes[SG_K_COUNT] = {0};
    int64_t launches[SG_K_COUNT] = {0};
};

struct Workspace {
    Prof prof;
    sg_frontier fr[2];
    DevStats *st = nullptr;        // 2 contiguous control blocks (fr[0].st, fr[1].st)
    DevStats *h_st = nullptr;      // pinned host mirror
    uint64_t *visited = nullptr;   // nw1 words
    uint64_t *vis_old = nullptr;   // nw1 words: visited before the current BFS superstep (k_bfs_diff)
    uint32_t *dist_old = nullptr;  // n: distances before the current SSSP superstep (k_sssp_diff)
    uint32_t *all_offsets = nullptr;   // one-layer ablation: identity word list
    sg_frontier *far = nullptr;        // delta-stepping SSSP: far pile
    HeavyItem *heavy = nullptr;
    uint32_t heavy_cap = 0;
    int32_t heavy_deg = 0;
    unsigned long long *scratch = nullptr;   // 8 device u64 counters (BC max, stack top, underflow ...)
    unsigned long long *h_scratch = nullptr;
    int32_t *stack = nullptr;      // BC: BFS order
    int32_t *exp_of_level = nullptr;
    double *delta = nullptr;
    double *sigma = nullptr;
    uint32_t *level = nullptr;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    // CUDA-graph driven BFS (ctrl.cu): instantiated once per (level buffer, tiers)
    BfsCtrl *ctrl = nullptr, *h_ctrl = nullptr;
    BfsResult *h_res = nullptr, *d_res = nullptr;   // mapped pinned: the graph-driven BFS's counters
    BfsProArgs pro_args{};                           // single GPU: the prologue node's argument block
    void *pro_slot[1] = {};
    cudaGraphNode_t pro_node = nullptr;
    unsigned int *bfs_done = nullptr;   // CTA completion counter of the BFS output kernels (self-resetting)
    unsigned int *gbar = nullptr;       // grid barrier of the sparse superstep kernel (2 u32)
    unsigned long long hnd[9] = {};     // conditional handles of bfs_graph (loop, push/pull/sweep/sparse x 2)
    // graph-driven SSSP (index 0) / CC (index 1): one graph per (result buffer, tiers, CC blocks)
    struct VGraph {
        cudaGraph_t graph = nullptr;
        cudaGraphExec_t exec = nullptr;
        void *result = nullptr;
        int32_t heavy = 0, small = 0, nb = 0;
        bool ccb = false;
        unsigned long long h[5] = {};   // loop, push x2, pull x2
    } vg[2];
    ValCtrl *vctrl = nullptr, *h_vctrl = nullptr;
    cudaGraph_t bfs_graph = nullptr;
    cudaGraphExec_t bfs_exec = nullptr;
    uint32_t *bfs_level = nullptr;
    int32_t bfs_heavy = 0, bfs_small = 0, bfs_seg = -1, bfs_cf = -1, bfs_scsr = -1, bfs_shape = -1;
    SegItem *seg = nullptr;        // destination-segmented hub queue (BFS)
    uint32_t seg_cap = 0;
    // source-batched BC (bcb.cu)
    BcbLaunch bcb{};
    bool bcb_ready = false;
    BcbCtrl *h_bcb = nullptr;
    cudaStream_t cap_stream = nullptr;
};

struct sg_graph {
    GraphView v;
    int64_t *rp = nullptr;
    int32_t *col = nullptr;
    uint8_t *w = nullptr;
    uint8_t *deg8 = nullptr;
    int32_t *fnbr = nullptr;        // pull candidate per vertex
    uint64_t *isolated = nullptr;   // bit v <=> deg(v) == 0
    int32_t *hub_idx = nullptr;     // hub index of u (deg >= SEG_MIN) or -1
    int32_t *hub_vertex = nullptr;
    uint32_t *hub_off = nullptr;    // [nhubs][nseg+1] segment offsets within the hub's row
    uint32_t *cbo = nullptr;        // [n][cbo_nb-1] first arc of each row into each CC label block (run_cc)
    int cbo_nb = 0;
    CcBlocks ccb;                   // block-major arc copy for the label-blocked CC pull (built lazily)
    int ccb_state = 0;              // 0 not built, 1 built (ccb.nb blocks), -1 unavailable (memory)
    int64_t nhubs = 0;
    ScsrStore scsr;                 // destination-segmented copy of the arcs (BFS heavy push), built lazily
    int scsr_state = 0;             // 0 not built, 1 built, -1 unavailable (segment block >= 2^32 arcs, unsorted rows)
    uint32_t max_w = 0;
    int device = 0;
    bool borrowed = false;          // SG_F_BORROW: rp / col / w are the caller's
    bool sorted = true;             // every row strictly ascending (checked at load)
    Workspace *ws = nullptr;
    // 1-D destination partition: v = push block, vl = pull block (owned rows);
    // single GPU: vl = v
    GraphView vl;
    int64_t nnz_global = 0;         // arcs of the whole graph (Beamer m_u, CC direction)
    int64_t *rpl = nullptr;         // pull block buffers (partitioned only)
    int32_t *coll = nullptr;
    Arena *ar = nullptr;            // exchange arena (partitioned only)
    int nranks = 1, rank = 0;
    sg_comm *comm = nullptr;        // partitioned: graph_free is collective over it
    int64_t n_iso = 0;              // isolated vertices (deg 0; directed: in-degree 0)
    bool directed = false;          // SG_F_DIRECTED: CSR = out-arcs, rpt / colt = the transpose (pull)
    int64_t *rpt = nullptr;
    int32_t *colt = nullptr;
};
static std::atomic<int> g_live_graphs{0};

// Result slots of graph-driven BFS runs (R20): mapped pinned host memory, carved from slabs that
// live for the process (a cudaHostAlloc / cudaFreeHost pair per graph load cost ~0.7 s of
// graph_load + graph_free in the end-to-end bench: freeing mapped memory synchronises and unmaps)
static std::mutex g_res_mu;
static std::vector<std::pair<BfsResult *, BfsResult *>> g_res_free;   // (host, device)
static int res_slot_alloc(BfsResult **h, BfsResult **d) {
    std::lock_guard<std::mutex> lk(g_res_mu);
    if (g_res_free.empty()) {
        constexpr int SLAB = 256;
        BfsResult *hs = nullptr, *ds = nullptr;
        CK(cudaHostAlloc(&hs, sizeof(BfsResult) * SLAB, cudaHostAllocMapped | cudaHostAllocPortable));
        CK(cudaHostGetDevicePointer(&ds, hs, 0));
        for (int i = SLAB - 1; i >= 0; i--) g_res_free.emplace_back(hs + i, ds + i);
    }
    *h = g_res_free.back().first;
    *d = g_res_free.back().second;
    g_res_free.pop_back();
    return SG_OK;
}
static void res_slot_free(BfsResult *h) {
    std::lock_guard<std::mutex> lk(g_res_mu);
    // the device pointer of a slot: same offset in its slab (slabs are never freed)
    BfsResult *d = nullptr;
    if (cudaHostGetDevicePointer(&d, h, 0) == cudaSuccess) g_res_free.emplace_back(h, d);
}

static const int32_t kDefaultHeavy = 2048;
static const int32_t kDefaultSmall = 32;

static int alloc_frontier_bufs(sg_frontier *f, const sg_graph *g, bool own_st) {
    f->g = g;
    CK(cudaMalloc(&f->bits, sizeof(uint64_t) * (size_t)(g->v.nw1 + 8)));   // +8: 16-B bulk copies of a unit's tail
    CK(cudaMalloc(&f->summ, sizeof(uint64_t) * (size_t)g->v.nw2));
    CK(cudaMalloc(&f->offsets, sizeof(uint32_t) * (size_t)g->v.nw1));
    if (own_st) CK(cudaMalloc(&f->st, sizeof(DevStats)));
    f->owns_st = own_st;
    CK(cudaMemset(f->bits, 0, sizeof(uint64_t) * (size_t)(g->v.nw1 + 8)));
    CK(cudaMemset(f->summ, 0, sizeof(uint64_t) * (size_t)g->v.nw2));
    if (own_st) CK(cudaMemset(f->st, 0, sizeof(DevStats)));
    return SG_OK;
}

static void free_frontier_bufs(sg_frontier *f) {
    if (f->in_arena) {
        f->bits = f->summ = nullptr;
        f->offsets = nullptr;
        f->st = nullptr;
        return;
    }
    cudaFree(f->bits);
    cudaFree(f->summ);
    cudaFree(f->offsets);
    if (f->owns_st) cudaFree(f->st);
    f->bits = f->summ = nullptr;
    f->offsets = nullptr;
    f->st = nullptr;
}

static int ensure_ws(sg_graph *g) {
    if (g->ws) return SG_OK;
    Workspace *ws = new Workspace();
    g->ws = ws;
    CK(cudaMallocHost(&ws->h_st, 3 * sizeof(DevStats)));
    if (g->ar) {   // partitioned: the two frontiers and their control blocks live in the arena
        ws->st = g->ar->st;
        for (int i = 0; i < 2; i++) {
            sg_frontier &f = ws->fr[i];
            f.g = g;
            f.bits = g->ar->bits[i];
            f.summ = g->ar->summ[i];
            f.offsets = g->ar->offsets[i];
            f.st = ws->st + i;
            f.owns_st = false;
            f.in_arena = true;
        }
    } else {
        CK(cudaMalloc(&ws->st, 3 * sizeof(DevStats)));   // fr[0], fr[1], one-layer ablation list
        CK(cudaMemset(ws->st, 0, 3 * sizeof(DevStats)));
        for (int i = 0; i < 2; i++) {
            TRY(alloc_frontier_bufs(&ws->fr[i], g, false));
            ws->fr[i].st = ws->st + i;
        }
    }
    CK(cudaMalloc(&ws->bfs_done, sizeof(unsigned int)));
    CK(cudaMemset(ws->bfs_done, 0, sizeof(unsigned int)));
    CK(cudaMalloc(&ws->gbar, 4 * sizeof(unsigned int)));
    CK(cudaMemset(ws->gbar, 0, 4 * sizeof(unsigned int)));
    CK(cudaMalloc(&ws->visited, sizeof(uint64_t) * (size_t)(g->v.nw1 + 8)));   // +8: 16-B bulk copies of a tail
    CK(cudaMalloc(&ws->vis_old, sizeof(uint64_t) * (size_t)g->v.nw1));
    CK(cudaMalloc(&ws->scratch, 8 * sizeof(unsigned long long)));
    CK(cudaMallocHost(&ws->h_scratch, 8 * sizeof(unsigned long long)));
    CK(cudaEventCreate(&ws->ev0));
    CK(cudaEventCreate(&ws->ev1));
    return SG_OK;
}

// heavy queue sized for the smallest heavy threshold used so far: sum over vertices with
// deg > T of ceil(deg / CHUNK) <= nnz / CHUNK + nnz / T.
static int ensure_heavy(sg_graph *g, int32_t heavy_deg) {
    Workspace *ws = g->ws;
    if (ws->heavy && ws->heavy_deg <= heavy_deg) return SG_OK;
    // (+ the sparse kernel's 256-arc items: <= SG_SPARSE_ARCS / 256 + one per listed word)
    const int64_t cap64 = g->v.nnz / HEAVY_CHUNK + g->v.nnz / heavy_deg + 64 + (1 << 16) / 256 + 4096 + 64;
    if (cap64 > 0xFFFFFFF0ll) return fail(SG_ERR_UNSUPPORTED, "heavy queue too large (heavy_degree too small)");
    cudaFree(ws->heavy);
    ws->heavy = nullptr;
    CK(cudaMalloc(&ws->heavy, sizeof(HeavyItem) * (size_t)cap64));
    ws->heavy_cap = (uint32_t)cap64;
    ws->heavy_deg = heavy_deg;
    // segmented hub queue: sum over hubs of ceil(deg / CHUNK) <= nnz / CHUNK + nhubs
    if (!ws->seg && g->nhubs > 0) {
        const int64_t scap = g->v.nnz / HEAVY_CHUNK + g->nhubs + 64;
        CK(cudaMalloc(&ws->seg, sizeof(SegItem) * (size_t)scap));
        ws->seg_cap = (uint32_t)scap;
    }
    return SG_OK;
}

static void free_ws(Workspace *ws) {
    if (!ws) return;
    const bool arena = ws->fr[0].in_arena;
    for (int i = 0; i < 2; i++) free_frontier_bufs(&ws->fr[i]);
    if (!arena) cudaFree(ws->st);
    cudaFreeHost(ws->h_st);
    cudaFree(ws->visited);
    cudaFree(ws->vis_old);
    cudaFree(ws->dist_old);
    cudaFree(ws->heavy);
    cudaFree(ws->seg);
    cudaFree(ws->all_offsets);
    if (ws->far) {
        free_frontier_bufs(ws->far);
        delete ws->far;
    }
    cudaFree(ws->scratch);
    cudaFreeHost(ws->h_scratch);
    cudaFree(ws->stack);
    cudaFree(ws->exp_of_level);
    cudaFree(ws->delta);
    cudaFree(ws->sigma);
    cudaFree(ws->level);
    if (ws->bfs_exec) cudaGraphExecDestroy(ws->bfs_exec);
    if (ws->bfs_graph) cudaGraphDestroy(ws->bfs_graph);
    {
        BcbLaunch &B = ws->bcb;
        cudaFree(B.F);
        cudaFree(B.V);
        cudaFree(B.M);
        cudaFree(B.VB);
        cudaFree(B.VS);
        cudaFree(B.s);
        cudaFree(B.delta);
        cudaFree(B.lv);
        cudaFree(B.lm);
        cudaFree(B.loff);
        cudaFree(B.maxb);
        cudaFree(B.c);
        cudaFreeHost(ws->h_bcb);
    }
    if (ws->cap_stream) cudaStreamDestroy(ws->cap_stream);
    for (auto &v : ws->vg) {
        if (v.exec) cudaGraphExecDestroy(v.exec);
        if (v.graph) cudaGraphDestroy(v.graph);
    }
    cudaFree(ws->vctrl);
    cudaFreeHost(ws->h_vctrl);
    cudaFree(ws->ctrl);
    cudaFree(ws->bfs_done);
    cudaFree(ws->gbar);
    cudaFreeHost(ws->h_ctrl);
    if (ws->h_res) res_slot_free(ws->h_res);
    if (ws->ev0) cudaEventDestroy(ws->ev0);
    if (ws->ev1) cudaEventDestroy(ws->ev1);
    for (cudaEvent_t e : ws->prof.pool) cudaEventDestroy(e);
    delete ws;
}

static int check_device(const void *p) {
    if (!p) return SG_OK;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return fail(SG_ERR_INVALID, "pointer %p is not a CUDA allocation", p);
    }
    if (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged)
        return fail(SG_ERR_INVALID, "pointer %p is not device memory", p);
    return SG_OK;
}

// ------------------------------------------------------------------------------------------
extern "C" {

SG_API const char *sg_last_error(void) { return t_err.c_str(); }
SG_API const char *sg_version(void) { return "sygraph-b200 0.1 (sm_100a)"; }

SG_API void sg_opts_default(sg_opts *o) {
    if (!o) return;
    memset(o, 0, sizeof *o);
    o->direction = SG_DIR_AUTO;
    o->alpha = 5.0;   // Beamer alpha / beta tuned on B200 (DESIGN R2; profiles/r02_alpha_beta.txt)
    o->beta = 48.0;
}

// ---- 1-D destination partition: bounds, blocks, exchange arena -------------------------------
static size_t al256(size_t x) { return (x + 255) & ~(size_t)255; }

// Allocate the IPC-shared arena, exchange handles over the communicator, map every peer's arena.
static int arena_create(sg_graph *g, cudaStream_t s) {
    Comm &C = g->comm->c;
    const GraphView &G = g->v;
    Arena *A = new Arena();
    g->ar = A;
    size_t off = 0;
    const size_t o_ctl = off;
    off += al256(sizeof(XCtl));
    size_t o_bits[2], o_summ[2], o_off[2];
    for (int i = 0; i < 2; i++) {
        o_bits[i] = off;
        off += al256(sizeof(uint64_t) * (size_t)(G.nw1 + 8));
        o_summ[i] = off;
        off += al256(sizeof(uint64_t) * (size_t)G.nw2);
        o_off[i] = off;
        off += al256(sizeof(uint32_t) * (size_t)G.nw1);
    }
    const size_t o_st = off;
    off += al256(3 * sizeof(DevStats));
    const size_t o_vals = off;
    off += al256(sizeof(uint32_t) * (size_t)(G.n + 4));
    A->bytes = off;
    CK(cudaMalloc(&A->base, A->bytes));   // plain cudaMalloc: exportable through cudaIpcGetMemHandle
    CK(cudaMemsetAsync(A->base, 0, A->bytes, s));
    CK(cudaStreamSynchronize(s));
    char *b = static_cast<char *>(A->base);
    A->ctl = reinterpret_cast<XCtl *>(b + o_ctl);
    for (int i = 0; i < 2; i++) {
        A->bits[i] = reinterpret_cast<uint64_t *>(b + o_bits[i]);
        A->summ[i] = reinterpret_cast<uint64_t *>(b + o_summ[i]);
        A->offsets[i] = reinterpret_cast<uint32_t *>(b + o_off[i]);
    }
    A->st = reinterpret_cast<DevStats *>(b + o_st);
    A->vals = reinterpret_cast<uint32_t *>(b + o_vals);
    struct Hello {
        cudaIpcMemHandle_t h;
        unsigned long long bytes;
        int device;
        int pad;
    } me{}, all[SG_MAX_RANKS];
    CK(cudaIpcGetMemHandle(&me.h, A->base));
    me.bytes = A->bytes;
    me.device = g->device;
    std::string err;
    if (comm_allgather(&C, &me, all, sizeof me, err) != 0) return fail(SG_ERR_NCCL, "arena handle exchange: %s", err.c_str());
    A->x.nranks = C.nranks;
    A->x.rank = C.rank;
    A->x.ctl = A->ctl;
    for (int j = 0; j < C.nranks; j++) {
        if (all[j].bytes != A->bytes) return fail(SG_ERR_INVALID, "ranks disagree on the graph size (arena %llu vs %llu B)",
                                                  (unsigned long long)all[j].bytes, (unsigned long long)A->bytes);
        if (j == C.rank) continue;
        void *p = nullptr;
        const cudaError_t e = cudaIpcOpenMemHandle(&p, all[j].h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(SG_ERR_NCCL, "cudaIpcOpenMemHandle of rank %d's arena (device %d) failed: %s", j, all[j].device,
                        cudaGetErrorString(e));
        }
        A->peer[j] = p;
        A->x.delta[j] = (long long)((char *)p - (char *)A->base);
    }
    // every rank has mapped every peer before any kernel may store into a peer's arena
    int one = 1, ones[SG_MAX_RANKS];
    if (comm_allgather(&C, &one, ones, sizeof one, err) != 0) return fail(SG_ERR_NCCL, "barrier: %s", err.c_str());
    return SG_OK;
}

static void arena_free(sg_graph *g) {
    Arena *A = g->ar;
    if (!A) return;
    for (int j = 0; j < SG_MAX_RANKS; j++)
        if (A->peer[j]) cudaIpcCloseMemHandle(A->peer[j]);
    // no rank frees its arena while a peer still maps it
    if (g->comm) {
        std::string err;
        int one = 1, ones[SG_MAX_RANKS];
        comm_allgather(&g->comm->c, &one, ones, sizeof one, err);
    }
    cudaFree(A->base);
    delete A;
    g->ar = nullptr;
}

// Partition the loaded full CSR (g->rp / col / w) across the communicator: bounds (agreed by
// all ranks), push block + pull block of this rank, exchange arena.
static int partition_graph(sg_graph *g, cudaStream_t s) {
    Comm &C = g->comm->c;
    const int P = C.nranks;
    const int64_t n = g->v.n, nnz = g->v.nnz;
    if (!g->sorted) return fail(SG_ERR_UNSUPPORTED, "a partitioned graph needs sorted rows (binary-searched row parts)");
    int64_t q[SG_MAX_RANKS] = {0};
    CK(part_quantiles(g->rp, n, nnz, P, q, s));
    int64_t bounds[SG_MAX_RANKS + 1];
    bounds[0] = 0;
    for (int r = 1; r < P; r++) {   // partition.py: partition_ranges (ALIGN = 4096)
        int64_t v = (q[r - 1] + 2048) / 4096 * 4096;
        if (v < bounds[r - 1]) v = bounds[r - 1];
        if (v > n) v = n;
        bounds[r] = v;
    }
    bounds[P] = n;
    struct Agree {
        int64_t n, nnz, bounds[SG_MAX_RANKS + 1];
    } me{}, all[SG_MAX_RANKS];
    me.n = n;
    me.nnz = nnz;
    for (int r = 0; r <= P; r++) me.bounds[r] = bounds[r];
    std::string err;
    if (comm_allgather(&C, &me, all, sizeof me, err) != 0) return fail(SG_ERR_NCCL, "partition exchange: %s", err.c_str());
    for (int j = 0; j < P; j++)
        if (memcmp(&all[j], &me, sizeof me) != 0)
            return fail(SG_ERR_INVALID, "rank %d loaded a different graph (n / nnz / partition bounds differ)", j);
    const int64_t lo = bounds[C.rank], hi = bounds[C.rank + 1];
    int64_t *rpp = nullptr, *rpl = nullptr;
    int32_t *colp = nullptr, *coll = nullptr;
    uint8_t *wp = nullptr;
    int64_t nnzp = 0, nnzl = 0;
    CK(part_push_block(g->rp, g->col, g->w, n, lo, hi, &rpp, &colp, &wp, &nnzp, s));
    CK(part_pull_block(g->rp, g->col, n, lo, hi, &rpl, &coll, &nnzl, s));
    if (!g->borrowed) {
        dev_free(g->rp);
        dev_free(g->col);
        dev_free(g->w);
    }
    g->borrowed = false;   // the blocks are the graph's own
    g->rp = rpp;
    g->col = colp;
    g->w = wp;
    g->rpl = rpl;
    g->coll = coll;
    GraphView &V = g->v;
    V.rp = rpp;
    V.col = colp;
    V.w = wp;
    V.nnz = nnzp;
    V.hub_idx = nullptr;   // the hub-segmented tier and the sweep are single-GPU structures
    V.hub_off = nullptr;
    g->scsr_state = -1;
    V.own_lo = lo;
    V.own_hi = hi;
    V.w1_lo = lo / 64;
    V.w1_hi = hi > lo ? (hi + 63) / 64 : lo / 64;
    V.w2_lo = V.w1_lo / 64;
    V.w2_hi = hi > lo ? (V.w1_hi + 63) / 64 : V.w1_lo / 64;
    g->vl = V;
    g->vl.rp = rpl;
    g->vl.col = coll;
    g->vl.w = nullptr;
    g->vl.nnz = nnzl;
    return arena_create(g, s);
}

// bytes readable from p to the end of its allocation (driver allocation range), -1 if unknown
// (cuMemGetAddressRange through cudaGetDriverEntryPoint: the library does not link libcuda)
static long long bytes_to_alloc_end(const void *p) {
    typedef CUresult (*range_fn)(CUdeviceptr *, size_t *, CUdeviceptr);
    static range_fn fn = nullptr;
    if (!fn) {
        void *f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !f) {
            cudaGetLastError();
            return -1;
        }
        fn = (range_fn)f;
    }
    CUdeviceptr base = 0;
    size_t size = 0;
    if (fn(&base, &size, (CUdeviceptr)p) != CUDA_SUCCESS) return -1;
    return (long long)((unsigned long long)base + size - (unsigned long long)p);
}

SG_API int graph_load_csr(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col_idx,
                          const uint8_t *weights, int mem, int flags, void *stream, sg_comm *comm, sg_graph **out) {
    t_err.clear();
    if (!out) return fail(SG_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (n <= 0 || n > 0x7FFFFFFFll) return fail(SG_ERR_INVALID, "n=%lld outside [1, 2^31-1]", (long long)n);
    if (nnz < 0 || nnz > (1ll << 40)) return fail(SG_ERR_INVALID, "nnz=%lld outside [0, 2^40]", (long long)nnz);
    if (!row_ptr || (nnz > 0 && !col_idx)) return fail(SG_ERR_INVALID, "row_ptr/col_idx NULL");
    if (mem != SG_MEM_HOST && mem != SG_MEM_DEVICE) return fail(SG_ERR_INVALID, "mem must be SG_MEM_HOST or SG_MEM_DEVICE");
    if (flags & ~(SG_F_BORROW | SG_F_VALIDATE | SG_F_DIRECTED)) return fail(SG_ERR_INVALID, "unknown flags 0x%x", flags);
    const bool directed = (flags & SG_F_DIRECTED) != 0;
    if (directed && comm && comm->c.nranks > 1)
        return fail(SG_ERR_UNSUPPORTED, "a partitioned graph must be symmetric (SG_F_DIRECTED is single-GPU)");
    const bool borrow = (flags & SG_F_BORROW) != 0;
    if (borrow && mem != SG_MEM_DEVICE) return fail(SG_ERR_INVALID, "SG_F_BORROW needs SG_MEM_DEVICE arrays");
    if (mem == SG_MEM_DEVICE) {
        TRY(check_device(row_ptr));
        TRY(check_device(col_idx));
        TRY(check_device(weights));
    } else {
        if (row_ptr[0] != 0 || row_ptr[n] != nnz) return fail(SG_ERR_INVALID, "row_ptr[0] != 0 or row_ptr[n] != nnz");
    }
    if (borrow) {   // the kernels read 16-B vectors of col_idx (and u32 quads of weights) up to 12 B past nnz
        if (((uintptr_t)col_idx & 15) || ((uintptr_t)row_ptr & 7))
            return fail(SG_ERR_INVALID, "SG_F_BORROW: col_idx must be 16-B aligned, row_ptr 8-B aligned");
        const long long cb = nnz ? bytes_to_alloc_end(col_idx) : 1 << 20;
        const long long wb = weights ? bytes_to_alloc_end(weights) : 1 << 20;
        if (cb < 0 || wb < 0) return fail(SG_ERR_INVALID, "SG_F_BORROW: cannot query the allocation of col_idx/weights");
        if (cb < nnz * 4 + 64 || wb < nnz + 64)
            return fail(SG_ERR_INVALID, "SG_F_BORROW: col_idx / weights allocations need >= 64 readable bytes past nnz");
    }
    cudaStream_t s = (cudaStream_t)stream;
    sg_graph *g = new sg_graph();
    g_live_graphs++;
    CK(cudaGetDevice(&g->device));
    g->v.n = n;
    g->v.nnz = nnz;
    g->v.nw1 = (n + 63) / 64;
    g->v.nw2 = (g->v.nw1 + 63) / 64;
    g->v.own_lo = 0;
    g->v.own_hi = n;
    g->v.w1_lo = 0;
    g->v.w1_hi = g->v.nw1;
    g->v.w2_lo = 0;
    g->v.w2_hi = g->v.nw2;
    g->nnz_global = nnz;
    g->borrowed = borrow;
    const bool part = comm && comm->c.nranks > 1;
    if (part) {
        g->comm = comm;
        g->nranks = comm->c.nranks;
        g->rank = comm->c.rank;
    }
    if (borrow) {
        g->rp = const_cast<int64_t *>(row_ptr);
        g->col = const_cast<int32_t *>(col_idx);
        g->w = const_cast<uint8_t *>(weights);
    } else {
        const cudaMemcpyKind kind = mem == SG_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
        // col_idx/weights get 64 B of zero padding: 16-B bulk copies may read up to 12 B past nnz
        CK(dev_alloc(&g->rp, sizeof(int64_t) * (size_t)(n + 1), s));
        CK(dev_alloc(&g->col, sizeof(int32_t) * (size_t)nnz + 64, s));
        CK(cudaMemsetAsync((char *)g->col + sizeof(int32_t) * (size_t)nnz, 0, 64, s));
        CK(cudaMemcpyAsync(g->rp, row_ptr, sizeof(int64_t) * (size_t)(n + 1), kind, s));
        if (nnz) CK(cudaMemcpyAsync(g->col, col_idx, sizeof(int32_t) * (size_t)nnz, kind, s));
        if (weights) {
            CK(dev_alloc(&g->w, (size_t)nnz + 64, s));
            CK(cudaMemsetAsync(g->w + nnz, 0, 64, s));
            if (nnz) CK(cudaMemcpyAsync(g->w, weights, (size_t)nnz, kind, s));
        }
    }
    g->v.rp = g->rp;
    g->v.col = g->col;
    g->v.w = g->w;
    unsigned long long *dscr = nullptr;
    CK(cudaMalloc(&dscr, 64));
    CK(cudaMemsetAsync(dscr, 0, 64, s));
    // structure first (the derived arrays below index with row_ptr / col_idx)
    launch_validate_csr(g->v, dscr, s);
    unsigned long long hv[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    CK(cudaMemcpyAsync(hv, dscr, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hv[0]) {
        cudaFree(dscr);
        graph_free(g);
        return fail(SG_ERR_INVALID, "CSR validation failed (%llu malformed row_ptr / col_idx entries)", hv[0]);
    }
    launch_row_check(g->v, dscr + 3, s);                           // [3] unsorted pairs, [4] self-loops
    if ((flags & SG_F_VALIDATE) && !directed) launch_symmetry(g->v, dscr + 5, s); // [5] arcs without reverse
    CK(dev_alloc(&g->deg8, (size_t)g->v.nw1 * 64, s));
    launch_deg8(g->rp, n, g->v.nw1 * 64, g->deg8, s);   // out-degree codes (push cost m_f)
    g->v.deg8 = g->deg8;
    g->directed = directed;
    if (directed) {   // pull steps read in-neighbours: the transpose ("CSR and CSC")
        CK(build_csc(g->rp, g->col, n, nnz, &g->rpt, &g->colt, s));
    }
    const int64_t *prp = directed ? g->rpt : g->rp;    // rows a pull step scans
    const int32_t *pcol = directed ? g->colt : g->col;
    CK(dev_alloc(&g->isolated, sizeof(uint64_t) * (size_t)g->v.nw1, s));
    if (directed) {   // unreachable = no in-arc (a directed vertex with out-arcs only is never reached)
        uint8_t *indeg8 = nullptr;
        CK(dev_alloc(&indeg8, (size_t)g->v.nw1 * 64, s));
        launch_deg8(prp, n, g->v.nw1 * 64, indeg8, s);
        launch_isolated(indeg8, n, g->v.nw1, g->isolated, s);
        CK(cudaFreeAsync(indeg8, s));
    } else {
        launch_isolated(g->deg8, n, g->v.nw1, g->isolated, s);
    }
    launch_popcount(g->isolated, g->v.nw1, dscr + 6, s);           // [6] isolated vertices
    CK(dev_alloc(&g->fnbr, sizeof(int32_t) * (size_t)(g->v.nw1 ? g->v.nw1 * 64 : 1), s));   // padded: 16-B quad loads
    launch_first_nbr(prp, pcol, g->deg8, n, g->v.nw1 * 64, g->fnbr, s);
    g->v.fnbr = g->fnbr;
    if (g->w) launch_max_weight(g->w, nnz, reinterpret_cast<unsigned int *>(dscr + 1), s);
    // hubs of the destination-segmented BFS tier (deg >= SEG_MIN): index map + vertex list
    const int64_t max_hubs = nnz / SEG_MIN + 1;
    CK(dev_alloc(&g->hub_idx, sizeof(int32_t) * (size_t)n, s));
    CK(dev_alloc(&g->hub_vertex, sizeof(int32_t) * (size_t)max_hubs, s));
    launch_hub_mark(g->rp, n, g->hub_idx, g->hub_vertex, reinterpret_cast<unsigned int *>(dscr + 2), s);
    CK(cudaMemcpyAsync(hv, dscr, 64, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    CK(cudaGetLastError());
    cudaFree(dscr);
    g->max_w = (uint32_t)(hv[1] & 0xffffffffu);
    g->n_iso = (int64_t)hv[6];
    if ((flags & SG_F_VALIDATE) && (hv[3] || hv[4] || hv[5])) {
        graph_free(g);
        return fail(SG_ERR_INVALID, "CSR validation failed: %llu unsorted/duplicate pairs, %llu self-loops, %llu arcs "
                    "without their reverse (rows must be strictly ascending, simple, symmetric)", hv[3], hv[4], hv[5]);
    }
    g->sorted = hv[3] == 0;
    if (!g->sorted) g->scsr_state = -1;   // the segment-major copy needs sorted rows
    g->nhubs = (int64_t)(hv[2] & 0xffffffffu);
    g->v.nseg = (int32_t)((n + SEG_V - 1) / SEG_V);
    if (part) {
        g->nhubs = 0;
        const int r = partition_graph(g, s);
        if (r != SG_OK) {
            const std::string msg = t_err;
            graph_free(g);
            t_err = msg;
            return r;
        }
    }
    if (g->nhubs > 0 && g->sorted) {   // hub segment offsets binary-search sorted rows
        CK(dev_alloc(&g->hub_off, sizeof(uint32_t) * (size_t)g->nhubs * (size_t)(g->v.nseg + 1), s));
        launch_hub_off(g->rp, g->col, g->hub_vertex, g->nhubs, g->v.nseg, g->hub_off, s);
        CK(cudaStreamSynchronize(s));
        CK(cudaGetLastError());
        g->v.hub_idx = g->hub_idx;
        g->v.hub_off = g->hub_off;
    }
    if (!part) g->vl = g->v;
    if (directed) {   // pull view: the CSC (in-neighbour rows), same frontier layout and degree codes
        g->vl.rp = g->rpt;
        g->vl.col = g->colt;
        g->vl.w = nullptr;
        g->vl.hub_idx = nullptr;
        g->vl.hub_off = nullptr;
    }
    *out = g;
    return SG_OK;
}

SG_API int graph_free(sg_graph *g) {
    if (!g) return SG_OK;
    cudaDeviceSynchronize();   // no pending work may use the buffers (cudaFree did this implicitly)
    free_ws(g->ws);
    g->ws = nullptr;
    arena_free(g);
    dev_free(g->rpl);
    dev_free(g->coll);
    dev_free(g->rpt);
    dev_free(g->colt);
    if (!g->borrowed) {
        dev_free(g->rp);
        dev_free(g->col);
        dev_free(g->w);
    }
    dev_free(g->deg8);
    dev_free(g->fnbr);
    dev_free(g->isolated);
    dev_free(g->hub_idx);
    dev_free(g->hub_vertex);
    dev_free(g->hub_off);
    dev_free(g->cbo);
    ccb_free(&g->ccb);
    if (g->scsr_state == 1) scsr_free(&g->scsr);
    delete g;
    if (--g_live_graphs == 0) {   // the last graph: give the pool's memory back to the device
        cudaDeviceSynchronize();
        dev_trim(0);
    }
    return SG_OK;
}

SG_API int graph_info(const sg_graph *g, int64_t *n, int64_t *nnz, const int64_t **row_ptr, const int32_t **col_idx,
                      const uint8_t **weights) {
    if (!g) return fail(SG_ERR_INVALID, "graph is NULL");
    if (n) *n = g->v.n;
    if (nnz) *nnz = g->v.nnz;
    if (row_ptr) *row_ptr = g->rp;
    if (col_idx) *col_idx = g->col;
    if (weights) *weights = g->w;
    return SG_OK;
}

SG_API int graph_partition(const sg_graph *g, int64_t *lo, int64_t *hi) {
    if (!g) return fail(SG_ERR_INVALID, "graph is NULL");
    if (lo) *lo = g->v.own_lo;
    if (hi) *hi = g->v.own_hi;
    return SG_OK;
}

// ---- communicator ---------------------------------------------------------------------------
SG_API int comm_unique_id(uint8_t id[128]) {
    t_err.clear();
    if (!id) return fail(SG_ERR_INVALID, "id is NULL");
    std::string err;
    if (comm_create_id(id, err) != 0) return fail(SG_ERR_NCCL, "comm_unique_id: %s", err.c_str());
    return SG_OK;
}

SG_API int comm_init(const uint8_t id[128], int nranks, int rank, int device, sg_comm **out) {
    t_err.clear();
    if (!id || !out) return fail(SG_ERR_INVALID, "NULL argument");
    *out = nullptr;
    if (nranks < 1 || nranks > SG_MAX_RANKS || rank < 0 || rank >= nranks)
        return fail(SG_ERR_INVALID, "nranks %d / rank %d outside [1, %d] / [0, nranks)", nranks, rank, SG_MAX_RANKS);
    sg_comm *c = new sg_comm();
    c->c.device = device;
    std::string err;
    if (nranks > 1 && comm_connect(&c->c, id, nranks, rank, err) != 0) {
        comm_close(&c->c);
        delete c;
        return fail(SG_ERR_NCCL, "comm_init: %s", err.c_str());
    }
    c->c.nranks = nranks;
    c->c.rank = rank;
    *out = c;
    return SG_OK;
}

SG_API int comm_free(sg_comm *c) {
    if (!c) return SG_OK;
    comm_close(&c->c);
    delete c;
    return SG_OK;
}

SG_API int comm_info(const sg_comm *c, int *nranks, int *rank) {
    if (!c) return fail(SG_ERR_INVALID, "comm is NULL");
    if (nranks) *nranks = c->c.nranks;
    if (rank) *rank = c->c.rank;
    return SG_OK;
}

// ---- frontier ----------------------------------------------------------------------------
SG_API int frontier_init(const sg_graph *g, sg_frontier **out) {
    t_err.clear();
    if (!g || !out) return fail(SG_ERR_INVALID, "NULL argument");
    sg_frontier *f = new sg_frontier();
    int r = alloc_frontier_bufs(f, g, true);
    if (r != SG_OK) {
        free_frontier_bufs(f);
        delete f;
        return r;
    }
    *out = f;
    return SG_OK;
}

SG_API int frontier_free(sg_frontier *f) {
    if (!f) return SG_OK;
    free_frontier_bufs(f);
    delete f;
    return SG_OK;
}

SG_API int frontier_insert(sg_frontier *f, const int32_t *v, int64_t k, int mem, void *stream) {
    t_err.clear();
    if (!f || (k > 0 && !v) || k < 0) return fail(SG_ERR_INVALID, "bad frontier_insert arguments");
    if (k == 0) return SG_OK;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = f->g->v.n;
    if (mem == SG_MEM_HOST) {
        for (int64_t i = 0; i < k; i++)
            if (v[i] < 0 || v[i] >= n) return fail(SG_ERR_INVALID, "vertex %d outside [0,%lld)", v[i], (long long)n);
        int32_t *d = nullptr;
        CK(cudaMallocAsync(&d, sizeof(int32_t) * (size_t)k, s));
        CK(cudaMemcpyAsync(d, v, sizeof(int32_t) * (size_t)k, cudaMemcpyHostToDevice, s));
        launch_insert(f->bits, f->summ, d, k, n, s);
        CK(cudaFreeAsync(d, s));
        CK(cudaStreamSynchronize(s));   // the host array may be released by the caller
    } else if (mem == SG_MEM_DEVICE) {
        launch_insert(f->bits, f->summ, v, k, n, s);
    } else {
        return fail(SG_ERR_INVALID, "bad mem");
    }
    CK(cudaGetLastError());
    return SG_OK;
}

SG_API int frontier_fill_all(sg_frontier *f, void *stream) {
    if (!f) return fail(SG_ERR_INVALID, "NULL frontier");
    const GraphView &g = f->g->v;
    launch_fill_all(f->bits, f->summ, g.n, g.nw1, g.nw2, (cudaStream_t)stream);
    CK(cudaGetLastError());
    return SG_OK;
}

static int clear_frontier(sg_frontier *f, cudaStream_t s) {
    const GraphView &g = f->g->v;
    CK(cudaMemsetAsync(f->bits, 0, sizeof(uint64_t) * (size_t)g.nw1, s));
    CK(cudaMemsetAsync(f->summ, 0, sizeof(uint64_t) * (size_t)g.nw2, s));
    return SG_OK;
}

SG_API int frontier_clear(sg_frontier *f, void *stream) {
    if (!f) return fail(SG_ERR_INVALID, "NULL frontier");
    return clear_frontier(f, (cudaStream_t)stream);
}

SG_API int frontier_count(const sg_frontier *f, int64_t *out, void *stream) {
    if (!f || !out) return fail(SG_ERR_INVALID, "NULL argument");
    cudaStream_t s = (cudaStream_t)stream;
    unsigned long long *d = nullptr, h = 0;
    CK(cudaMallocAsync(&d, sizeof(unsigned long long), s));
    CK(cudaMemsetAsync(d, 0, sizeof(unsigned long long), s));
    launch_popcount(f->bits, f->g->v.nw1, d, s);
    CK(cudaMemcpyAsync(&h, d, sizeof h, cudaMemcpyDeviceToHost, s));
    CK(cudaFreeAsync(d, s));
    CK(cudaStreamSynchronize(s));
    CK(cudaGetLastError());
    *out = (int64_t)h;
    return SG_OK;
}

SG_API int frontier_view(const sg_frontier *f, uint64_t **bits, uint64_t **summ, int64_t *nw1, int64_t *nw2) {
    if (!f) return fail(SG_ERR_INVALID, "NULL frontier");
    if (bits) *bits = f->bits;
    if (summ) *summ = f->summ;
    if (nw1) *nw1 = f->g->v.nw1;
    if (nw2) *nw2 = f->g->v.nw2;
    return SG_OK;
}

SG_API int frontier_op(sg_frontier *dst, const sg_frontier *src, int op, void *stream) {
    if (!dst || !src || dst->g->v.n != src->g->v.n || op < 0 || op > 3)
        return fail(SG_ERR_INVALID, "bad frontier_op arguments");
    cudaStream_t s = (cudaStream_t)stream;
    const GraphView &g = dst->g->v;
    launch_setop(dst->bits, src->bits, g.nw1, op, s);
    launch_rebuild_summary(dst->bits, dst->summ, g.nw1, g.nw2, s);
    CK(cudaGetLastError());
    return SG_OK;
}

SG_API int frontier_filter(sg_frontier *in, sg_frontier *out, int pred, const void *array, double a, double b,
                           void *stream) {
    t_err.clear();
    if (!in || pred < SG_PRED_DEGREE_RANGE || pred > SG_PRED_IN_BITMAP) return fail(SG_ERR_INVALID, "bad filter arguments");
    if (pred != SG_PRED_DEGREE_RANGE && !array) return fail(SG_ERR_INVALID, "predicate needs an array");
    if (out && out->g->v.n != in->g->v.n) return fail(SG_ERR_INVALID, "frontiers of different graphs");
    const GraphView &g = in->g->v;
    if (out && out != in)
        launch_filter(g, in->bits, out->bits, out->summ, pred, array, a, b, 0, (cudaStream_t)stream);
    else
        launch_filter(g, in->bits, in->bits, in->summ, pred, array, a, b, 1, (cudaStream_t)stream);
    CK(cudaGetLastError());
    return SG_OK;
}

SG_API int compute_execute(const sg_frontier *f, int op, void *array, double value, void *stream) {
    t_err.clear();
    if (!f || !array || op < SG_OP_SET_U32 || op > SG_OP_ADD_F64) return fail(SG_ERR_INVALID, "bad compute arguments");
    launch_compute(f->g->v, f->bits, op, array, value, (cudaStream_t)stream);
    CK(cudaGetLastError());
    return SG_OK;
}

SG_API int frontier_or_into(const sg_frontier *f, uint64_t *dst, void *stream) {
    if (!f || !dst) return fail(SG_ERR_INVALID, "NULL argument");
    launch_or_all(f->bits, f->g->v.nw1, dst, (cudaStream_t)stream);
    CK(cudaGetLastError());
    return SG_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------------------------
// L2 residency for the array every arc probes (CC labels): a persisting access-policy window on
// the stream for the duration of a run_* call, so the col_idx stream does not evict it (B200:
// 126 MB L2, 82.9 MB persisting carve-out).  Measured on config 3 it is SLOWER (18.2 vs 13.0 ms:
// the carve-out shrinks the L2 left for everything else), so it is opt-in (SG_L2PIN=1) and kept
// for the record.  Best effort: errors ignored.
struct L2Pin {
    cudaStream_t s;
    bool on = false;
    L2Pin(const void *p, size_t bytes, cudaStream_t st) : s(st) {
        if (!getenv("SG_L2PIN")) return;
        int dev = 0, maxp = 0, maxw = 0;
        if (cudaGetDevice(&dev) != cudaSuccess) return;
        cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
        cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev);
        if (maxp <= 0 || maxw <= 0 || !p || !bytes) return;
        size_t limit = 0;
        cudaDeviceGetLimit(&limit, cudaLimitPersistingL2CacheSize);
        if (limit < (size_t)maxp) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp);
        cudaStreamAttrValue a = {};
        a.accessPolicyWindow.base_ptr = const_cast<void *>(p);
        a.accessPolicyWindow.num_bytes = bytes < (size_t)maxw ? bytes : (size_t)maxw;
        const double ratio = (double)maxp / (double)a.accessPolicyWindow.num_bytes;
        a.accessPolicyWindow.hitRatio = (float)(ratio < 1.0 ? ratio : 1.0);
        a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        on = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &a) == cudaSuccess;
        cudaGetLastError();
    }
    ~L2Pin() {
        if (!on) return;
        cudaStreamAttrValue a = {};
        a.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &a);
        cudaCtxResetPersistingL2Cache();
        cudaGetLastError();
    }
};

// ------------------------------------------------------------------------------------------
// superstep helpers
struct Tiers {
    int32_t heavy, small;
    int32_t seg;   // destination-segmented hub tier for BFS: 0 off, 1 auto, 2 always
    int32_t cf;    // words per warp grab (coarsening factor); 0 = auto
    int32_t scsr;  // BFS push over the segment-major arc copy: 0 off, 1 auto (m_f >= threshold), 2 always
};
// auto mode: the sweep (scsr.cu) takes a push superstep whose estimated frontier arcs reach
// SG_SWEEP_FRAC64/64 of all arcs (it streams every arc of each active 4096-vertex unit, so it
// pays only when most arcs are active); the copy is built only for graphs of at least
// SG_SWEEP_MIN_M Mi arcs unless forced (scsr = 2)
#ifndef SG_SWEEP_FRAC64
#define SG_SWEEP_FRAC64 32
#endif
#ifndef SG_SWEEP_MIN_M
#define SG_SWEEP_MIN_M 16
#endif
static unsigned long long env_or(const char *name, long long dflt) {
    const char *e = getenv(name);
    return (unsigned long long)(e ? atoll(e) : dflt);
}
static unsigned long long sweep_threshold(int64_t nnz) {
    const unsigned long long f = env_or("SG_SWEEP_FRAC64", SG_SWEEP_FRAC64);
    const unsigned long long t = (unsigned long long)nnz * f / 64ull;
    return t ? t : 1ull;
}
// auto mode: the segmented tier pays for its per-segment slice loads only on heavy supersteps
#ifndef SG_SEG_THRESHOLD_M
#define SG_SEG_THRESHOLD_M 8   // (32 in r01; 8: an 18 M-arc level-2 hub push 133 -> 121 us)
#endif
static const unsigned long long kSegThreshold = (unsigned long long)SG_SEG_THRESHOLD_M << 20;   // est. frontier arcs

static Tiers tiers_from(const sg_opts *o) {
    Tiers t{kDefaultHeavy, kDefaultSmall, 1, 0, 1};
    if (o && o->coarsening > 0) t.cf = o->coarsening > 64 ? 64 : o->coarsening;
    if (o && o->heavy_degree > 0) t.heavy = o->heavy_degree;
    if (o && o->small_degree > 0) t.small = o->small_degree;
    if (o && o->small_degree < 0) t.small = 0;           // no thread tier
    if (t.small > t.heavy) t.small = t.heavy;
    if (o) t.seg = o->segmented == 1 ? 0 : (o->segmented == 2 ? 2 : 1);
    if (o) t.scsr = o->scsr == 1 ? 0 : (o->scsr == 2 ? 2 : 1);
    return t;
}

// zero the control block, compact the summary layer into offsets, optional n_f / m_f
static int compact(const sg_graph *g, const sg_frontier *f, bool stats, cudaStream_t s) {
    CK(cudaMemsetAsync(f->st, 0, sizeof(DevStats), s));
    launch_compact(f->summ, g->v.nw2, f->offsets, f->st, s);
    if (stats) launch_frontier_stats(g->v, f->bits, f->st, s);
    return SG_OK;
}

static PushLaunch push_launch(const sg_graph *g, const sg_frontier *in, Tiers t, int64_t count_hint) {
    PushLaunch L;
    L.g = g->v;
    L.in_bits = in->bits;
    L.offsets = in->offsets;
    L.st = in->st;
    L.heavy = g->ws->heavy;
    L.heavy_cap = g->ws->heavy_cap;
    L.heavy_deg = t.heavy;
    L.small_deg = t.small;
    const int maxg = push_max_grid_words();
    // batch = words per warp grab (coarsening factor): ~4 grabs per warp, 1..8 words
    if (count_hint < 0) {
        L.batch = 4;
        L.grid_words = maxg;
    } else {
        int64_t cf = count_hint / ((int64_t)maxg * 8 * 4);
        if (cf < 1) cf = 1;
        if (cf > 8) cf = 8;
        L.batch = (int32_t)cf;
        int64_t gw = (count_hint + 8 * L.batch - 1) / (8 * L.batch);
        if (gw < 1) gw = 1;
        if (gw > maxg) gw = maxg;
        L.grid_words = (int)gw;
    }
    if (t.cf > 0) {
        L.batch = t.cf;
        if (count_hint >= 0) {
            int64_t gw = (count_hint + 8 * L.batch - 1) / (8 * L.batch);
            L.grid_words = (int)(gw < 1 ? 1 : (gw > maxg ? maxg : gw));
        }
    }
    L.grid_heavy = push_max_grid_heavy();
    L.seg = g->ws->seg;
    L.seg_cap = g->ws->seg_cap;
    L.seg_mode = g->v.hub_idx ? t.seg : 0;
    L.seg_threshold = kSegThreshold;
    return L;
}

static int read_stats(Workspace *ws, cudaStream_t s) {
    CK(cudaMemcpyAsync(ws->h_st, ws->st, 3 * sizeof(DevStats), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    CK(cudaGetLastError());
    return SG_OK;
}

static cudaEvent_t prof_event(Prof &P) {
    if (P.used == P.pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        P.pool.push_back(e);
    }
    return P.pool[P.used++];
}
// returns the record index (or -1 when profiling is off)
static int prof_begin(Workspace *ws, int cls, cudaStream_t s) {
    Prof &P = ws->prof;
    if (!P.on) return -1;
    ProfRec r{cls, prof_event(P), prof_event(P), 0.0};
    if (!r.a || !r.b) return -1;
    cudaEventRecord(r.a, s);
    P.recs.push_back(r);
    return (int)P.recs.size() - 1;
}
static void prof_end(Workspace *ws, int idx, cudaStream_t s) {
    if (idx >= 0) cudaEventRecord(ws->prof.recs[idx].b, s);
}
static void prof_bytes(Workspace *ws, int idx, double bytes) {
    if (idx >= 0) ws->prof.recs[idx].bytes = bytes;
}
// after the stream is synchronised: fold the records into the per-class totals
static void prof_flush(Workspace *ws) {
    Prof &P = ws->prof;
    for (const ProfRec &r : P.recs) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, r.a, r.b) == cudaSuccess) {
            P.ms[r.cls] += ms;
            P.bytes[r.cls] += r.bytes;
            P.launches[r.cls] += 1;
        }
    }
    cudaGetLastError();
    P.recs.clear();
    P.used = 0;
}

static unsigned long long *ws_scratch(sg_graph *g) { return g->ws->scratch; }

static cudaStream_t stream_of(const sg_opts *o) { return o ? (cudaStream_t)o->stream : (cudaStream_t)0; }

extern "C" {

// ---- generic advance ---------------------------------------------------------------------
SG_API int advance(const sg_graph *gc, const sg_frontier *in, sg_frontier *out, int functor, const void *state,
                   void *stream) {
    t_err.clear();
    if (!gc || !in || !state) return fail(SG_ERR_INVALID, "NULL argument");
    if (gc->ar) return fail(SG_ERR_UNSUPPORTED, "advance on a partitioned graph: use run_bfs / run_sssp / run_cc");
    if (in->g != gc || (out && out->g != gc)) return fail(SG_ERR_INVALID, "frontier belongs to another graph");
    sg_graph *g = const_cast<sg_graph *>(gc);
    cudaStream_t s = (cudaStream_t)stream;
    TRY(ensure_ws(g));
    const Tiers t{kDefaultHeavy, kDefaultSmall};
    TRY(ensure_heavy(g, t.heavy));
    TRY(compact(g, in, false, s));
    const PushLaunch L = push_launch(g, in, t, -1);
    uint64_t *ob = out ? out->bits : nullptr, *os = out ? out->summ : nullptr;
    switch (functor) {
        case SG_FN_BFS: {
            const sg_bfs_state *st = (const sg_bfs_state *)state;
            if (!st->level || !st->visited) return fail(SG_ERR_STATE, "BFS state needs level and visited");
            launch_push_bfs(L, BfsArgs{st->visited, st->level, st->depth + 1, ob, os}, s);
            break;
        }
        case SG_FN_SSSP: {
            const sg_sssp_state *st = (const sg_sssp_state *)state;
            if (!st->dist) return fail(SG_ERR_STATE, "SSSP state needs dist");
            if (!g->w) return fail(SG_ERR_INVALID, "SSSP needs graph weights");
            launch_push_sssp(L, SsspArgs{st->dist, ob, os}, s);
            break;
        }
        case SG_FN_CC: {
            const sg_cc_state *st = (const sg_cc_state *)state;
            if (!st->label) return fail(SG_ERR_STATE, "CC state needs label");
            launch_push_cc(L, CcArgs{st->label, ob, os}, s);
            break;
        }
        case SG_FN_BC_SIGMA: {
            const sg_bc_state *st = (const sg_bc_state *)state;
            if (!st->level || !st->visited || !st->sigma || !st->exp2_per_level)
                return fail(SG_ERR_STATE, "BC state needs level, visited, sigma and exp2_per_level");
            if (!out) return fail(SG_ERR_STATE, "BC sigma advance needs an output frontier");
            launch_push_bc(L, BcArgs{st->visited, st->sigma, st->level, st->depth + 1, ob, os}, s);
            // finish level depth+1 (reading C20): scale it by 2^-k, k = floor(log2 max sigma), and
            // record E[depth+1] = E[depth] + k (bc.cu; the output holds exactly the new level)
            TRY(compact(g, out, false, s));
            unsigned long long *d_max = ws_scratch(g) + 4;
            CK(cudaMemsetAsync(d_max, 0, sizeof(unsigned long long), s));
            launch_bc_level_max(st->sigma, out->bits, out->offsets, out->st, g->v.nw1, d_max, s);
            launch_bc_level_scale_and_stack(st->sigma, out->bits, out->offsets, out->st, g->v.nw1, d_max,
                                            st->exp2_per_level, st->depth + 1, nullptr, nullptr, ws_scratch(g) + 5, s);
            break;
        }
        default:
            return fail(SG_ERR_INVALID, "unknown functor %d", functor);
    }
    CK(cudaGetLastError());
    return SG_OK;
}

}  // extern "C"

// ---- CUDA-graph driven BFS (no host round trip per superstep; ctrl.cu) -------------------
static int capture_begin(cudaStream_t cs, cudaGraph_t graph, const std::vector<cudaGraphNode_t> &deps) {
    CK(cudaStreamBeginCaptureToGraph(cs, graph, deps.empty() ? nullptr : deps.data(), nullptr, deps.size(),
                                     cudaStreamCaptureModeRelaxed));
    return SG_OK;
}
static int capture_end(cudaStream_t cs, std::vector<cudaGraphNode_t> &leaves) {
    cudaStreamCaptureStatus cst;
    const cudaGraphNode_t *d = nullptr;
    size_t nd = 0;
    CK(cudaStreamGetCaptureInfo(cs, &cst, nullptr, nullptr, &d, &nd));
    leaves.assign(d, d + nd);
    cudaGraph_t gout;
    CK(cudaStreamEndCapture(cs, &gout));
    return SG_OK;
}
// add a conditional node (IF / WHILE) after `deps`; returns its body graph
static int add_cond(cudaGraph_t graph, const std::vector<cudaGraphNode_t> &deps, cudaGraphConditionalHandle h,
                    cudaGraphConditionalNodeType type, cudaGraphNode_t *node, cudaGraph_t *body) {
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = type;
    p.conditional.size = 1;
    CK(cudaGraphAddNode(node, graph, deps.empty() ? nullptr : deps.data(), deps.size(), &p));
    *body = p.conditional.phGraph_out[0];
    return SG_OK;
}

// The segment-major arc copy (scsr.cu), built at the first run_bfs that uses it: when forced
// (scsr = 2) or for a push-only BFS.  A direction-optimising BFS pulls its dense supersteps, so
// in auto mode it never builds the copy (~13 ms and 4 GB at config 4, which would otherwise land
// inside whichever BFS first met a dense push superstep); it uses the copy if a push-only BFS of
// the same graph built it.  A graph whose segment blocks would
// exceed 2^32 arcs, whose rows are not sorted, or for which the memory is not available keeps
// the word path (the copy is a performance structure only).
static bool sweep_size_ok(const sg_graph *g) {
    return (unsigned long long)g->v.nnz >= (env_or("SG_SWEEP_MIN_M", SG_SWEEP_MIN_M) << 20);
}
static bool scsr_ready(sg_graph *g, const Tiers &t, bool want_now, cudaStream_t s) {
    if (t.scsr == 0) return false;
    if (g->scsr_state == 0) {
        if (t.scsr == 1 && !sweep_size_ok(g)) return false;
        if (t.scsr == 1 && !want_now) return false;   // auto: only a push-only BFS builds it
        const int32_t sw = (int32_t)env_or("SG_SCSR_WORDS", 0);   // test knob: narrower segments (0: 16,384 words)
        const cudaError_t e = scsr_build(g->rp, g->col, g->v.n, g->v.nnz, sw, &g->scsr, s);
        if (e != cudaSuccess) {
            cudaGetLastError();
            g->scsr_state = -1;
        } else {
            g->scsr_state = 1;
        }
    }
    return g->scsr_state == 1;
}

static int build_bfs_graph(sg_graph *g, Tiers t) {
    Workspace *ws = g->ws;
    const GraphView &G = g->v;
    if (ws->bfs_exec) cudaGraphExecDestroy(ws->bfs_exec);
    if (ws->bfs_graph) cudaGraphDestroy(ws->bfs_graph);
    ws->bfs_exec = nullptr;
    ws->bfs_graph = nullptr;
    if (!ws->cap_stream) CK(cudaStreamCreateWithFlags(&ws->cap_stream, cudaStreamNonBlocking));
    if (!ws->ctrl) {
        CK(cudaMalloc(&ws->ctrl, sizeof(BfsCtrl)));
        CK(cudaMallocHost(&ws->h_ctrl, sizeof(BfsCtrl)));
        TRY(res_slot_alloc(&ws->h_res, &ws->d_res));
    }
    cudaStream_t cs = ws->cap_stream;
    cudaGraph_t root;
    CK(cudaGraphCreate(&root, 0));
    ws->bfs_graph = root;
    cudaGraphConditionalHandle h_loop, h_push[2], h_pull[2], h_sweep[2], h_sparse[2] = {};
    // the fused small-frontier loop's IF nodes exist only when it is enabled (SG_SPARSE=1): an
    // untaken IF still costs ~0.4 us per superstep
    const bool sp = env_or("SG_SPARSE", 0) != 0;
    const bool sc = t.scsr != 0 && g->scsr_state == 1;
    CK(cudaGraphConditionalHandleCreate(&h_loop, root, 0, cudaGraphCondAssignDefault));
    for (int i = 0; i < 2; i++) {
        CK(cudaGraphConditionalHandleCreate(&h_push[i], root, 0, cudaGraphCondAssignDefault));
        CK(cudaGraphConditionalHandleCreate(&h_pull[i], root, 0, cudaGraphCondAssignDefault));
        if (sc) CK(cudaGraphConditionalHandleCreate(&h_sweep[i], root, 0, cudaGraphCondAssignDefault));
        if (sp) CK(cudaGraphConditionalHandleCreate(&h_sparse[i], root, 0, cudaGraphCondAssignDefault));
    }
    sg_frontier *F[2] = {&ws->fr[0], &ws->fr[1]};
    std::vector<cudaGraphNode_t> leaves;
    // prologue: level = INF, frontiers cleared, visited = isolated, seed src, compact + decide
    TRY(capture_begin(cs, root, {}));
    // (the output frontier F[1] is written whole by the first output kernel: only F[0] is zeroed)
    const bool pro_node = !g->ar && env_or("SG_PRO_PARAMS", 1) != 0;
    ws->pro_node = nullptr;
    if (pro_node) {   // single GPU: one kernel node (memsets / copies folded in; init as its parameter)
        BfsProArgs &pa = ws->pro_args;
        pa.c = ws->ctrl;
        pa.n = G.n;
        pa.nw1 = G.nw1;
        pa.nw2 = G.nw2;
        pa.deg8 = G.deg8;
        pa.isolated = g->isolated;
        pa.bits = F[0]->bits;
        pa.summ = F[0]->summ;
        pa.offsets = F[0]->offsets;
        pa.st = F[0]->st;
        pa.st_out = F[1]->st;
        pa.visited = ws->visited;
        pa.vis_old = ws->vis_old;
        cudaKernelNodeParams kp;
        bfs_prologue1_node(&pa, ws->pro_slot, &kp);
        TRY(capture_end(cs, leaves));   // (nothing captured)
        CK(cudaGraphAddKernelNode(&ws->pro_node, root, nullptr, 0, &kp));
        leaves = {ws->pro_node};
    } else {
        CK(cudaMemsetAsync(F[0]->bits, 0, sizeof(uint64_t) * (size_t)G.nw1, cs));
        CK(cudaMemsetAsync(F[0]->summ, 0, sizeof(uint64_t) * (size_t)G.nw2, cs));
        CK(cudaMemsetAsync(ws->st, 0, 2 * sizeof(DevStats), cs));
        CK(cudaMemcpyAsync(ws->visited, g->isolated, sizeof(uint64_t) * (size_t)G.nw1, cudaMemcpyDeviceToDevice, cs));
        CK(cudaMemcpyAsync(ws->vis_old, g->isolated, sizeof(uint64_t) * (size_t)G.nw1, cudaMemcpyDeviceToDevice, cs));
        launch_bfs_prologue(ws->ctrl, G.n, G.deg8, F[0]->bits, F[0]->summ, F[0]->offsets, F[0]->st, ws->visited,
                            ws->vis_old, g->ar ? g->ar->x : Xchg{}, cs);
    }
    // the handles go to the device with every run's control block (run_bfs_graph)
    ws->hnd[0] = (unsigned long long)h_loop;
    for (int i = 0; i < 2; i++) {
        ws->hnd[1 + i] = (unsigned long long)h_push[i];
        ws->hnd[3 + i] = (unsigned long long)h_pull[i];
        ws->hnd[5 + i] = sc ? (unsigned long long)h_sweep[i] : 0ull;
        ws->hnd[7 + i] = sp ? (unsigned long long)h_sparse[i] : 0ull;
    }
    if (!pro_node) TRY(capture_end(cs, leaves));
    cudaGraphNode_t wnode;
    cudaGraph_t body;
    TRY(add_cond(root, leaves, h_loop, cudaGraphCondTypeWhile, &wnode, &body));
    // body: superstep A->B then B->A
    std::vector<cudaGraphNode_t> deps;
    for (int half = 0; half < 2; half++) {
        sg_frontier *in = F[half], *out = F[half ^ 1];
        cudaGraphNode_t n_push, n_pull;
        cudaGraph_t b_push, b_pull;
        TRY(add_cond(body, deps, h_push[half], cudaGraphCondTypeIf, &n_push, &b_push));
        TRY(add_cond(body, deps, h_pull[half], cudaGraphCondTypeIf, &n_pull, &b_pull));
        cudaGraphNode_t n_sweep = nullptr, n_sparse = nullptr;
        cudaGraph_t b_sweep = nullptr, b_sparse = nullptr;
        if (sc) TRY(add_cond(body, deps, h_sweep[half], cudaGraphCondTypeIf, &n_sweep, &b_sweep));
        if (sp) TRY(add_cond(body, deps, h_sparse[half], cudaGraphCondTypeIf, &n_sparse, &b_sparse));
        PushLaunch L = push_launch(g, in, t, -1);
        L.batch = t.cf;   // 0: coarsening factor computed on the device from the count
        L.sparse_ok = 1;  // n_f of every BFS frontier is exact (prologue statistics / output kernels)
        BfsArgs a{ws->visited, nullptr, 0u, nullptr, nullptr, &ws->ctrl->next, &ws->ctrl->level, 1u};
        // output of the superstep (out->st was zeroed by the previous decision / the prologue);
        // the output kernel's last CTA decides the next superstep (handles of the other half)
        BfsOut bo{ws->vis_old, out->bits, out->summ, out->offsets, nullptr, 0u, &ws->ctrl->next,
                  &ws->ctrl->level, out->st, ws->ctrl, in->st, ws->bfs_done};
        if (g->ar) bo.x = g->ar->x;   // partitioned: owned slice replicated to the peers + barrier
        else bo.rp = G.rp, bo.col = G.col, bo.visited = ws->visited;   // dead-end lookahead
        bo.half = half;
        TRY(capture_begin(cs, b_push, {}));
        launch_push_bfs(L, a, cs);
        launch_bfs_diff(G, ws->visited, bo, cs);
        TRY(capture_end(cs, leaves));
        if (sc) {   // dense push supersteps (m_f >= threshold) take the sweep instead
            TRY(capture_begin(cs, b_sweep, {}));
            launch_push_sweep(g->scsr.v, G.rp, in->bits, in->summ, in->offsets, G.nw2, in->st, ws->visited, 0ull, cs);
            launch_bfs_diff(G, ws->visited, bo, cs);
            TRY(capture_end(cs, leaves));
        }
        TRY(capture_begin(cs, b_pull, {}));
        launch_pull_bfs(g->vl, in->bits, ws->visited, in->st, bo, cs);   // writes its output itself
        TRY(capture_end(cs, leaves));
        if (sp) {   // small frontiers: the whole superstep in one kernel (sparse.cu)
            BfsOut bs = bo;
            bs.sparse = 1;
            PushLaunch Ls = push_launch(g, in, t, -1);
            TRY(capture_begin(cs, b_sparse, {}));
            launch_bfs_sparse(Ls, a, bs, in->bits, in->summ, ws->gbar, cs);
            TRY(capture_end(cs, leaves));
        }
        deps = {n_push, n_pull};
        if (n_sparse) deps.push_back(n_sparse);
        if (n_sweep) deps.push_back(n_sweep);
    }
    CK(cudaGraphInstantiate(&ws->bfs_exec, root, 0));
    ws->bfs_heavy = t.heavy;
    ws->bfs_small = t.small;
    ws->bfs_seg = t.seg;
    ws->bfs_cf = t.cf;
    ws->bfs_scsr = t.scsr != 0 && g->scsr_state == 1 ? t.scsr : 0;
    return SG_OK;
}

// partitioned runs: a peer that missed a superstep barrier (timeout) poisons the run
static int check_peers(sg_graph *g) {
    if (!g->ar) return SG_OK;
    unsigned long long err = 0;
    CK(cudaMemcpy(&err, &g->ar->ctl->error, sizeof err, cudaMemcpyDeviceToHost));
    if (err) return fail(SG_ERR_NCCL, "a peer rank did not reach a superstep barrier within the timeout");
    return SG_OK;
}

static int run_bfs_graph(sg_graph *g, int32_t src, uint32_t *level, const sg_opts &o, Tiers t, int64_t max_iters,
                         sg_stats *stats) {
    Workspace *ws = g->ws;
    cudaStream_t s = stream_of(&o);
    const int32_t sc_mode = t.scsr != 0 && g->scsr_state == 1 ? t.scsr : 0;
    const int shape = (env_or("SG_SPARSE", 0) != 0 ? 1 : 0) | (env_or("SG_PULL_WARP_FRAC", 8) != 0 ? 2 : 0) |
                      ((int)env_or("SG_PULL_WORD_MAX", 16) << 2);   // knobs baked into the captured graph
    if (!ws->bfs_exec || ws->bfs_heavy != t.heavy || ws->bfs_small != t.small || ws->bfs_seg != t.seg ||
        ws->bfs_cf != t.cf || ws->bfs_scsr != sc_mode || ws->bfs_shape != shape) {
        TRY(build_bfs_graph(g, t));
        ws->bfs_shape = shape;
    }
    BfsCtrl &c = *ws->h_ctrl;
    memset(&c, 0, sizeof c);
    c.level = level;
    c.mu = g->nnz_global;
    c.n = g->v.n;
    c.max_iters = max_iters;
    c.alpha = o.alpha;
    c.beta = o.beta;
    c.src = src;
    c.pull = o.direction == SG_DIR_PULL;
    c.auto_dir = o.direction == SG_DIR_AUTO;
    c.reached = 1;
    c.sweep_mode = (uint32_t)sc_mode;
    c.sweep_thr = sweep_threshold(g->v.nnz);
    // the fused small-frontier loop (sparse.cu) beats the 4-kernel push superstep only across runs
    // of >= 2 consecutive small supersteps (12 vs 21 us each, path graph); on config 4 it loses
    // its first superstep to the extra clear + launch (measured 578 vs 543 us per BFS),
    // so it is opt-in: SG_SPARSE=1
    c.sparse_mode = (uint32_t)env_or("SG_SPARSE", 0);
    c.sparse_words = env_or("SG_SPARSE_WORDS", 4096);
    c.sparse_arcs = env_or("SG_SPARSE_ARCS", 1 << 16);
    c.pull_warp_frac = (uint32_t)env_or("SG_PULL_WARP_FRAC", 8);
    c.n_iso = g->n_iso;
    // counters back through mapped host memory (SG_RES_MAPPED=1, ~7 us less per BFS) or the
    // device->host copy (default): with the mapped path on, the end-to-end bench's graph_load /
    // graph_free cycle slowed 4-8x in 4 of 5 runs (0.7-1.3 vs 5.6 GTEPS e2e), cause not isolated
    static const bool res_mapped = env_or("SG_RES_MAPPED", 0) != 0;
    c.res = res_mapped ? ws->d_res : nullptr;
    memset((void *)ws->h_res, 0, sizeof(BfsResult));   // (the previous run's graph has completed)
    c.hl = ws->hnd[0];
    for (int i = 0; i < 2; i++) {
        c.hpush[i] = ws->hnd[1 + i];
        c.hpull[i] = ws->hnd[3 + i];
        c.hsweep[i] = ws->hnd[5 + i];
        c.hsparse[i] = ws->hnd[7 + i];
    }
    CK(cudaEventRecord(ws->ev0, s));
    // the control block up to the trace arrays (those are read on demand by sg_bfs_trace)
    const size_t hot = offsetof(BfsCtrl, t_ns);
    if (ws->pro_node) {   // single GPU: the control block's init rides on the prologue node's parameters
        memcpy(ws->pro_args.hot, ws->h_ctrl, hot);
        cudaKernelNodeParams kp;
        bfs_prologue1_node(&ws->pro_args, ws->pro_slot, &kp);
        CK(cudaGraphExecKernelNodeSetParams(ws->bfs_exec, ws->pro_node, &kp));
    } else {
        CK(cudaMemcpyAsync(ws->ctrl, ws->h_ctrl, hot, cudaMemcpyHostToDevice, s));
    }
    CK(cudaGraphLaunch(ws->bfs_exec, s));
    if (g->ar && !o.owned_only) {   // result gather: owned level slices into every rank's replica
        const Arena *A = g->ar;
        launch_publish_owned(level, A->vals, g->v.own_lo, g->v.own_hi, A->x, s);
        launch_xbarrier(A->x, s);
        CK(cudaMemcpyAsync(level, A->vals, sizeof(uint32_t) * (size_t)g->v.n, cudaMemcpyDeviceToDevice, s));
    }
    if (!res_mapped) CK(cudaMemcpyAsync(ws->h_ctrl, ws->ctrl, hot, cudaMemcpyDeviceToHost, s));
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    if (res_mapped) {   // the counters the stopping decision wrote into mapped host memory
        const volatile BfsResult *r = ws->h_res;
        if (!r->done) return fail(SG_ERR_STATE, "the BFS graph ended without a stopping decision");
        c.iters = r->iters;
        c.push_steps = r->push_steps;
        c.pull_steps = r->pull_steps;
        c.arcs_pushed = r->arcs_pushed;
        c.arcs_pulled = r->arcs_pulled;
        c.reached = r->reached;
        c.sweep_steps = r->sweep_steps;
        c.sparse_steps = r->sparse_steps;
        c.overflow = r->overflow;
    }
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    TRY(check_peers(g));
    if (c.overflow) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
    {
        // kernels the graph executed: the prologue kernel + the
        // taken IF bodies (push = word + CTA tier [+ hub segment tier] + output, sweep = arc
        // count + sweep + output, pull = 1)
        const long long per_push = 3 + (t.seg && ws->seg && g->v.hub_idx ? 1 : 0);
        const long long k = 1 + per_push * (long long)(c.push_steps - c.sweep_steps - c.sparse_steps) +
                            3 * (long long)c.sweep_steps + (long long)c.sparse_steps +
                            (ws->bfs_shape & 2 ? 2 : 1) * (long long)c.pull_steps;
        for (long long i = 0; i < k; i++) note_launch();
    }
    if (stats) {
        stats->iterations = (int64_t)c.iters;
        stats->push_steps = (int64_t)c.push_steps;
        stats->pull_steps = (int64_t)c.pull_steps;
        stats->arcs_pushed = (int64_t)c.arcs_pushed;
        stats->arcs_pulled = (int64_t)c.arcs_pulled;
        stats->reached = (int64_t)c.reached;
        stats->device_ms = ms;
    }
    return SG_OK;
}

extern "C" {

// ---- BFS (Listing 1 + Beamer direction optimisation) --------------------------------------
SG_API int run_bfs(const sg_graph *gc, int32_t src, uint32_t *level, const sg_opts *opts, sg_stats *stats) {
    t_err.clear();
    if (!gc || !level) return fail(SG_ERR_INVALID, "NULL argument");
    sg_graph *g = const_cast<sg_graph *>(gc);
    const GraphView &G = g->v;
    if (src < 0 || src >= G.n) return fail(SG_ERR_INVALID, "src %d outside [0,%lld)", src, (long long)G.n);
    sg_opts o;
    if (opts) o = *opts; else sg_opts_default(&o);
    if (o.alpha <= 0) o.alpha = 5.0;
    if (o.beta <= 0) o.beta = 48.0;
    const int64_t max_iters = o.max_iters > 0 ? o.max_iters : G.n + 1;
    cudaStream_t s = stream_of(&o);
    TRY(ensure_ws(g));
    Tiers t = tiers_from(&o);
    TRY(ensure_heavy(g, t.heavy));
    Workspace *ws = g->ws;
    if (g->ar) {   // partitioned: the device-driven loop (every superstep ends in the peer barrier)
        if (o.host_loop || o.one_layer)
            return fail(SG_ERR_UNSUPPORTED, "a partitioned BFS runs device-driven only (no host_loop / one_layer)");
        t.seg = 0;
        t.scsr = 0;
        return run_bfs_graph(g, src, level, o, t, max_iters, stats);
    }
    const bool scsr_on =
        !o.one_layer && scsr_ready(g, t, o.direction == SG_DIR_PUSH || env_or("SG_SCSR_EAGER", 0) != 0, s);
    if (!ws->prof.on && !o.host_loop && !o.one_layer) return run_bfs_graph(g, src, level, o, t, max_iters, stats);
    CK(cudaEventRecord(ws->ev0, s));
    CK(cudaMemsetAsync(level, 0xFF, sizeof(uint32_t) * (size_t)G.n, s));
    launch_set_u32(level, src, 0u, s);
    sg_frontier *in = &ws->fr[0], *out = &ws->fr[1];
    TRY(clear_frontier(in, s));
    TRY(clear_frontier(out, s));
    // visited starts as the isolated vertices (unreachable: level stays INF) plus src
    CK(cudaMemcpyAsync(ws->visited, g->isolated, sizeof(uint64_t) * (size_t)G.nw1, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(ws->vis_old, g->isolated, sizeof(uint64_t) * (size_t)G.nw1, cudaMemcpyDeviceToDevice, s));
    launch_seed(in->bits, in->summ, ws->visited, src, s, ws->vis_old);   // in = {src}, visited |= {src}
    const bool auto_dir = o.direction == SG_DIR_AUTO;
    static const bool trace = getenv("SG_TRACE") != nullptr;
    TRY(compact(g, in, true, s));
    TRY(read_stats(ws, s));
    int64_t mu = G.nnz, nf_prev = 0;
    bool pull = o.direction == SG_DIR_PULL;
    int64_t iters = 0, push_steps = 0, pull_steps = 0, arcs_pushed = 0, arcs_pulled = 0;
    int64_t reached = 1;
    uint32_t d = 0;
    int in_idx = 0;
    int64_t src_iso = 0;   // the source is one of the never-reachable vertices (bfs_decide's rule)
    {
        uint64_t w = 0;
        CK(cudaMemcpy(&w, g->isolated + (src >> 6), sizeof w, cudaMemcpyDeviceToHost));
        src_iso = (int64_t)((w >> (src & 63)) & 1ull);
    }
    for (;;) {
        const DevStats &hs = ws->h_st[in_idx];
        const int64_t count = (int64_t)hs.count;
        if (count == 0) break;
        const int64_t nf = (int64_t)hs.nf, mf = (int64_t)hs.mf;
        if (iters > 0) reached += nf;
        if (reached + g->n_iso - src_iso >= G.n) break;   // every vertex visited (bfs_decide)
        if (iters > 0 && hs.pad2) break;                   // dead-end lookahead of the output kernel
        if (iters >= max_iters) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
        mu -= mf;
        if (auto_dir) {   // Beamer: push -> pull on a growing frontier with m_f > m_u / alpha,
                          // pull -> push on a shrinking frontier with n_f < n / beta
            if (!pull && nf > nf_prev && (double)mf > (double)mu / o.alpha) pull = true;
            else if (pull && nf < nf_prev && (double)nf < (double)G.n / o.beta) pull = false;
        }
        nf_prev = nf;
        const int64_t reached_before = reached;
        const bool sweep = !pull && scsr_on && (t.scsr == 2 || (unsigned long long)mf >= sweep_threshold(G.nnz));
        CK(cudaMemsetAsync(out->st, 0, sizeof(DevStats), s));
        BfsOut bo{ws->vis_old, out->bits, out->summ, out->offsets, level, d + 1, nullptr, nullptr, out->st};
        if (!o.one_layer) {   // dead-end lookahead (bfsstep.cuh): needs the output kernel's done counter
            bo.rp = G.rp;
            bo.col = G.col;
            bo.visited = ws->visited;
            bo.done = ws->bfs_done;
        }
        {   // late pulls: warp-owned layer-2 words (same rule as bfs_decide)
            const long long frac = (long long)env_or("SG_PULL_WARP_FRAC", 8), live = G.n - g->n_iso;
            bo.pull_warp = frac > 0 && (live - reached) * frac < live ? 1 : 0;
        }
        const int pr = prof_begin(ws, pull ? SG_K_PULL : (sweep ? SG_K_SWEEP : SG_K_PUSH), s);
        if (pull) {
            launch_pull_bfs(g->vl, in->bits, ws->visited, in->st, bo, s);   // writes its output itself
            pull_steps++;
        } else if (sweep) {
            launch_push_sweep(g->scsr.v, G.rp, in->bits, in->summ, in->offsets, G.nw2, in->st, ws->visited, 0ull, s);
            push_steps++;
        } else {
            PushLaunch L = push_launch(g, in, t, o.one_layer ? G.nw1 : count);
            L.sparse_ok = o.one_layer ? 0 : 1;
            if (o.one_layer) {   // Fig. 7 ablation: no summary layer, every word is visited
                if (!ws->all_offsets) CK(cudaMalloc(&ws->all_offsets, sizeof(uint32_t) * (size_t)G.nw1));
                launch_list_all(ws->all_offsets, ws->st + 2, in->st, G.nw1, s);
                L.offsets = ws->all_offsets;
                L.st = ws->st + 2;
            }
            BfsArgs a{ws->visited, level, d + 1, nullptr, nullptr};
            a.diff = 1;
            launch_push_bfs(L, a, s);
            push_steps++;
        }
        prof_end(ws, pr, s);
        // output of a push superstep (the pull writes its own): new = visited & ~vis_old -> the
        // whole out 2LB (no clearing needed) + word list, level, n_f / m_f
        const int pc = pull ? -1 : prof_begin(ws, SG_K_COMPACT, s);
        if (!pull) launch_bfs_diff(G, ws->visited, bo, s);
        if (!pull) prof_end(ws, pc, s);
        TRY(read_stats(ws, s));
        {
            // algorithmic bytes of this step.  push: col_idx 4 B/arc, row_ptr 16 B
            // per expanded vertex, 8 B per input word, 8 B per visited word updated.  Output pass
            // (k_bfs_diff): visited + vis_old 16 B per word read, output word 8 B per word
            // written, level 4 B + degree code 1 B per new vertex, vis_old 8 B + list entry 4 B
            // per output word, layer 2 8 B per word.  pull (with its output): visited 8 B per
            // word read, fnbr / col_idx 4 B per candidate / arc tested, output word 8 B per word,
            // level + degree code 5 B per new vertex, visited + vis_old 16 B + list entry 4 B
            // per output word, layer 2 8 B per word, row_ptr 16 B per list-scanned vertex
            const DevStats &ho = ws->h_st[in_idx ^ 1];
            const double n_new = (double)ho.nf, c_out = (double)ho.count;
            double bytes;
            if (pull)   // + 16 B of row_ptr per list-scanned vertex (candidate missed)
                bytes = 16.0 * (double)G.nw1 + 4.0 * (double)ws->h_st[in_idx].arcs +
                        16.0 * (double)ws->h_st[in_idx].scans + 5.0 * n_new + 20.0 * c_out + 8.0 * (double)G.nw2;
            else
                bytes = 4.0 * (double)ws->h_st[in_idx].arcs + 16.0 * (double)nf + 8.0 * (double)count + 8.0 * c_out;
            prof_bytes(ws, pr, bytes);
            if (!pull) prof_bytes(ws, pc, 24.0 * (double)G.nw1 + 5.0 * n_new + 12.0 * c_out + 8.0 * (double)G.nw2);
        }
        if (pull) arcs_pulled += (int64_t)ws->h_st[in_idx].arcs;
        else arcs_pushed += (int64_t)ws->h_st[o.one_layer ? 2 : in_idx].arcs;
        if (trace)
            fprintf(stderr, "[sygraph bfs] level %u %s in: words %lld n_f %lld m_f~%lld | arcs %llu | out: n_f %llu\n", d,
                    pull ? "pull" : "push", (long long)count, (long long)nf, (long long)mf,
                    (unsigned long long)ws->h_st[in_idx].arcs, (unsigned long long)ws->h_st[in_idx ^ 1].nf);
        std::swap(in, out);
        in_idx ^= 1;
        d++;
        iters++;
    }
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    prof_flush(ws);
    if (stats) {
        stats->iterations = iters;
        stats->push_steps = push_steps;
        stats->pull_steps = pull_steps;
        stats->arcs_pushed = arcs_pushed;
        stats->arcs_pulled = arcs_pulled;
        stats->reached = reached;
        stats->device_ms = ms;
    }
    return SG_OK;
}

}  // extern "C"

// Label blocks of the CC pull (label block <= SG_CC_LBLOCK_KB stays in L2).  Returns the number
// of blocks to pull with and sets *ccb: the block-major copy (preferred; SG_CC_CCB=0 disables),
// else the per-row block offsets (cbo), else 1 block (unblocked; needs no extra memory).
static int cc_blocks(sg_graph *g, const GraphView &GL, int direction, cudaStream_t s, bool *ccb) {
    *ccb = false;
    if (direction == SG_DIR_PUSH || !g->sorted) return 1;
    const long long lblock = (long long)env_or("SG_CC_LBLOCK_KB", 32768) << 10;
    int nb = (int)(((long long)GL.n * 4 + lblock - 1) / (lblock > 0 ? lblock : 1));
    if (nb < 1 || lblock <= 0) nb = 1;
    if (nb > 64) nb = 64;
    if (nb == 1) return 1;
    const int64_t S = (GL.n + nb - 1) / nb;
    if (env_or("SG_CC_CCB", 1) != 0 && GL.nnz < 0xFFFFFFF0ll) {
        if (g->ccb_state == 1 && g->ccb.nb == nb && g->ccb.S == S) {
            *ccb = true;
            return nb;
        }
        if (g->ccb_state != -1) {
            if (g->ccb_state == 1) {
                cudaStreamSynchronize(s);
                ccb_free(&g->ccb);
                g->ccb_state = 0;
            }
            if (ccb_build(GL.rp, GL.col, GL.n, nb, S, &g->ccb, s) == cudaSuccess) {
                g->ccb_state = 1;
                *ccb = true;
                return nb;
            }
            cudaGetLastError();
            g->ccb_state = -1;   // memory short: per-row offsets instead
        }
    }
    if (g->cbo_nb != nb) {
        if (g->cbo) {
            cudaStreamSynchronize(s);
            dev_free(g->cbo);
            g->cbo = nullptr;
            g->cbo_nb = 0;
        }
        // n x (nb - 1) block offsets: if they do not fit, pull unblocked (same result, more L2 misses)
        if (dev_alloc(&g->cbo, sizeof(uint32_t) * (size_t)GL.n * (size_t)(nb - 1), s) != cudaSuccess) {
            cudaGetLastError();
            g->cbo = nullptr;
            return 1;
        }
        launch_cc_block_offsets(GL.rp, GL.col, GL.n, nb, S, g->cbo, s);
        g->cbo_nb = nb;
    }
    return nb;
}
static void cc_pull_blocked(sg_graph *g, const GraphView &GL, int nb, bool ccb, int32_t *label, uint64_t *out_bits,
                            DevStats *st, cudaStream_t s) {
    for (int b = 0; b < nb; b++) {
        if (ccb)
            launch_pull_ccb(GL, label, out_bits, st, g->ccb.off + (size_t)b * (size_t)(GL.n + 1),
                            g->ccb.col + g->ccb.h_base[b], b, s);
        else
            launch_pull_cc_block(GL, label, out_bits, st, g->cbo, nb, b, s);
    }
}

// ---- graph-driven SSSP / CC (no host round trip per superstep) -----------------------------
// WHILE { half 0 | half 1 }; half h = IF(push_h) [push kernels + k_value_diff] and, for CC,
// IF(pull_h) [label-blocked pull passes + k_value_diff]; k_value_diff's last CTA decides the next
// superstep (val_decide).  The value array doubles as the functor state; old = ws->dist_old.
static int build_val_graph(sg_graph *g, bool cc, uint32_t *val, Tiers t, int nb, bool ccb) {
    Workspace *ws = g->ws;
    const GraphView &G = g->v;
    Workspace::VGraph &V = ws->vg[cc ? 1 : 0];
    if (V.exec) cudaGraphExecDestroy(V.exec);
    if (V.graph) cudaGraphDestroy(V.graph);
    V.exec = nullptr;
    V.graph = nullptr;
    if (!ws->cap_stream) CK(cudaStreamCreateWithFlags(&ws->cap_stream, cudaStreamNonBlocking));
    if (!ws->vctrl) {
        CK(cudaMalloc(&ws->vctrl, sizeof(ValCtrl)));
        CK(cudaMallocHost(&ws->h_vctrl, sizeof(ValCtrl)));
    }
    if (!ws->dist_old) CK(cudaMalloc(&ws->dist_old, sizeof(uint32_t) * (size_t)(G.n + 4)));
    cudaStream_t cs = ws->cap_stream;
    cudaGraph_t root;
    CK(cudaGraphCreate(&root, 0));
    V.graph = root;
    cudaGraphConditionalHandle hl, hpush[2], hpull[2] = {};
    CK(cudaGraphConditionalHandleCreate(&hl, root, 0, cudaGraphCondAssignDefault));
    for (int i = 0; i < 2; i++) {
        CK(cudaGraphConditionalHandleCreate(&hpush[i], root, 0, cudaGraphCondAssignDefault));
        if (cc) CK(cudaGraphConditionalHandleCreate(&hpull[i], root, 0, cudaGraphCondAssignDefault));
    }
    sg_frontier *F[2] = {&ws->fr[0], &ws->fr[1]};
    std::vector<cudaGraphNode_t> leaves;
    TRY(capture_begin(cs, root, {}));
    CK(cudaMemsetAsync(F[0]->bits, 0, sizeof(uint64_t) * (size_t)G.nw1, cs));
    CK(cudaMemsetAsync(F[0]->summ, 0, sizeof(uint64_t) * (size_t)G.nw2, cs));
    CK(cudaMemsetAsync(ws->st, 0, 2 * sizeof(DevStats), cs));
    if (cc) {
        launch_iota_i32(reinterpret_cast<int32_t *>(val), G.n, cs);
        CK(cudaMemcpyAsync(ws->dist_old, val, sizeof(uint32_t) * (size_t)G.n, cudaMemcpyDeviceToDevice, cs));
        launch_fill_all(F[0]->bits, F[0]->summ, G.n, G.nw1, G.nw2, cs);   // advance::vertices
        launch_compact(F[0]->summ, G.nw2, F[0]->offsets, F[0]->st, cs);
        launch_frontier_stats(G, F[0]->bits, F[0]->st, cs);
        launch_val_first(ws->vctrl, F[0]->st, cs);
    } else {
        CK(cudaMemsetAsync(val, 0xFF, sizeof(uint32_t) * (size_t)G.n, cs));
        CK(cudaMemsetAsync(ws->dist_old, 0xFF, sizeof(uint32_t) * (size_t)G.n, cs));
        launch_val_seed(ws->vctrl, val, ws->dist_old, F[0]->bits, F[0]->summ, F[0]->offsets, F[0]->st, cs);
    }
    TRY(capture_end(cs, leaves));
    cudaGraphNode_t wnode;
    cudaGraph_t body;
    TRY(add_cond(root, leaves, hl, cudaGraphCondTypeWhile, &wnode, &body));
    std::vector<cudaGraphNode_t> deps;
    for (int half = 0; half < 2; half++) {
        sg_frontier *in = F[half], *out = F[half ^ 1];
        BfsOut bo{};
        bo.out_bits = out->bits;
        bo.out_summ = out->summ;
        bo.out_offsets = out->offsets;
        bo.st = out->st;
        bo.prev = in->st;
        bo.done = ws->bfs_done;
        bo.half = half;
        bo.vctrl = ws->vctrl;
        cudaGraphNode_t n_push, n_pull = nullptr;
        cudaGraph_t b_push, b_pull = nullptr;
        TRY(add_cond(body, deps, hpush[half], cudaGraphCondTypeIf, &n_push, &b_push));
        if (cc) TRY(add_cond(body, deps, hpull[half], cudaGraphCondTypeIf, &n_pull, &b_pull));
        PushLaunch L = push_launch(g, in, t, -1);
        L.batch = t.cf;   // 0: coarsening factor from the device-side count
        TRY(capture_begin(cs, b_push, {}));
        if (cc) {
            launch_push_cc(L, CcArgs{reinterpret_cast<int32_t *>(val), nullptr, nullptr}, cs);
        } else {
            SsspArgs sa{val, nullptr, nullptr};
            sa.diff = 1;
            launch_push_sssp(L, sa, cs);
        }
        launch_value_diff(G, val, ws->dist_old, bo, cc ? 1 : 0, cs);
        TRY(capture_end(cs, leaves));
        if (cc) {
            TRY(capture_begin(cs, b_pull, {}));
            if (nb > 1) cc_pull_blocked(g, g->vl, nb, ccb, reinterpret_cast<int32_t *>(val), out->bits, in->st, cs);
            else launch_pull_cc(g->vl, reinterpret_cast<int32_t *>(val), out->bits, out->summ, in->st, cs);
            launch_value_diff(G, val, ws->dist_old, bo, 1, cs);
            TRY(capture_end(cs, leaves));
        }
        deps = {n_push};
        if (n_pull) deps.push_back(n_pull);
    }
    CK(cudaGraphInstantiate(&V.exec, root, 0));
    V.result = val;
    V.heavy = t.heavy;
    V.small = t.small;
    V.nb = nb;
    V.ccb = ccb;
    V.h[0] = (unsigned long long)hl;
    for (int i = 0; i < 2; i++) {
        V.h[1 + i] = (unsigned long long)hpush[i];
        V.h[3 + i] = cc ? (unsigned long long)hpull[i] : 0ull;
    }
    return SG_OK;
}

static int run_value_graph(sg_graph *g, bool cc, int32_t src, uint32_t *val, const sg_opts &o, int64_t max_iters,
                           sg_stats *stats) {
    Workspace *ws = g->ws;
    cudaStream_t s = stream_of(&o);
    Tiers t = tiers_from(&o);
    t.seg = 0;
    TRY(ensure_heavy(g, t.heavy));
    bool use_ccb = false;
    const int nb = cc ? cc_blocks(g, g->vl, o.direction, s, &use_ccb) : 1;
    Workspace::VGraph &V = ws->vg[cc ? 1 : 0];
    if (!V.exec || V.result != val || V.heavy != t.heavy || V.small != t.small || V.nb != nb || V.ccb != use_ccb)
        TRY(build_val_graph(g, cc, val, t, nb, use_ccb));
    ValCtrl &c = *ws->h_vctrl;
    memset(&c, 0, sizeof c);
    c.max_iters = max_iters;
    c.nnz = g->nnz_global;
    c.cc = cc ? 1u : 0u;
    c.direction = (uint32_t)o.direction;
    c.src = src;
    c.hl = V.h[0];
    for (int i = 0; i < 2; i++) {
        c.hpush[i] = V.h[1 + i];
        c.hpull[i] = V.h[3 + i];
    }
    CK(cudaEventRecord(ws->ev0, s));
    CK(cudaMemcpyAsync(ws->vctrl, ws->h_vctrl, sizeof(ValCtrl), cudaMemcpyHostToDevice, s));
    CK(cudaGraphLaunch(V.exec, s));
    CK(cudaMemcpyAsync(ws->h_vctrl, ws->vctrl, sizeof(ValCtrl), cudaMemcpyDeviceToHost, s));
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    if (c.overflow) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
    {   // kernels the graph executed: prologue (SSSP 1, CC 4) + per push step 3, per pull step nb + 1
        const long long k = (cc ? 4 : 1) + 3 * (long long)c.push_steps + (long long)(nb + 1) * (long long)c.pull_steps;
        for (long long i = 0; i < k; i++) note_launch();
    }
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = (int64_t)c.iters;
        stats->push_steps = (int64_t)c.push_steps;
        stats->pull_steps = (int64_t)c.pull_steps;
        stats->arcs_pushed = (int64_t)c.arcs_pushed;
        stats->arcs_pulled = (int64_t)c.arcs_pulled;
        stats->reached = cc ? g->v.n : -1;
        stats->device_ms = ms;
    }
    return SG_OK;
}

// ---- SSSP / CC over the 1-D destination partition (xchg.cuh) ------------------
// Every rank holds the replicated value array (arena vals) and frontier; a superstep = the local
// advance over the push block (SSSP relax / CC push: atomicMin on owned destinations only) or the
// pull over the owned rows (CC), then k_value_diff over the owned words: the vertices whose value
// decreased form the owned slice of the next frontier, and it stores the changed values, the
// output words and the word list into every peer's replica and runs the superstep barrier.  The
// host reads one control block per superstep (global count / n_f / m_f / arcs), as the single-GPU
// SSSP / CC loops do.  A peer's values of superstep e may land while this rank still relaxes
// superstep e: asynchronous relaxation (reading C12), same fixed point.
static int run_value_part(sg_graph *g, bool cc, int32_t src, uint32_t *result, const sg_opts &o, sg_stats *stats) {
    Workspace *ws = g->ws;
    Arena *A = g->ar;
    const GraphView &G = g->v;
    cudaStream_t s = stream_of(&o);
    Tiers t = tiers_from(&o);
    t.seg = 0;
    t.scsr = 0;
    TRY(ensure_heavy(g, t.heavy));
    const int64_t max_iters = o.max_iters > 0 ? o.max_iters : G.n + 1;
    uint32_t *vals = A->vals;
    if (!ws->dist_old) CK(cudaMalloc(&ws->dist_old, sizeof(uint32_t) * (size_t)(G.n + 4)));
    // label-blocked pull over the owned rows (CC, as run_cc)
    bool use_ccb = false;
    const int cc_nb = cc ? cc_blocks(g, g->vl, o.direction, s, &use_ccb) : 1;
    CK(cudaEventRecord(ws->ev0, s));
    if (cc) {
        launch_iota_i32(reinterpret_cast<int32_t *>(vals), G.n, s);
    } else {
        CK(cudaMemsetAsync(vals, 0xFF, sizeof(uint32_t) * (size_t)G.n, s));
        launch_set_u32(vals, src, 0u, s);
    }
    CK(cudaMemcpyAsync(ws->dist_old, vals, sizeof(uint32_t) * (size_t)G.n, cudaMemcpyDeviceToDevice, s));
    sg_frontier *in = &ws->fr[0], *out = &ws->fr[1];
    TRY(clear_frontier(in, s));
    TRY(clear_frontier(out, s));
    CK(cudaMemsetAsync(ws->st, 0, 2 * sizeof(DevStats), s));
    if (cc) launch_fill_all(in->bits, in->summ, G.n, G.nw1, G.nw2, s);   // advance::vertices
    else launch_seed(in->bits, in->summ, nullptr, src, s);
    TRY(compact(g, in, cc, s));          // identical on every rank (replicated input)
    launch_xbarrier(A->x, s);            // every rank initialised before any peer writes into it
    TRY(read_stats(ws, s));
    int64_t iters = 0, push_steps = 0, pull_steps = 0, arcs_pushed = 0, arcs_pulled = 0;
    int in_idx = 0;
    for (;;) {
        const int64_t count = (int64_t)ws->h_st[in_idx].count;
        if (count == 0) break;
        if (iters >= max_iters) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
        const bool pull = cc && (o.direction == SG_DIR_PULL ||
                                 (o.direction == SG_DIR_AUTO && (double)ws->h_st[in_idx].mf * 4.0 > (double)g->nnz_global));
        if (pull && cc_nb > 1) {
            cc_pull_blocked(g, g->vl, cc_nb, use_ccb, reinterpret_cast<int32_t *>(vals), out->bits, in->st, s);
        } else if (pull) {
            launch_pull_cc(g->vl, reinterpret_cast<int32_t *>(vals), out->bits, out->summ, in->st, s);
        } else {
            const PushLaunch L = push_launch(g, in, t, count);
            if (cc) {
                launch_push_cc(L, CcArgs{reinterpret_cast<int32_t *>(vals), nullptr, nullptr}, s);
            } else {
                SsspArgs sa{vals, nullptr, nullptr};
                sa.diff = 1;
                launch_push_sssp(L, sa, s);
            }
        }
        (pull ? pull_steps : push_steps)++;
        BfsOut bo{};
        bo.out_bits = out->bits;
        bo.out_summ = out->summ;
        bo.out_offsets = out->offsets;
        bo.st = out->st;
        bo.prev = in->st;      // zeroed by the last CTA before it publishes (the next output)
        bo.done = ws->bfs_done;
        bo.x = A->x;
        launch_value_diff(G, vals, ws->dist_old, bo, cc ? 1 : 0, s);
        TRY(read_stats(ws, s));
        (pull ? arcs_pulled : arcs_pushed) += (int64_t)ws->h_st[in_idx ^ 1].pad;   // global arcs of the step
        std::swap(in, out);
        in_idx ^= 1;
        iters++;
    }
    CK(cudaMemcpyAsync(result, vals, sizeof(uint32_t) * (size_t)G.n, cudaMemcpyDeviceToDevice, s));
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    TRY(check_peers(g));
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = iters;
        stats->push_steps = push_steps;
        stats->pull_steps = pull_steps;
        stats->arcs_pushed = arcs_pushed;
        stats->arcs_pulled = arcs_pulled;
        stats->reached = cc ? G.n : -1;
        stats->device_ms = ms;
    }
    return SG_OK;
}

extern "C" {

// ---- SSSP (frontier Bellman-Ford) --------------------------------------------------
SG_API int run_sssp(const sg_graph *gc, int32_t src, uint32_t *dist, const sg_opts *opts, sg_stats *stats) {
    t_err.clear();
    if (!gc || !dist) return fail(SG_ERR_INVALID, "NULL argument");
    sg_graph *g = const_cast<sg_graph *>(gc);
    const GraphView &G = g->v;
    if (src < 0 || src >= G.n) return fail(SG_ERR_INVALID, "src %d outside [0,%lld)", src, (long long)G.n);
    if (!g->w) return fail(SG_ERR_INVALID, "SSSP needs graph weights");
    if ((double)g->max_w * (double)(G.n - 1) >= 4294967295.0)
        return fail(SG_ERR_UNSUPPORTED, "max_weight*(n-1) does not fit uint32 distances");
    sg_opts o;
    if (opts) o = *opts; else sg_opts_default(&o);
    const int64_t max_iters = o.max_iters > 0 ? o.max_iters : G.n + 1;
    cudaStream_t s = stream_of(&o);
    TRY(ensure_ws(g));
    if (g->ar) {
        if (o.sssp_delta > 0) return fail(SG_ERR_UNSUPPORTED, "delta-stepping runs on single-GPU graphs only");
        return run_value_part(g, false, src, dist, o, stats);
    }
    // default: device-driven loop (CUDA graph); host_loop = 1 keeps the host-driven one below
    if (!o.host_loop && o.sssp_delta <= 0 && env_or("SG_SSSP_DIFF", 1) != 0)
        return run_value_graph(g, false, src, dist, o, max_iters, stats);
    const Tiers t = tiers_from(&o);
    TRY(ensure_heavy(g, t.heavy));
    Workspace *ws = g->ws;
    CK(cudaEventRecord(ws->ev0, s));
    CK(cudaMemsetAsync(dist, 0xFF, sizeof(uint32_t) * (size_t)G.n, s));
    launch_set_u32(dist, src, 0u, s);
    sg_frontier *in = &ws->fr[0], *out = &ws->fr[1];
    TRY(clear_frontier(in, s));
    TRY(clear_frontier(out, s));
    launch_seed(in->bits, in->summ, nullptr, src, s);
    TRY(compact(g, in, false, s));
    TRY(read_stats(ws, s));
    int64_t iters = 0, arcs = 0;
    int in_idx = 0;
    if (o.sssp_delta > 0) {
        // near-far delta-stepping (the paper uses plain Bellman-Ford): only the
        // vertices with dist < T (near) are advanced; improved vertices at >= T wait in `far`; when
        // near empties, T jumps to the bucket of far's minimum and those vertices move to near.
        if (!ws->far) {
            ws->far = new sg_frontier();
            TRY(alloc_frontier_bufs(ws->far, g, true));
        }
        sg_frontier *near = in, *far = ws->far;
        TRY(clear_frontier(far, s));
        const double D = (double)o.sssp_delta;
        double T = D;
        unsigned int *d_min = reinterpret_cast<unsigned int *>(ws->scratch);
        for (;;) {
            while (ws->h_st[0].count) {
                if (iters >= max_iters) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
                const PushLaunch L = push_launch(g, near, t, (int64_t)ws->h_st[0].count);
                launch_push_sssp(L, SsspArgs{dist, out->bits, out->summ}, s);
                TRY(clear_frontier(near, s));
                launch_filter(G, out->bits, near->bits, near->summ, SG_PRED_U32_RANGE, dist, 0.0, T, 0, s);
                launch_filter(G, out->bits, far->bits, far->summ, SG_PRED_U32_RANGE, dist, T, 4294967296.0, 0, s);
                TRY(clear_frontier(out, s));
                TRY(compact(g, near, false, s));
                TRY(read_stats(ws, s));
                iters++;
            }
            CK(cudaMemsetAsync(d_min, 0xFF, sizeof(unsigned int), s));
            launch_min_over_bits(G, far->bits, dist, d_min, s);
            unsigned int hmin = 0;
            CK(cudaMemcpyAsync(&hmin, d_min, sizeof hmin, cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            if (hmin == INF32) break;
            T = (std::floor((double)hmin / D) + 1.0) * D;
            launch_filter(G, far->bits, near->bits, near->summ, SG_PRED_U32_RANGE, dist, 0.0, T, 0, s);
            launch_filter(G, far->bits, far->bits, far->summ, SG_PRED_U32_RANGE, dist, T, 4294967296.0, 1, s);
            TRY(compact(g, near, false, s));
            TRY(read_stats(ws, s));
        }
        arcs = -1;   // not accumulated in this mode
    }
    // diff mode (default): the push only relaxes (fire-and-forget red.min), k_sssp_diff derives
    // the output frontier (dist < dist_old) and its word list in one pass over dist
    static const bool sssp_diff = env_or("SG_SSSP_DIFF", 1) != 0;
    if (o.sssp_delta <= 0 && sssp_diff) {
        if (!ws->dist_old) CK(cudaMalloc(&ws->dist_old, sizeof(uint32_t) * (size_t)(G.n ? G.n : 1)));
        CK(cudaMemcpyAsync(ws->dist_old, dist, sizeof(uint32_t) * (size_t)G.n, cudaMemcpyDeviceToDevice, s));
    }
    for (; o.sssp_delta <= 0;) {
        const int64_t count = (int64_t)ws->h_st[in_idx].count;
        if (count == 0) break;
        if (iters >= max_iters) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
        const PushLaunch L = push_launch(g, in, t, count);
        if (sssp_diff) {
            CK(cudaMemsetAsync(out->st, 0, sizeof(DevStats), s));
            SsspArgs sa{dist, nullptr, nullptr};
            sa.diff = 1;
            launch_push_sssp(L, sa, s);
            launch_sssp_diff(G, dist, ws->dist_old, out->bits, out->summ, out->offsets, out->st, s);
        } else {
            launch_push_sssp(L, SsspArgs{dist, out->bits, out->summ}, s);
            TRY(clear_frontier(in, s));
            TRY(compact(g, out, false, s));
        }
        TRY(read_stats(ws, s));
        arcs += (int64_t)ws->h_st[in_idx].arcs;
        std::swap(in, out);
        in_idx ^= 1;
        iters++;
    }
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = iters;
        stats->push_steps = iters;
        stats->arcs_pushed = arcs;
        stats->reached = -1;
        stats->device_ms = ms;
    }
    return SG_OK;
}

// ---- CC (label propagation) --------------------------------------------------------
SG_API int run_cc(const sg_graph *gc, int32_t *label, const sg_opts *opts, sg_stats *stats) {
    t_err.clear();
    if (!gc || !label) return fail(SG_ERR_INVALID, "NULL argument");
    sg_graph *g = const_cast<sg_graph *>(gc);
    const GraphView &G = g->v;
    sg_opts o;
    if (opts) o = *opts; else sg_opts_default(&o);
    const int64_t max_iters = o.max_iters > 0 ? o.max_iters : G.n + 1;
    cudaStream_t s = stream_of(&o);
    TRY(ensure_ws(g));
    if (g->directed) return fail(SG_ERR_UNSUPPORTED, "CC by label propagation needs a symmetric graph (reading C8)");
    if (g->ar) return run_value_part(g, true, 0, reinterpret_cast<uint32_t *>(label), o, stats);
    // default: device-driven loop (CUDA graph); host_loop = 1 keeps the host-driven one below
    if (!o.host_loop) return run_value_graph(g, true, 0, reinterpret_cast<uint32_t *>(label), o, max_iters, stats);
    const Tiers t = tiers_from(&o);
    TRY(ensure_heavy(g, t.heavy));
    Workspace *ws = g->ws;
    L2Pin pin(label, sizeof(int32_t) * (size_t)G.n, s);   // labels are probed once per arc: keep them in L2
    // label blocks for the pull step: labels of one block (<= SG_CC_LBLOCK_KB) stay in L2
    bool use_ccb = false;
    const int cc_nb = cc_blocks(g, G, o.direction, s, &use_ccb);
    CK(cudaEventRecord(ws->ev0, s));
    launch_iota_i32(label, G.n, s);
    sg_frontier *in = &ws->fr[0], *out = &ws->fr[1];
    launch_fill_all(in->bits, in->summ, G.n, G.nw1, G.nw2, s);    // advance::vertices
    TRY(clear_frontier(out, s));
    TRY(compact(g, in, true, s));
    TRY(read_stats(ws, s));
    int64_t iters = 0, push_steps = 0, pull_steps = 0, arcs_pushed = 0, arcs_pulled = 0;
    int in_idx = 0;
    for (;;) {
        const int64_t count = (int64_t)ws->h_st[in_idx].count;
        if (count == 0) break;
        if (iters >= max_iters) return fail(SG_ERR_STATE, "iteration cap %lld reached", (long long)max_iters);
        // direction: a dense superstep (frontier arcs > nnz/4) pulls — every vertex takes the min of
        // its neighbours' labels without atomics; a sparse one pushes from the changed vertices
        const bool pull = o.direction == SG_DIR_PULL ||
                          (o.direction == SG_DIR_AUTO && (double)ws->h_st[in_idx].mf * 4.0 > (double)G.nnz);
        if (pull && cc_nb > 1) {   // label-blocked pull: one pass per L2-sized label block
            cc_pull_blocked(g, G, cc_nb, use_ccb, label, out->bits, in->st, s);
            launch_rebuild_summary(out->bits, out->summ, G.nw1, G.nw2, s);
            pull_steps++;
        } else if (pull) {
            launch_pull_cc(G, label, out->bits, out->summ, in->st, s);
            pull_steps++;
        } else {
            const PushLaunch L = push_launch(g, in, t, count);
            launch_push_cc(L, CcArgs{label, out->bits, out->summ}, s);
            push_steps++;
        }
        TRY(clear_frontier(in, s));
        TRY(compact(g, out, true, s));
        TRY(read_stats(ws, s));
        (pull ? arcs_pulled : arcs_pushed) += (int64_t)ws->h_st[in_idx].arcs;
        std::swap(in, out);
        in_idx ^= 1;
        iters++;
    }
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = iters;
        stats->push_steps = push_steps;
        stats->pull_steps = pull_steps;
        stats->arcs_pushed = arcs_pushed;
        stats->arcs_pulled = arcs_pulled;
        stats->reached = G.n;
        stats->device_ms = ms;
    }
    return SG_OK;
}

}  // extern "C"

// ---- source-batched BC (bcb.cu): 32 sources per CUDA-graph launch -------------------------
static int bcb_alloc(sg_graph *g) {
    Workspace *ws = g->ws;
    BcbLaunch &B = ws->bcb;
    const int64_t n = g->v.n;
    B.g = g->v;
    B.cap = (int32_t)(n + 1 < (1 << 20) ? n + 1 : (1 << 20));
    B.lcap = n * 32;   // each (vertex, source) pair is in at most one level entry
    CK(cudaMalloc(&B.F, sizeof(uint32_t) * (size_t)n * 3));
    CK(cudaMalloc(&B.V, sizeof(uint32_t) * (size_t)n));
    CK(cudaMalloc(&B.M, sizeof(uint32_t) * (size_t)n * 3));
    CK(cudaMalloc(&B.s, sizeof(double) * (size_t)n * 32));
    CK(cudaMalloc(&B.delta, sizeof(double) * (size_t)n * 32));
    CK(cudaMalloc(&B.lv, sizeof(int32_t) * (size_t)B.lcap));
    CK(cudaMalloc(&B.lm, sizeof(uint32_t) * (size_t)B.lcap));
    CK(cudaMalloc(&B.loff, sizeof(unsigned long long) * (size_t)(B.cap + 2)));
    CK(cudaMalloc(&B.maxb, sizeof(unsigned long long) * (size_t)(B.cap + 1) * 32));
    CK(cudaMalloc(&B.c, sizeof(BcbCtrl)));
    CK(cudaMallocHost(&ws->h_bcb, sizeof(BcbCtrl)));
    CK(cudaMalloc(&B.VB, sizeof(uint64_t) * (size_t)g->v.nw1));
    CK(cudaMalloc(&B.VS, sizeof(uint64_t) * (size_t)g->v.nw2));
    CK(cudaMemset(B.VB, 0, sizeof(uint64_t) * (size_t)g->v.nw1));
    CK(cudaMemset(B.VS, 0, sizeof(uint64_t) * (size_t)g->v.nw2));
    CK(cudaMemset(B.F, 0, sizeof(uint32_t) * (size_t)n * 3));
    CK(cudaMemset(B.V, 0, sizeof(uint32_t) * (size_t)n));
    CK(cudaMemset(B.M, 0, sizeof(uint32_t) * (size_t)n * 3));
    CK(cudaMemset(B.delta, 0, sizeof(double) * (size_t)n * 32));   // backward accumulators
    CK(cudaMemset(B.maxb, 0, sizeof(unsigned long long) * (size_t)(B.cap + 1) * 32));
    ws->bcb_ready = true;
    return SG_OK;
}

// returns SG_ERR_OOM (caller falls back to the per-source path) if the batch buffers do not fit
static int run_bc_batched(sg_graph *g, const int32_t *sources, int32_t k, double *bc, cudaStream_t s,
                          sg_stats *stats) {
    Workspace *ws = g->ws;
    if (!ws->bcb_ready) {
        const int r = bcb_alloc(g);
        if (r != SG_OK) return r;
    }
    ws->bcb.bc = bc;
    CK(cudaEventRecord(ws->ev0, s));
    CK(cudaMemsetAsync(bc, 0, sizeof(double) * (size_t)g->v.n, s));
    int64_t levels = 0;
    for (int32_t b0 = 0; b0 < k; b0 += 32) {
        BcbCtrl &c = *ws->h_bcb;
        memset(&c, 0, sizeof c);
        c.nsrc = k - b0 < 32 ? k - b0 : 32;
        for (int j = 0; j < c.nsrc; j++) c.src[j] = sources[b0 + j];
        CK(cudaMemcpyAsync(ws->bcb.c, &c, sizeof(BcbCtrl), cudaMemcpyHostToDevice, s));
        CK(bcb_run_batch(ws->bcb, s));
        CK(cudaMemcpyAsync(&c, ws->bcb.c, sizeof(BcbCtrl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (c.overflow) {
            // entries past the list capacity were not recorded: clear every per-batch array
            CK(cudaMemsetAsync(ws->bcb.delta, 0, sizeof(double) * (size_t)g->v.n * 32, s));
            CK(cudaMemsetAsync(ws->bcb.F, 0, sizeof(uint32_t) * (size_t)g->v.n * 3, s));
            CK(cudaMemsetAsync(ws->bcb.V, 0, sizeof(uint32_t) * (size_t)g->v.n, s));
            CK(cudaMemsetAsync(ws->bcb.M, 0, sizeof(uint32_t) * (size_t)g->v.n * 3, s));
            CK(cudaMemsetAsync(ws->bcb.VB, 0, sizeof(uint64_t) * (size_t)g->v.nw1, s));
            CK(cudaMemsetAsync(ws->bcb.VS, 0, sizeof(uint64_t) * (size_t)g->v.nw2, s));
            CK(cudaStreamSynchronize(s));
            return fail(SG_ERR_UNSUPPORTED, "batched BC: level/list capacity exceeded");
        }
        levels += c.depth;
        if (getenv("SG_TRACE"))
            fprintf(stderr, "[sygraph bc] batch %d: %d levels, %llu entries, phase ms fwdA %.2f fwdA2 %.2f fwdB %.2f bwdA %.2f bwdB %.2f\n",
                    b0 / 32, c.depth, c.ltop, c.t_ns[0] / 1e6, c.t_ns[1] / 1e6, c.t_ns[2] / 1e6, c.t_ns[3] / 1e6,
                    c.t_ns[4] / 1e6);
    }
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = 2 * levels;
        stats->push_steps = levels;
        stats->device_ms = ms;
    }
    return SG_OK;
}

extern "C" {

// ---- BC (Brandes forward sigma + backward delta) -----------------------------------
SG_API int run_bc(const sg_graph *gc, const int32_t *sources, int32_t k, double *bc, const sg_opts *opts,
                  sg_stats *stats) {
    t_err.clear();
    if (!gc || !bc || (k > 0 && !sources) || k < 0) return fail(SG_ERR_INVALID, "bad run_bc arguments");
    if (gc->ar) return fail(SG_ERR_UNSUPPORTED, "BC shards sources over full replicas (SURVEY 8(e)), not a partitioned graph");
    if (gc->directed) return fail(SG_ERR_UNSUPPORTED, "BC (pull-style backward sweep) needs a symmetric graph");
    sg_graph *g = const_cast<sg_graph *>(gc);
    const GraphView &G = g->v;
    for (int32_t i = 0; i < k; i++)
        if (sources[i] < 0 || sources[i] >= G.n) return fail(SG_ERR_INVALID, "source %d outside [0,%lld)", sources[i], (long long)G.n);
    sg_opts o;
    if (opts) o = *opts; else sg_opts_default(&o);
    cudaStream_t s = stream_of(&o);
    TRY(ensure_ws(g));
    const Tiers t = tiers_from(&o);
    TRY(ensure_heavy(g, t.heavy));
    Workspace *ws = g->ws;
    if (!o.host_loop && k > 0) {   // default: source-batched (f1); falls back when memory is short
        const int r = run_bc_batched(g, sources, k, bc, s, stats);
        if (r != SG_ERR_OOM) return r;
        cudaGetLastError();
        t_err.clear();
    }
    if (!ws->sigma) {
        CK(cudaMalloc(&ws->sigma, sizeof(double) * (size_t)G.n));
        CK(cudaMalloc(&ws->delta, sizeof(double) * (size_t)G.n));
        CK(cudaMalloc(&ws->level, sizeof(uint32_t) * (size_t)G.n));
        CK(cudaMalloc(&ws->stack, sizeof(int32_t) * (size_t)G.n));
        CK(cudaMalloc(&ws->exp_of_level, sizeof(int32_t) * (size_t)(G.n + 1)));
    }
    CK(cudaEventRecord(ws->ev0, s));
    CK(cudaMemsetAsync(bc, 0, sizeof(double) * (size_t)G.n, s));
    int64_t total_iters = 0, arcs = 0;
    std::vector<int64_t> level_off;
    unsigned long long *d_max = ws->scratch, *d_top = ws->scratch + 1, *d_under = ws->scratch + 2;
    for (int32_t si = 0; si < k; si++) {
        const int32_t src = sources[si];
        CK(cudaMemsetAsync(ws->level, 0xFF, sizeof(uint32_t) * (size_t)G.n, s));
        CK(cudaMemsetAsync(ws->sigma, 0, sizeof(double) * (size_t)G.n, s));
        CK(cudaMemsetAsync(ws->visited, 0, sizeof(uint64_t) * (size_t)G.nw1, s));
        CK(cudaMemsetAsync(ws->scratch, 0, 8 * sizeof(unsigned long long), s));
        CK(cudaMemsetAsync(ws->exp_of_level, 0, sizeof(int32_t), s));
        launch_set_u32(ws->level, src, 0u, s);
        launch_set_f64(ws->sigma, src, 1.0, s);
        launch_set_i32(ws->stack, 0, src, s);
        launch_set_u32(reinterpret_cast<uint32_t *>(d_top), 0, 1u, s);
        sg_frontier *in = &ws->fr[0], *out = &ws->fr[1];
        TRY(clear_frontier(in, s));
        TRY(clear_frontier(out, s));
        launch_seed(in->bits, in->summ, ws->visited, src, s);
        TRY(compact(g, in, false, s));
        TRY(read_stats(ws, s));
        level_off.assign(1, 0);
        level_off.push_back(1);
        uint32_t d = 0;
        int in_idx = 0;
        for (;;) {
            const int64_t count = (int64_t)ws->h_st[in_idx].count;
            if (count == 0) break;
            if ((int64_t)d > G.n) return fail(SG_ERR_STATE, "BC level cap reached");
            const PushLaunch L = push_launch(g, in, t, count);
            launch_push_bc(L, BcArgs{ws->visited, ws->sigma, ws->level, d + 1, out->bits, out->summ}, s);
            TRY(clear_frontier(in, s));
            TRY(compact(g, out, false, s));
            // finish level d+1: visited |= out, per-level scale, BFS stack
            launch_or_listed(out->bits, out->offsets, out->st, ws->visited, G.nw1, s);
            CK(cudaMemsetAsync(d_max, 0, sizeof(unsigned long long), s));
            launch_bc_level_max(ws->sigma, out->bits, out->offsets, out->st, G.nw1, d_max, s);
            launch_bc_level_scale_and_stack(ws->sigma, out->bits, out->offsets, out->st, G.nw1, d_max,
                                            ws->exp_of_level, d + 1, ws->stack, d_top, d_under, s);
            CK(cudaMemcpyAsync(ws->h_scratch, ws->scratch, 8 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
            TRY(read_stats(ws, s));
            arcs += (int64_t)ws->h_st[in_idx].arcs;
            std::swap(in, out);
            in_idx ^= 1;
            d++;
            total_iters++;
            if (ws->h_st[in_idx].count) level_off.push_back((int64_t)ws->h_scratch[1]);
        }
        if (ws->h_scratch[2]) return fail(SG_ERR_UNSUPPORTED, "sigma dynamic range within a BFS level exceeds fp64");
        // backward: levels depth-1 .. 1 (level 0 = the source: delta_s(s) excluded)
        const int64_t depth = (int64_t)level_off.size() - 1;   // number of levels
        for (int64_t lv = depth - 1; lv >= 1; lv--)
            launch_bc_backward_level(G, ws->stack, level_off[lv], level_off[lv + 1], ws->level, ws->sigma, ws->delta,
                                     ws->exp_of_level, (uint32_t)lv, bc, src, s);
        total_iters += depth;
    }
    CK(cudaEventRecord(ws->ev1, s));
    CK(cudaEventSynchronize(ws->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ws->ev0, ws->ev1));
    CK(cudaGetLastError());
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = total_iters;
        stats->push_steps = total_iters;
        stats->arcs_pushed = arcs;
        stats->device_ms = ms;
    }
    return SG_OK;
}

// ---- measurement ---------------------------------------------------------------------------
SG_API int sg_profile(sg_graph *g, int enable) {
    if (!g) return fail(SG_ERR_INVALID, "NULL graph");
    TRY(ensure_ws(g));
    Prof &P = g->ws->prof;
    P.on = enable != 0;
    P.recs.clear();
    P.used = 0;
    for (int i = 0; i < SG_K_COUNT; i++) {
        P.ms[i] = 0;
        P.bytes[i] = 0;
        P.launches[i] = 0;
    }
    return SG_OK;
}

SG_API int sg_profile_read(const sg_graph *g, sg_kprof *out) {
    if (!g || !out) return fail(SG_ERR_INVALID, "NULL argument");
    for (int i = 0; i < SG_K_COUNT; i++) {
        out[i].ms = g->ws ? g->ws->prof.ms[i] : 0.0;
        out[i].bytes = g->ws ? g->ws->prof.bytes[i] : 0.0;
        out[i].launches = g->ws ? g->ws->prof.launches[i] : 0;
    }
    return SG_OK;
}

SG_API int64_t sg_launch_count(void) { return (int64_t)g_launches.load(); }

SG_API int sg_ablation_bfs(const sg_graph *g, int32_t src, uint32_t *level, int32_t word_bits, void *stream,
                           sg_stats *stats) {
    t_err.clear();
    if (!g || !level || (word_bits != 32 && word_bits != 64)) return fail(SG_ERR_INVALID, "bad sg_ablation_bfs arguments");
    if (src < 0 || src >= g->v.n) return fail(SG_ERR_INVALID, "src outside [0, n)");
    if (g->ar) return fail(SG_ERR_UNSUPPORTED, "ablation paths are single-GPU");
    int64_t it = 0;
    float ms = 0.f;
    if (ablation_bfs_words(g->v, src, level, word_bits, (cudaStream_t)stream, &it, &ms) != 0)
        return fail(SG_ERR_CUDA, "ablation BFS failed: %s", cudaGetErrorString(cudaGetLastError()));
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->iterations = it;
        stats->push_steps = it;
        stats->device_ms = ms;
    }
    return SG_OK;
}

SG_API int sg_ctrl_debug(const sg_graph *g, int64_t out[16]) {
    if (!g || !g->ws || !g->ws->h_ctrl || !out) return fail(SG_ERR_STATE, "no device-driven BFS has run on this graph");
    CK(cudaMemcpy(g->ws->h_ctrl, g->ws->ctrl, sizeof(BfsCtrl), cudaMemcpyDeviceToHost));
    for (int i = 0; i < 16; i++) out[i] = (int64_t)g->ws->h_ctrl->dbg[i];
    return SG_OK;
}

SG_API int sg_bfs_trace(const sg_graph *g, int64_t *t_ns, int32_t *kind, int64_t *count, int64_t *nf, int64_t *mf,
                        int32_t cap) {
    if (!g || !g->ws || !g->ws->h_ctrl) return fail(SG_ERR_STATE, "no device-driven BFS has run on this graph");
    CK(cudaMemcpy(g->ws->h_ctrl, g->ws->ctrl, sizeof(BfsCtrl), cudaMemcpyDeviceToHost));
    const BfsCtrl &c = *g->ws->h_ctrl;
    const int n = (int)(c.tr_n < (unsigned long long)SG_TRACE_STEPS ? c.tr_n : SG_TRACE_STEPS);
    for (int i = 0; i < n && i < cap; i++) {
        if (t_ns) t_ns[i] = (int64_t)(c.t_ns[i] - c.t_ns[0]);
        if (kind) kind[i] = (int32_t)c.kind[i];
        if (count) count[i] = (int64_t)c.tr_count[i];
        if (nf) nf[i] = (int64_t)c.tr_nf[i];
        if (mf) mf[i] = (int64_t)c.tr_mf[i];
    }
    return n < cap ? n : cap;
}

}  // extern "C"
