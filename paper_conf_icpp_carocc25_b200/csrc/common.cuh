// common.cuh — shared device/host definitions of the B200 Two-Layer-Bitmap advance.
// Layout (DESIGN.md §4, §4.1 and :253 §4.3, readings C1-C3):
//   layer 1  uint64 bits[nw1], nw1 = ceil(n/64): vertex v = bit (v & 63) of word (v >> 6)
//   layer 2  uint64 summ[nw2], nw2 = ceil(nw1/64): bit (w & 63) of word (w >> 6) <=> bits[w] != 0
#pragma once
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

namespace sg {

constexpr uint32_t INF32 = 0xFFFFFFFFu;
constexpr int WARP = 32;

// ---- 1-D destination partition over peer memory (xchg.cuh, comm.cu) ----------
constexpr int SG_MAX_RANKS = 8;
// One rank's contribution to a superstep's statistics, published into every peer's control
// block (double-buffered by epoch parity).
struct XSlot {
    unsigned long long epoch;   // barrier number this slot belongs to (written last, release)
    unsigned long long nf, mf, arcs;
};
// Exchange control block: lives at the start of each rank's IPC-shared arena.
struct XCtl {
    unsigned long long epoch;   // barriers passed by this rank (local)
    unsigned long long error;   // a peer did not arrive within the timeout (host reports SG_ERR_NCCL)
    unsigned long long pad[6];
    XSlot slots[2][SG_MAX_RANKS];
};
// Kernel-visible exchange descriptor (by value).  nranks <= 1: single GPU, every helper is local.
// Every rank's arena has the same layout, so the peer copy of a local arena pointer p is
// p + delta[j] (bytes; delta[rank] = 0).
struct Xchg {
    int32_t nranks = 0, rank = 0;
    long long delta[SG_MAX_RANKS] = {};
    XCtl *ctl = nullptr;
};

// Graph as the kernels see it (device pointers).
struct GraphView {
    const int64_t *__restrict__ rp;    // row_ptr[n+1]
    const int32_t *__restrict__ col;   // col_idx[nnz] (+16 B zero padding for 16-B bulk copies)
    const uint8_t *__restrict__ w;     // weights[nnz] or nullptr
    const uint8_t *__restrict__ deg8;  // 8-bit log-coded degrees, nw1*64 bytes (direction policy only)
    const int32_t *__restrict__ fnbr;  // pull candidate: neighbour of largest degree among the first arcs, -1 if none
    int64_t n, nnz;
    int64_t nw1, nw2;
    const int32_t *__restrict__ hub_idx;   // hub index of u (deg >= SEG_MIN) or -1; nullptr: no segmentation
    const uint32_t *__restrict__ hub_off;  // [nhubs][nseg+1] neighbours of the hub with id < b*SEG_V
    int32_t nseg;                          // ceil(n / SEG_V)
    // owned destination range (1-D partition); single GPU: everything.  Ranges are
    // 4,096-vertex aligned (except hi = n), so owned layer-1 and layer-2 words are whole.
    int64_t own_lo = 0, own_hi = 0;        // vertices
    int64_t w1_lo = 0, w1_hi = 0;          // layer-1 words
    int64_t w2_lo = 0, w2_hi = 0;          // layer-2 words
};

// Destination-segmented copy of the arcs (scsr.cu): segment b = vertices [b*sv, (b+1)*sv), sv =
// 64*sw <= 2^20; block b = for u = 0..n-1 the arcs of u into segment b, each stored as
// (u mod 4096) << 20 | (v - b*sv).
struct ScsrView {
    const uint32_t *__restrict__ col;    // tagged segment-major arcs (+64 B padding)
    const uint32_t *__restrict__ base;   // [nseg][nw1+1] first arc of word w's parts, relative to start[b]
    const int64_t *__restrict__ start;   // [nseg] first arc of block b
    uint32_t *qc;                        // [nseg] work-item counters (zeroed before each advance)
    int64_t nw1, sv;
    int32_t nseg, sw;
};

// Per-superstep control block, device resident; host reads it back with one 64-B copy.
struct DevStats {
    unsigned long long count;        // non-zero layer-1 words listed in offsets (summary compaction)
    unsigned long long nf;           // active vertices (popcount) — direction policy
    unsigned long long mf;           // sum of active vertices' degrees — direction policy
    unsigned long long arcs;         // arcs inspected by the advance
    unsigned long long batch;        // push: next word batch (dynamic CTA scheduling)
    unsigned long long heavy_count;  // push: CTA/grid-tier chunks queued
    unsigned long long seg_count;    // push: destination-segmented hub chunks queued (BFS)
    unsigned long long pad;          // partitioned host loops: the superstep's global arcs
    unsigned long long scans;        // pull: vertices whose candidate missed (a row_ptr pair + list scan)
    unsigned long long pad2;
};

constexpr int SG_TRACE_STEPS = 48;

// Device-resident state of a graph-driven SSSP / CC run (vloop: WHILE { half 0 | half 1 }, per
// half an IF(push) and an IF(pull) node; the output kernel's last CTA decides).
struct ValCtrl {
    unsigned long long iters, push_steps, pull_steps, arcs_pushed, arcs_pulled;
    long long max_iters, nnz;
    uint32_t overflow;
    uint32_t cc;             // 1: CC (pull when the frontier's arcs exceed nnz/4 in AUTO), 0: SSSP (push)
    uint32_t direction;      // SG_DIR_*
    uint32_t pull;           // direction of the superstep being launched
    uint32_t hmask;          // current IF handle values (bit 2k+b: kind k (0 push, 1 pull) of buffer b; bit 8 loop)
    int32_t src;             // SSSP source (the prologue kernel seeds it)
    unsigned long long hl, hpush[2], hpull[2];
};

// A graph-driven BFS's final counters, written by the stopping decision straight into mapped
// pinned host memory (no device->host copy after the graph: ~7 us per BFS, scripts/micro/bfs_fixed_cost.py)
struct BfsResult {
    unsigned long long iters, push_steps, pull_steps, arcs_pushed, arcs_pulled, reached, sweep_steps, sparse_steps,
        hub_steps;
    uint32_t overflow, done;
};

// Device-resident state of a graph-driven BFS (written by k_bfs_decide, read back once per run).
struct BfsCtrl {
    unsigned long long iters, push_steps, pull_steps, arcs_pushed, arcs_pulled, reached;
    long long mu;            // sum of degrees of unvisited vertices (Beamer m_u, estimate)
    long long nf_prev;
    long long n, max_iters;
    double alpha, beta;
    uint32_t *level;         // output buffer of this run (kernels read the pointer: one graph serves any buffer)
    int32_t src;
    uint32_t next;           // level value written by the superstep being launched
    uint32_t pull;           // direction of the superstep being launched
    uint32_t auto_dir;
    uint32_t overflow;       // iteration cap hit
    uint32_t sweep_mode;     // push supersteps through the sweep: 0 never, 1 when m_f >= sweep_thr, 2 always
    unsigned long long sweep_thr;
    unsigned long long sweep_steps;
    // fused small-frontier supersteps (sparse.cu): taken when count <= sparse_words and m_f <= sparse_arcs
    uint32_t sparse_mode;    // 0 off, 1 on
    uint32_t pad0;
    unsigned long long sparse_words, sparse_arcs, sparse_steps;
    // frontier buffer b still holds a consumed frontier (dirty[b]) whose word list had
    // saved_count[b] entries (~0: unknown, clear every word); the sparse kernel needs an all-zero
    // output buffer and clears it first when dirty
    uint32_t dirty[2];
    unsigned long long saved_count[2];
    // conditional handles of the graph (cudaGraphConditionalHandle values; 0 = no such node):
    // the loop, and per frontier buffer b the IF nodes of the supersteps whose input is buffer b
    unsigned long long hl, hpush[2], hpull[2], hsweep[2], hsparse[2];
    unsigned long long dbg[16];   // phase time accumulators of the fused sparse loop (CTA 0, ns; sg_ctrl_debug)
    uint32_t pull_warp[2];   // a pull whose input is buffer b runs warp-owned layer-2 words (late pulls);
                             // indexed by buffer: the decision writes the next input's entry while
                             // both pull kernels of the current superstep read the current one
    uint32_t pull_warp_frac; // ... when unvisited non-isolated vertices < (n - n_iso) / pull_warp_frac
    long long n_iso;         // isolated vertices (visited from the start, never reached)
    long long src_iso;       // 1 iff the source itself is one of them (counted in reached too)
    BfsResult *res;          // mapped host memory: the stopping decision writes the run's counters there
    uint32_t sp_kind;        // the fused sparse loop's last decision (read by all its CTAs)
    uint32_t sp_epoch;       // bumped by CTA 0 once sp_kind is written (the loop's broadcast)
    uint32_t hmask;          // current values of the IF handles (bit 2k+b: kind k of buffer b; bit 8: loop);
    uint32_t pad1;           // only changed handles are set (cudaGraphSetConditional costs ~0.4 us)
    // per-superstep trace (sg_bfs_trace): globaltimer at each decision, the decision taken
    // (0 stop, 1 push, 2 pull, 3 sweep, 4 sparse) and the frontier it was taken on
    unsigned long long tr_n;
    unsigned long long t_ns[SG_TRACE_STEPS];
    uint32_t kind[SG_TRACE_STEPS];
    unsigned long long tr_count[SG_TRACE_STEPS], tr_nf[SG_TRACE_STEPS], tr_mf[SG_TRACE_STEPS];
};

// Device-resident control of one source-batched BC batch (bcb.cu).
struct BcbCtrl {
    int32_t src[32];
    int32_t nsrc;
    int32_t d;                 // current level
    int32_t par;               // frontier-mask parity
    int32_t depth;             // number of levels
    unsigned long long ltop;   // entries appended to the level lists
    int32_t overflow;          // level / list capacity exceeded
    int32_t pad;
    unsigned long long t_ns[6];   // per-phase time (globaltimer, CTA 0 view): fwd A, A2, B; bwd A, B
};

// One CTA/grid-tier work unit: a contiguous piece of one vertex's adjacency list.
struct HeavyItem {
    int64_t begin;   // first arc index
    int32_t len;     // number of arcs (<= HEAVY_CHUNK)
    int32_t u;       // source vertex
};

constexpr int HEAVY_CHUNK = 4096;     // arcs per CTA-tier work unit (16 KB of col_idx)

// Destination-segmented hub tier (BFS): the visited bitmap is processed in segments of SEG_V
// vertices whose slice (SEG_V/8 bytes) fits one CTA's shared memory; hub rows (deg >= SEG_MIN)
// carry per-segment offsets computed at graph load.
constexpr int SEG_WORDS = 24576;                       // 192 KB of layer-1 words per slice
constexpr int64_t SEG_V = (int64_t)SEG_WORDS * 64;     // 1,572,864 vertices per segment
#ifndef SG_SEG_MIN
#define SG_SEG_MIN 256
#endif
constexpr int SEG_MIN = SG_SEG_MIN;                    // hub threshold (degree)
struct SegItem {
    int64_t begin;   // first arc of the chunk
    int64_t row;     // row_ptr[u] (segment offsets are relative to it)
    int32_t len;     // arcs in the chunk (<= HEAVY_CHUNK)
    int32_t h;       // hub index (row of the segment-offset table)
};

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// 8-bit log-coded degree (graph load, frontier.cu k_deg8): exact below 32, else 3 mantissa bits
__device__ __forceinline__ uint32_t deg8_decode(uint32_t c) {
    if (c < 32u) return c;
    const uint32_t e = ((c - 32u) >> 3) + 5u, m = (c - 32u) & 7u;
    return ((8u + m) << (e - 3u)) + (1u << (e - 4u));
}

__device__ __forceinline__ unsigned long long atomic_or_u64(uint64_t *p, uint64_t m) {
    return atomicOr(reinterpret_cast<unsigned long long *>(p), (unsigned long long)m);
}

// Insert v into a 2LB frontier; returns true iff this call flipped v's bit (0 -> 1).
// The summary bit is touched only on the word's 0 -> non-zero transition.
__device__ __forceinline__ bool insert_2lb(uint64_t *bits, uint64_t *summ, int32_t v) {
    const uint64_t m = 1ull << (v & 63);
    const unsigned long long old = atomic_or_u64(bits + (v >> 6), m);
    if (old == 0ull) atomic_or_u64(summ + (v >> 12), 1ull << ((v >> 6) & 63));
    return (old & m) == 0ull;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T x) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane_id() >= o) x += y;
    }
    return x;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

// Plain (L1-cacheable) 64-bit load of a word that other threads may be updating with
// atomics during the kernel: a stale value only costs an extra atomic, never correctness.
__device__ __forceinline__ uint64_t ld_word(const uint64_t *p) { return *p; }

// Load row_ptr bounds for the (up to) two vertices a = 64w + lane, b = 64w + 32 + lane of a
// word.  Dense words read rp[64w .. 64w+64] coalesced (3 warp loads); sparse words let only
// active lanes read their two entries.
__device__ __forceinline__ void word_bounds(const GraphView &g, int64_t w, uint64_t x, int64_t &sa, int64_t &ea,
                                            int64_t &sb, int64_t &eb) {
    const int lane = lane_id();
    const bool act_a = (x >> lane) & 1ull, act_b = (x >> (lane + 32)) & 1ull;
    const int64_t base = w * 64;
    if (__popcll(x) > 12) {
        const int64_t n = g.n;
        const int64_t r0 = __ldg(g.rp + min(base + lane, n));
        const int64_t r1 = __ldg(g.rp + min(base + 32 + lane, n));
        const int64_t r2 = __ldg(g.rp + min(base + 64, n));
        const int64_t r0n = __shfl_down_sync(0xffffffffu, r0, 1);
        const int64_t r1n = __shfl_down_sync(0xffffffffu, r1, 1);
        const int64_t r1f = __shfl_sync(0xffffffffu, r1, 0);
        sa = r0; ea = lane < 31 ? r0n : r1f;
        sb = r1; eb = lane < 31 ? r1n : r2;
        if (!act_a) ea = sa;
        if (!act_b) eb = sb;
    } else {
        sa = ea = sb = eb = 0;
        if (act_a) { sa = __ldg(g.rp + base + lane); ea = __ldg(g.rp + base + lane + 1); }
        if (act_b) { sb = __ldg(g.rp + base + 32 + lane); eb = __ldg(g.rp + base + 33 + lane); }
    }
}

}  // namespace sg

// ---- host helpers --------------------------------------------------------------------------
namespace sg {
// SM count of the current device, queried once per device (grid sizing: multiples of the SM count)
inline int num_sms() {
    static int cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148;
    if (!cache[dev]) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cache[dev] = n > 0 ? n : 148;
    }
    return cache[dev];
}

// ---- device memory: one private stream-ordered pool per device (release threshold = infinity),
// so a graph loaded after another one of similar size reuses its memory without new driver
// mappings (graph_load_csr / graph_free in a loop: the e2e step).  Private, so the process's
// default pool (used by NCCL or torch's cudaMallocAsync backend) keeps its own policy; graph_free
// trims the pool back to what is still allocated once it is idle (dev_trim).
inline cudaMemPool_t graph_pool() {
    static cudaMemPool_t pools[64] = {};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
    if (!pools[dev]) {
        cudaMemPoolProps p = {};
        p.allocType = cudaMemAllocationTypePinned;
        p.handleTypes = cudaMemHandleTypeNone;
        p.location.type = cudaMemLocationTypeDevice;
        p.location.id = dev;
        cudaMemPool_t pool;
        if (cudaMemPoolCreate(&pool, &p) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        uint64_t thr = ~0ull;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = pool;
    }
    return pools[dev];
}
inline cudaError_t dev_alloc(void **p, size_t bytes, cudaStream_t s) {
    static const bool dflt = getenv("SG_DEFAULT_POOL") != nullptr;   // A/B knob: the device's default pool
    if (dflt) return cudaMallocAsync(p, bytes, s);
    cudaMemPool_t pool = graph_pool();
    if (!pool) return cudaMallocAsync(p, bytes, s);
    return cudaMallocFromPoolAsync(p, bytes, pool, s);
}
template <class T>
inline cudaError_t dev_alloc(T **p, size_t bytes, cudaStream_t s) {
    return dev_alloc(reinterpret_cast<void **>(p), bytes, s);
}
// the caller guarantees no pending work uses p (graph_free synchronises the device first)
inline void dev_free(void *p) {
    if (p) cudaFreeAsync(p, 0);
}
// release the pool's unused memory beyond `keep` bytes (graph_free with no other graph alive)
inline void dev_trim(size_t keep) {
    cudaMemPool_t pool = graph_pool();
    if (pool) cudaMemPoolTrimTo(pool, keep);
}
}  // namespace sg
