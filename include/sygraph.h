/*
 * sygraph.h — C ABI of the B200-native Two-Layer-Bitmap frontier advance
 * (SYgraph, De Caro/Cordasco/Cosenza, ICPP'25; /root/reference/PAPER.md = "P:<line>").
 *
 * Plain C: pointers + sizes, no torch/C++ types.  Every function returns an int status
 * (SG_OK = 0, < 0 on error) and never throws; sg_last_error() gives a thread-local message.
 * Handles are not thread-safe (one host thread per handle at a time).  Device pointers are
 * CUDA device addresses on the current device; `stream` arguments are cudaStream_t values
 * (NULL = legacy default stream).
 *
 * Data layout (readings C1-C3):
 *   graph     symmetric CSR, vertex ids int32, row_ptr int64[n+1], col_idx int32[nnz] with
 *             every row sorted ascending, no self-loops or multi-edges (§3.1; C8, C9);
 *             optional weights uint8[nnz] (SSSP; w(u,v) = w(v,u); C11).
 *   frontier  Two-Layer Bitmap (§4.3): layer 1 = uint64 bits[ceil(n/64)], vertex v is
 *             bit (v & 63) of word (v >> 6) (LSB first; §4.1); layer 2 = uint64
 *             summ[ceil(n/4096)], bit (w & 63) of word (w >> 6) is set iff bits[w] != 0.
 *             Bits >= n are always 0.
 */
#ifndef SYGRAPH_H
#define SYGRAPH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SG_API __attribute__((visibility("default")))

enum sg_status {
    SG_OK = 0,
    SG_ERR_INVALID = -1,      /* bad argument (range, NULL, malformed CSR under SG_F_VALIDATE) */
    SG_ERR_OOM = -2,          /* device allocation failed */
    SG_ERR_CUDA = -3,         /* CUDA runtime/launch error (message in sg_last_error) */
    SG_ERR_NCCL = -4,         /* partition exchange failure (bootstrap socket, IPC mapping, peer timeout) */
    SG_ERR_UNSUPPORTED = -5,  /* valid request outside the implemented envelope */
    SG_ERR_STATE = -6         /* missing functor state / iteration cap hit / handle misuse */
};
enum { SG_MEM_HOST = 0, SG_MEM_DEVICE = 1 };          /* where input arrays live */
/* graph_load_csr flags:
 *   SG_F_BORROW    with SG_MEM_DEVICE: keep the caller's row_ptr / col_idx / weights pointers (no
 *                  copy; e.g. torch tensors).  The caller keeps them alive and unmodified until
 *                  graph_free.  col_idx must be 16-B aligned and its allocation must extend >= 64
 *                  readable bytes past nnz*4 (16-B vector loads of a row's tail; torch's caching
 *                  allocator rounds blocks to 512 B); weights likewise past nnz.  Checked, else
 *                  SG_ERR_INVALID.
 *   SG_F_VALIDATE  O(nnz log deg) device check of the CSR contract (§3.1; readings C8, C9):
 *                  row_ptr[0] = 0, row_ptr[n] = nnz, row_ptr monotone, 0 <= col < n, every row
 *                  strictly ascending (sorted, no multi-edges), no self-loops, and symmetric
 *                  (every arc (u,v) has its reverse (v,u)).  Any violation -> SG_ERR_INVALID.
 *   Without SG_F_VALIDATE row order is still checked (O(nnz), every load): a graph whose rows are
 *   not sorted loads, but its hub-segmented push tier, segment-major sweep and label-blocked CC
 *   pull (which binary-search sorted rows) are disabled for it; results stay exact.             */
/*   SG_F_DIRECTED  the CSR holds out-arcs of a directed graph (§3.1 "CSR and CSC"; P:299
 *                  directed datasets): the library builds the transpose (CSC, rows
 *                  sorted) for pull steps, and a vertex with no in-arc is unreachable.  run_bfs /
 *                  run_sssp / advance follow arc direction; run_cc / run_bc need a symmetric graph
 *                  (SG_ERR_UNSUPPORTED); SG_F_VALIDATE skips the symmetry check; single GPU only. */
enum { SG_F_BORROW = 1, SG_F_VALIDATE = 2, SG_F_DIRECTED = 4 };
enum { SG_FN_BFS = 0, SG_FN_SSSP = 1, SG_FN_CC = 2, SG_FN_BC_SIGMA = 3 };   /* advance functors */
enum { SG_DIR_AUTO = 0, SG_DIR_PUSH = 1, SG_DIR_PULL = 2 };                 /* BFS direction */

typedef struct sg_graph sg_graph;
typedef struct sg_frontier sg_frontier;
typedef struct sg_comm sg_comm;         /* ranks of a 1-D destination partition (one process per GPU) */

/* Functor states for advance(): device pointers + scalars (Table 2: an advance functor
 * (src, dst, edge, weight) -> bool decides whether dst enters the output frontier). */
typedef struct {              /* BFS (Listing 1): dst enters iff not yet visited; the   */
    uint32_t *level;          /* inserting thread writes level[dst] = depth + 1 and sets visited.  */
    uint64_t *visited;        /* layer-1-shaped bitmap (ceil(n/64) words), updated in place        */
    uint32_t depth;
} sg_bfs_state;
typedef struct {              /* SSSP relax (P:161 Bellman-Ford): nd = dist[src] + w; dst enters  */
    uint32_t *dist;           /* iff atomicMin(&dist[dst], nd) > nd.  Weights come from the graph. */
} sg_sssp_state;
typedef struct {              /* CC label propagation: dst enters iff                      */
    int32_t *label;           /* atomicMin(&label[dst], label[src]) > label[src].                  */
} sg_cc_state;
typedef struct {              /* BC forward sigma (P:161 Brandes): dst not in `visited` (frozen for */
    uint32_t *level;          /* the step) gets sigma[dst] += sigma[src] and enters the output; its */
    uint64_t *visited;        /* inserting thread writes level[dst] = depth + 1.  The caller ORs   */
    double *sigma;            /* the output into `visited` afterwards (frontier_or_into).           */
    int32_t *exp2_per_level;  /* device int32[>= depth + 2]: sigma of level L is stored as          */
    uint32_t depth;           /* sigma_true * 2^-E[L] (reading C20 / DESIGN R5).  After the step the */
} sg_bc_state;                /* new level (the output frontier, which must start empty) is scaled */
                              /* so its maximum lies in [1, 2) and E[depth+1] = E[depth] + k is     */
                              /* written (E[0] = 0 is the caller's).  Without it sigma overflows    */
                              /* fp64 on high-diameter graphs: NULL -> SG_ERR_STATE.                */

typedef struct {
    void *stream;             /* cudaStream_t; NULL = legacy default stream */
    int direction;            /* SG_DIR_* for run_bfs (default AUTO = Beamer direction optimising) */
    double alpha, beta;       /* Beamer thresholds (defaults 5, 48: tuned on B200, DESIGN R2): push->pull when m_f > m_u/alpha,
                                 pull->push when n_f < n/beta */
    int64_t max_iters;        /* superstep cap (0 = n + 1); exceeding it returns SG_ERR_STATE */
    int32_t heavy_degree;     /* push tiers: degree > heavy_degree goes to the CTA/grid tier (0 = default) */
    int32_t small_degree;     /* degree <= small_degree uses the thread-granular packed tier (0 = default, <0 = none) */
    int32_t host_loop;        /* run_bfs: 1 = host-driven superstep loop (one control read per level);
                                 0 = one CUDA graph with device-side control (default) */
    int32_t segmented;        /* BFS hub tier with the visited slice in shared memory:
                                 0 = auto (heavy supersteps), 1 = off, 2 = always */
    int32_t one_layer;        /* ablation (Fig. 7): 1 = push visits every layer-1 word (plain bitmap,
                                 no summary-layer compaction); host-driven loop only */
    int32_t coarsening;       /* push: layer-1 words per warp grab (CF); 0 = auto */
    int32_t sssp_delta;       /* run_sssp: 0 = frontier Bellman-Ford (the paper); D > 0 = near-far
                                 delta-stepping with bucket width D (P:161 refs [23,34]) */
    int32_t scsr;             /* run_bfs: heavy push supersteps over the destination-segmented arc copy
                                 (visited slice in shared memory, built at the first run_bfs that can use
                                 it, nnz x 4 B extra): 0 = auto (frontier arcs >= 4 Mi), 1 = off, 2 = always */
    int32_t owned_only;       /* partitioned graphs: 1 = run_bfs leaves level[] valid on this rank's owned
                                 range only (no result gather; each rank holds its part, as in Graph500);
                                 0 = level[] complete on every rank (default) */
    int32_t reserved[1];
} sg_opts;

typedef struct {
    int64_t iterations;       /* supersteps executed */
    int64_t push_steps, pull_steps;
    int64_t arcs_pushed;      /* sum of frontier degrees over push steps (arcs inspected by push) */
    int64_t arcs_pulled;      /* arcs scanned by pull steps (early exit at the first parent) */
    int64_t reached;          /* vertices with a finite result (BFS/SSSP) */
    double device_ms;         /* CUDA-event time of the call on its stream */
} sg_stats;

/* ---- communicator (§6 "static graph partitioning") ------------ */
/* The ranks of a 1-D destination partition: one process per GPU on one node.  The communicator
 * is a host-side bootstrap (TCP on 127.0.0.1, or SG_COMM_ADDR) used at graph-load time to agree
 * on the partition and to exchange the CUDA IPC handles of each rank's exchange arena; every
 * per-superstep exchange then runs inside the kernels over peer memory (NVLink P2P; two ranks
 * may share one GPU, e.g. for tests).  Usage: rank 0 calls comm_unique_id, the caller broadcasts
 * the 128 bytes (e.g. torch.distributed.broadcast_object_list), every rank calls comm_init with
 * its rank and the CUDA device it uses.  Blocking; 120 s connect timeout -> SG_ERR_NCCL. */
SG_API int comm_unique_id(uint8_t id[128]);
SG_API int comm_init(const uint8_t id[128], int nranks, int rank, int device, sg_comm **out);
SG_API int comm_free(sg_comm *c);
SG_API int comm_info(const sg_comm *c, int *nranks, int *rank);

/* ---- graph ---------------------------------------------------------------------------- */
/* Copy a symmetric CSR to device memory owned by the returned handle (§3.1; timing of
 * the paper excludes this transfer).  mem = SG_MEM_HOST | SG_MEM_DEVICE says where the
 * three input arrays live; weights may be NULL.  n in [1, 2^31-1], nnz in [0, 2^40].
 * flags: SG_F_BORROW / SG_F_VALIDATE (above).  Synchronises `stream` before returning.
 * comm (nullable; nranks == 1 behaves as NULL): collective over the communicator's ranks, which
 * all pass the same full CSR (SG_ERR_INVALID if their partitions disagree).  Rank r keeps only
 * its partition: owned destinations [lo_r, hi_r) (4,096-aligned, arc-balanced;
 * graph_partition), the push block (arcs of every source into the owned range) and the pull
 * block (the owned rows).  Rows must be sorted (SG_ERR_UNSUPPORTED otherwise).  run_bfs /
 * run_sssp / run_cc on such a graph are collective (every rank calls them with the same
 * arguments, in the same order); advance / run_bc return SG_ERR_UNSUPPORTED (BC shards sources
 * over full replicas instead). */
SG_API int graph_load_csr(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col_idx,
                          const uint8_t *weights, int mem, int flags, void *stream, sg_comm *comm, sg_graph **out);
/* Owned destination range of a partitioned graph ([0, n) for a single-GPU graph). */
SG_API int graph_partition(const sg_graph *g, int64_t *lo, int64_t *hi);
SG_API int graph_free(sg_graph *g);
SG_API int graph_info(const sg_graph *g, int64_t *n, int64_t *nnz, const int64_t **row_ptr,
                      const int32_t **col_idx, const uint8_t **weights);

/* ---- frontier (§3.1, §3.2, Listing 1) -------------------------------------- */
/* Empty 2LB frontier sized for g (library-owned device memory). */
SG_API int frontier_init(const sg_graph *g, sg_frontier **out);
SG_API int frontier_free(sg_frontier *f);
/* Insert k vertex ids (host or device array per `mem`); ids outside [0,n) -> SG_ERR_INVALID
 * (host arrays are checked; device arrays are range-masked on the device). Async. */
SG_API int frontier_insert(sg_frontier *f, const int32_t *v, int64_t k, int mem, void *stream);
/* All vertices active (advance::vertices, Table 2). Async. */
SG_API int frontier_fill_all(sg_frontier *f, void *stream);
SG_API int frontier_clear(sg_frontier *f, void *stream);
/* Number of active vertices (popcount); synchronises `stream`. */
SG_API int frontier_count(const sg_frontier *f, int64_t *out, void *stream);
/* Device pointers of the two layers and their word counts (read/write views). */
SG_API int frontier_view(const sg_frontier *f, uint64_t **bits, uint64_t **summ, int64_t *nw1, int64_t *nw2);
/* Frontier set operators (§3.1, §4.1), word-parallel: dst = dst OP src,
 * op 0 = union (OR), 1 = intersection (AND), 2 = subtraction (AND NOT), 3 = symmetric
 * difference (XOR).  The summary layer is rebuilt. Async. */
SG_API int frontier_op(sg_frontier *dst, const sg_frontier *src, int op, void *stream);
/* OR the layer-1 words of f into a plain bitmap `dst` (ceil(n/64) words). Async. */
SG_API int frontier_or_into(const sg_frontier *f, uint64_t *dst, void *stream);

/* ---- filter / compute (Table 2, §3.1) ---------------------------------- */
/* The paper's Filter / Compute functors are C++ lambdas; across this ABI they are a predicate /
 * operation code with parameters.  Predicates on vertex v (a, b are doubles):
 *   SG_PRED_DEGREE_RANGE  a <= deg(v) < b               (array unused)
 *   SG_PRED_U32_RANGE     a <= ((uint32*)array)[v] < b   (device array[n])
 *   SG_PRED_I32_RANGE     a <= ((int32*)array)[v] < b
 *   SG_PRED_F64_RANGE     a <= ((double*)array)[v] < b
 *   SG_PRED_IN_BITMAP     bit v of the layer-1-shaped device bitmap `array`                  */
enum { SG_PRED_DEGREE_RANGE = 0, SG_PRED_U32_RANGE = 1, SG_PRED_I32_RANGE = 2, SG_PRED_F64_RANGE = 3,
       SG_PRED_IN_BITMAP = 4 };
/* filter::inplace(G, F, pred) when out == NULL: removes failing elements from `in`; a word that
 * becomes 0 resets its layer-2 bit.  filter::external(G, In, Out, pred) otherwise:
 * passing elements are inserted into `out` (not cleared first).  Async. */
SG_API int frontier_filter(sg_frontier *in, sg_frontier *out, int pred, const void *array, double a, double b,
                           void *stream);
/* compute::execute(G, F, op): for every active v:
 *   SG_OP_SET_U32 / SG_OP_SET_I32 / SG_OP_SET_F64: array[v] = value
 *   SG_OP_ADD_U32 / SG_OP_ADD_F64:                 array[v] += value      (device array[n]). Async. */
enum { SG_OP_SET_U32 = 0, SG_OP_SET_I32 = 1, SG_OP_SET_F64 = 2, SG_OP_ADD_U32 = 3, SG_OP_ADD_F64 = 4 };
SG_API int compute_execute(const sg_frontier *f, int op, void *array, double value, void *stream);

/* ---- advance (Table 2; §4.2-4.3) ----------------------------------- */
/* One push advance superstep: compacts the summary layer of `in` into the offsets buffer
 * (P:255), then expands every active vertex's adjacency with the degree-tiered load balance,
 * applying `functor` (SG_FN_*) per edge with `functor_state` (pointer to the matching
 * sg_*_state struct, host memory, read at call time).  Vertices for which the functor
 * returns true are inserted into `out` (both layers); out may be NULL (advance without an
 * output frontier).  `out` is not cleared first.  Stream-ordered, returns after
 * enqueue (the paper's returned event). SG_FN_SSSP needs graph weights. */
SG_API int advance(const sg_graph *g, const sg_frontier *in, sg_frontier *out, int functor,
                   const void *functor_state, void *stream);

/* ---- algorithms (§3.4) — return when the result is complete on opts->stream ------ */
/* BFS levels from src (Listing 1): level[src] = 0, UINT32_MAX = unreached. level: device[n]. */
SG_API int run_bfs(const sg_graph *g, int32_t src, uint32_t *level, const sg_opts *opts, sg_stats *stats);
/* SSSP distances (Bellman-Ford by frontier relaxation, no delta-stepping).
 * dist: device[n], UINT32_MAX = unreached. Needs weights; SG_ERR_UNSUPPORTED if
 * max_weight * (n-1) >= 2^32-1. */
SG_API int run_sssp(const sg_graph *g, int32_t src, uint32_t *dist, const sg_opts *opts, sg_stats *stats);
/* Connected components by label propagation: label[v] = min id of v's component. */
SG_API int run_cc(const sg_graph *g, int32_t *label, const sg_opts *opts, sg_stats *stats);
/* Betweenness centrality (Brandes, forward sigma + backward delta): bc[v] = sum over
 * the k host-array sources of delta_s(v), unnormalised (reading C14). bc: device[n], overwritten. */
SG_API int run_bc(const sg_graph *g, const int32_t *sources, int32_t k, double *bc, const sg_opts *opts,
                  sg_stats *stats);

/* ---- measurement (bench.py roofline; not needed for correctness) ----------------------- */
enum { SG_K_COMPACT = 0, SG_K_STATS = 1, SG_K_PUSH = 2, SG_K_PULL = 3, SG_K_BC = 4, SG_K_SWEEP = 5, SG_K_COUNT = 6 };
/* SG_K_SWEEP: push supersteps taken by the destination-segmented sweep (sg_opts.scsr). */
typedef struct {
    double ms;                /* summed CUDA-event time of the class's launches (launching stream) */
    double bytes;             /* summed algorithmic HBM bytes */
    int64_t launches;         /* profiled launches (a push advance = its word + CTA-tier kernels) */
} sg_kprof;
/* Enable (1) / disable (0) per-kernel-class event timing for run_bfs on g; resets totals. */
SG_API int sg_profile(sg_graph *g, int enable);
/* Copy the SG_K_COUNT per-class totals. */
SG_API int sg_profile_read(const sg_graph *g, sg_kprof *out);
/* Kernel launches issued by this library since load (host-side counter). */
SG_API int64_t sg_launch_count(void);
/* Per-superstep trace of the last device-driven run_bfs on g: for decision i (i = 0 is the
 * prologue's), globaltimer ns since decision 0, the decision (0 stop, 1 push, 2 pull, 3 sweep,
 * 4 fused sparse superstep) and the frontier it was taken on (words, n_f, m_f).  Returns the
 * number of entries (<= cap); pointers may be NULL. */
/* Word-width ablation (§4.3 "32-bit integer to match a warp on NVIDIA"): a
 * self-contained push-only Two-Layer-Bitmap BFS with word_bits = 32 (one bit per lane) or 64 (two
 * per lane) words in both layers, the paper's warp-per-word / lanes-stride-the-list mapping,
 * host-driven loop.  Same levels as run_bfs (level: device[n]); device_ms = its time. */
SG_API int sg_ablation_bfs(const sg_graph *g, int32_t src, uint32_t *level, int32_t word_bits, void *stream,
                           sg_stats *stats);
/* Debug accumulators of the last device-driven run_bfs (fused sparse loop phase times, ns). */
SG_API int sg_ctrl_debug(const sg_graph *g, int64_t out[16]);
SG_API int sg_bfs_trace(const sg_graph *g, int64_t *t_ns, int32_t *kind, int64_t *count, int64_t *nf, int64_t *mf,
                        int32_t cap);

/* Defaults for sg_opts (stream NULL, AUTO direction, alpha 5, beta 48). */
SG_API void sg_opts_default(sg_opts *o);
/* Thread-local message of the last error on this thread ("" if none). */
SG_API const char *sg_last_error(void);
/* Library build/version string. */
SG_API const char *sg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SYGRAPH_H */
