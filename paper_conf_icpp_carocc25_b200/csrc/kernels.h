// kernels.h — host-side launchers of the sm_100a kernels (internal to libsygraph).
#pragma once
#include <cstddef>
#include <cuda_runtime.h>
#include <cstdint>
#include <vector>
#include "common.cuh"

namespace sg {

struct PushParams;

// host-side count of kernel launches issued by the library (bench evidence: gpu_launches)
void note_launch();

// frontier.cu
void launch_fill_all(uint64_t *bits, uint64_t *summ, int64_t n, int64_t nw1, int64_t nw2, cudaStream_t s);
void launch_insert(uint64_t *bits, uint64_t *summ, const int32_t *v, int64_t k, int64_t n, cudaStream_t s);
void launch_setop(uint64_t *dst, const uint64_t *src, int64_t nw1, int op, cudaStream_t s);
void launch_rebuild_summary(const uint64_t *bits, uint64_t *summ, int64_t nw1, int64_t nw2, cudaStream_t s);
void launch_compact(const uint64_t *summ, int64_t nw2, uint32_t *offsets, DevStats *st, cudaStream_t s);
void launch_frontier_stats(const GraphView &g, const uint64_t *bits, DevStats *st, cudaStream_t s);
void launch_isolated(const uint8_t *deg8, int64_t n, int64_t nw1, uint64_t *iso, cudaStream_t s);
void launch_deg8(const int64_t *rp, int64_t n, int64_t npad, uint8_t *deg8, cudaStream_t s);
void launch_first_nbr(const int64_t *rp, const int32_t *col, const uint8_t *deg8, int64_t n, int64_t npad,
                      int32_t *fn, cudaStream_t s);
void launch_popcount(const uint64_t *bits, int64_t nw1, unsigned long long *out, cudaStream_t s);
void launch_or_listed(const uint64_t *bits, const uint32_t *offsets, const DevStats *st, uint64_t *dst,
                      int64_t max_words, cudaStream_t s);
void launch_or_all(const uint64_t *bits, int64_t nw1, uint64_t *dst, cudaStream_t s);
void launch_set_u32(uint32_t *p, int64_t i, uint32_t v, cudaStream_t s);
void launch_set_i32(int32_t *p, int64_t i, int32_t v, cudaStream_t s);
void launch_set_f64(double *p, int64_t i, double v, cudaStream_t s);
void launch_iota_i32(int32_t *p, int64_t n, cudaStream_t s);
void launch_seed(uint64_t *bits, uint64_t *summ, uint64_t *visited, int32_t src, cudaStream_t s,
                 uint64_t *vis_old = nullptr);
void launch_validate_csr(const GraphView &g, unsigned long long *bad, cudaStream_t s);
// bad[0] += unsorted / duplicate pairs inside rows, bad[1] += self-loops (warp per row)
void launch_row_check(const GraphView &g, unsigned long long *bad, cudaStream_t s);
// bad[0] += arcs (v, u) whose reverse (u, v) is missing (rows must be sorted)
void launch_symmetry(const GraphView &g, unsigned long long *bad, cudaStream_t s);
void launch_max_weight(const uint8_t *w, int64_t nnz, unsigned int *out, cudaStream_t s);

// push.cu — one push advance = k_push_words (+ k_push_heavy), functor selected by `fn`.
struct PushLaunch {
    GraphView g;
    const uint64_t *in_bits;
    const uint32_t *offsets;
    DevStats *st;
    HeavyItem *heavy;
    uint32_t heavy_cap;
    int32_t heavy_deg, small_deg;
    int32_t batch;      // words per warp grab (coarsening factor; 0 = from the device-side count)
    int grid_words;     // CTAs for k_push_words
    int grid_heavy;     // CTAs for k_push_heavy
    SegItem *seg = nullptr;          // destination-segmented hub tier (BFS only)
    uint32_t seg_cap = 0;
    int32_t seg_mode = 0;            // 0 off, 1 auto, 2 always
    unsigned long long seg_threshold = 0;
    unsigned long long skip_mf = ~0ull;   // k_push_words returns at once if the frontier's m_f >= skip_mf (SCSR path)
    int32_t sparse_ok = 0;           // st->nf is exact (BFS): sparse frontiers take the thread-per-word path
};
void launch_hub_mark(const int64_t *rp, int64_t n, int32_t *hub_idx, int32_t *hub_vertex, unsigned int *count,
                     cudaStream_t s);
void launch_hub_off(const int64_t *rp, const int32_t *col, const int32_t *hub_vertex, int64_t nh, int nseg,
                    uint32_t *off, cudaStream_t s);
struct BfsArgs {
    uint64_t *visited;
    uint32_t *level;
    uint32_t next;
    uint64_t *out_bits, *out_summ;
    const uint32_t *next_ptr = nullptr;    // graph mode: read `next` / `level` from BfsCtrl
    uint32_t *const *level_pp = nullptr;
    uint32_t diff = 0;                     // 1: visited marks only; k_bfs_diff builds the output
};
struct SsspArgs { uint32_t *dist; uint64_t *out_bits, *out_summ; uint32_t diff = 0; };
struct CcArgs { int32_t *label; uint64_t *out_bits, *out_summ; };
struct BcArgs { const uint64_t *visited; double *sigma; uint32_t *level; uint32_t next; uint64_t *out_bits, *out_summ; };
void launch_push_bfs(const PushLaunch &L, const BfsArgs &a, cudaStream_t s);
void launch_push_sssp(const PushLaunch &L, const SsspArgs &a, cudaStream_t s);
void launch_push_cc(const PushLaunch &L, const CcArgs &a, cudaStream_t s);
void launch_push_bc(const PushLaunch &L, const BcArgs &a, cudaStream_t s);
int push_max_grid_words();
int push_max_grid_heavy();

// Output of a BFS superstep: new = visited & ~vis_old -> out 2LB, level[new] = next,
// vis_old |= new, the output's compacted word list (out offsets, st->count) and st->nf / st->mf
// (st zeroed before).  Every layer-1 and layer-2 word of the output is written (zero or not), so
// a BFS frontier never needs clearing.  Graph mode reads `next` / `level` through next_ptr /
// level_pp and, with ctrl set, the last CTA to finish runs the device-side direction policy
// (k_bfs_decide's logic: handles of the next superstep, prev = the input's control block).
struct BfsOut {
    uint64_t *vis_old;
    uint64_t *out_bits, *out_summ;
    uint32_t *out_offsets;
    uint32_t *level;
    uint32_t next;
    const uint32_t *next_ptr;
    uint32_t *const *level_pp;
    DevStats *st;
    BfsCtrl *ctrl;                    // NULL: host loop (no device-side decision; handles in ctrl)
    DevStats *prev;
    unsigned int *done;               // CTA completion counter (self-resetting)
    Xchg x;                           // partitioned: peers' replicas of the output (xchg.cuh)
    int32_t half = 0;                 // graph mode: index (0/1) of the INPUT frontier buffer
    int32_t sparse = 0;               // 1: the superstep consumed (zeroed) its input (sparse.cu)
    int32_t pull_warp = 0;            // host loop: 1 = the pull runs warp-owned layer-2 words (graph mode: ctrl)
    int32_t word_max = 16;            // CTA pull: word mode when no layer-1 word has more unvisited vertices
                                      // (SG_PULL_WORD_MAX at launch / capture; 0 = off)
    ValCtrl *vctrl = nullptr;         // graph-driven SSSP / CC: the last CTA runs val_decide
    // single-GPU BFS: the graph for the dead-end lookahead of a tiny output frontier (bfsstep.cuh)
    const int64_t *rp = nullptr;
    const int32_t *col = nullptr;
    const uint64_t *visited = nullptr;
};
// device-driven SSSP / CC: the first decision (after the prologue compacted the input), one thread
void launch_val_first(ValCtrl *c, const DevStats *st, cudaStream_t s);
void launch_val_seed(ValCtrl *c, uint32_t *dist, uint32_t *dist_old, uint64_t *bits, uint64_t *summ,
                     uint32_t *offsets, DevStats *st, cudaStream_t s);
// pull.cu — bottom-up BFS step (direction-optimising, Beamer): writes its output `o`
// itself (no k_bfs_diff after it); o.out_bits == NULL: marks visited only (k_bfs_diff after it)
void launch_pull_bfs(const GraphView &g, const uint64_t *in_bits, uint64_t *visited, DevStats *st, const BfsOut &o,
                     cudaStream_t s);
// sparse.cu — a whole small-frontier BFS superstep in one persistent kernel (graph mode only):
// push with direct output insertion, the input zeroed as consumed, the decision by its last CTA.
// gbar: 2 zeroed u32 (grid barrier).
void launch_bfs_sparse(const PushLaunch &L, const BfsArgs &a, const BfsOut &o, uint64_t *in_bits, uint64_t *in_summ,
                       unsigned int *gbar, cudaStream_t s);
// frontier.cu — output of a diff-mode BFS superstep (push word path / sweep): see BfsOut
void launch_bfs_diff(const GraphView &g, const uint64_t *visited, const BfsOut &o, cudaStream_t s);

// frontier.cu — output of a diff-mode SSSP superstep: the vertices whose distance decreased
// (dist < dist_old) -> the whole output 2LB + word list + st->count (st zeroed before);
// dist_old = dist
void launch_sssp_diff(const GraphView &g, const uint32_t *dist, uint32_t *dist_old, uint64_t *out_bits,
                      uint64_t *out_summ, uint32_t *out_offsets, DevStats *st, cudaStream_t s);
// the general form (SSSP dist / CC labels): output o (out_bits / out_summ / out_offsets / st,
// prev = the input's control block, x = peers), n_f (+ m_f when want_mf) into o.st; partitioned:
// owned words only, changed values + output replicated to the peers, superstep barrier at the end
void launch_value_diff(const GraphView &g, uint32_t *value, uint32_t *old, const BfsOut &o, int want_mf,
                       cudaStream_t s);

// filter.cu — filter::inplace / external, compute::execute (Table 2)
void launch_filter(const GraphView &g, const uint64_t *in_bits, uint64_t *out_bits, uint64_t *out_summ, int pred,
                   const void *array, double a, double b, int inplace, cudaStream_t s);
void launch_compute(const GraphView &g, const uint64_t *bits, int op, void *array, double value, cudaStream_t s);
void launch_min_over_bits(const GraphView &g, const uint64_t *bits, const uint32_t *a, unsigned int *out,
                          cudaStream_t s);

// pull_cc.cu — label-blocked pull for CC: per-row offsets of each label block (rows sorted),
// and one pass per block (out_bits written by pass 0, ORed by the others; summary by the caller)
void launch_cc_block_offsets(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, uint32_t *cbo,
                             cudaStream_t s);
void launch_pull_cc_block(const GraphView &g, int32_t *label, uint64_t *out_bits, DevStats *st, const uint32_t *cbo,
                          int nb, int b, cudaStream_t s);
// pull_cc.cu — block-major arc copy for the label-blocked CC pull: block b holds, for every v,
// v's neighbours in [b*S, (b+1)*S) contiguously at col[h_base[b] + off[b*(n+1) + v] ..)
struct CcBlocks {
    int nb = 0;
    int64_t S = 0;
    uint32_t *off = nullptr;       // [nb][n+1] offsets relative to the block's base
    int64_t *base = nullptr;       // [nb+1] device copy of h_base
    int32_t *col = nullptr;        // block-major arcs (+64 B padding)
    int64_t total = 0;
    std::vector<int64_t> h_base;
};
cudaError_t ccb_build(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, CcBlocks *out, cudaStream_t s);
void ccb_free(CcBlocks *B);
void launch_ccb_count(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, uint32_t *cnt, cudaStream_t s);
void launch_ccb_fill(const int64_t *rp, const int32_t *col, int64_t n, int nb, int64_t S, const uint32_t *off,
                     const int64_t *base, int32_t *out, cudaStream_t s);
// one label-blocked pull pass over block b (off = off[b], bcol = col + h_base[b])
void launch_pull_ccb(const GraphView &g, int32_t *label, uint64_t *out_bits, DevStats *st, const uint32_t *off,
                     const int32_t *bcol, int b, cudaStream_t s);
// pull_cc.cu — pull label-propagation step (dense CC supersteps)
void launch_pull_cc(const GraphView &g, int32_t *label, uint64_t *out_bits, uint64_t *out_summ, DevStats *st,
                    cudaStream_t s);

// scsr.cu — destination-segmented copy of the arcs + the sweep advance (BFS, diff mode)
struct ScsrStore {
    ScsrView v{};
    uint32_t *col = nullptr;
    uint32_t *base = nullptr;
    int64_t *start = nullptr;
    uint32_t *qc = nullptr;
    uint32_t nx = 0;        // vertices with a part >= 255 arcs (build statistics)
    size_t bytes = 0;
};
// sw: slice words (<= 16,384; out of range = default).  cudaErrorInvalidValue: a segment block
// would exceed 2^32 arcs or a row is not sorted (the caller keeps the word path).
cudaError_t scsr_build(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int32_t sw, ScsrStore *out,
                       cudaStream_t s);
void scsr_free(ScsrStore *S);
// visited |= every neighbour of the input frontier's active vertices (zeroes v.qc first); runs
// only if the frontier's m_f >= min_mf (0: always), so a CUDA graph can hold both push paths
void launch_push_sweep(const ScsrView &v, const int64_t *rp, const uint64_t *in_bits, const uint64_t *in_summ,
                       const uint32_t *offsets, int64_t nw2, DevStats *st, uint64_t *visited,
                       unsigned long long min_mf, cudaStream_t s);

// ablate.cu — word-width ablation (f3): push-only 2LB BFS with 32- or 64-bit words, host loop;
// returns 0 on success, the supersteps and the device time
int ablation_bfs_words(const GraphView &g, int32_t src, uint32_t *level, int word_bits, cudaStream_t s, int64_t *iters,
                       float *ms);
// ctrl.cu — device-side superstep control (CUDA-graph driven loops)
// level init + seed + the seed frontier's word list / statistics + first decision, one kernel
// single-GPU: the same with the frontier, visited / vis_old and control-block initialisation folded
// in, added to the graph as a kernel node whose argument block carries the run's control-block
// initialisation (`hot`: the leading BFS_CTRL_HOT_WORDS words of BfsCtrl)
constexpr int BFS_CTRL_HOT_WORDS = (int)((offsetof(BfsCtrl, t_ns) + 7) / 8);
struct BfsProArgs {
    BfsCtrl *c;
    int64_t n, nw1, nw2;
    const uint8_t *deg8;
    const uint64_t *isolated;
    uint64_t *bits, *summ;
    uint32_t *offsets;
    DevStats *st, *st_out;
    uint64_t *visited, *vis_old;
    unsigned long long hot[BFS_CTRL_HOT_WORDS];
};
void bfs_prologue1_node(BfsProArgs *a, void **arg_slot, cudaKernelNodeParams *kp);
void launch_bfs_prologue(BfsCtrl *c, int64_t n, const uint8_t *deg8, uint64_t *bits, uint64_t *summ,
                         uint32_t *offsets, DevStats *st, uint64_t *visited, uint64_t *vis_old, const Xchg &x,
                         cudaStream_t s);
void launch_clear_listed(uint64_t *bits, uint64_t *summ, const uint32_t *offsets, const DevStats *st, int64_t nw1,
                         int64_t nw2, DevStats *zero_st, cudaStream_t s);
void launch_zero_u64(unsigned long long *p, int64_t n, cudaStream_t s);
// partition (xchg.cuh): barrier across ranks (one thread); owned slice [lo, hi) of src into
// every rank's replica vals
void launch_xbarrier(const Xchg &x, cudaStream_t s);
void launch_publish_owned(const uint32_t *src, uint32_t *vals, int64_t lo, int64_t hi, const Xchg &x, cudaStream_t s);

// partition.cu — graph-load side of the 1-D destination partition
// h_out[r-1] = first vertex whose row starts at or after nnz*r/P (r = 1..P-1); synchronises s
cudaError_t part_quantiles(const int64_t *rp, int64_t n, int64_t nnz, int P, int64_t *h_out, cudaStream_t s);
// push block: the arcs of every row into [lo, hi) (CSR over all n rows; +64 B padding)
cudaError_t part_push_block(const int64_t *rp, const int32_t *col, const uint8_t *w, int64_t n, int64_t lo, int64_t hi,
                            int64_t **rpp, int32_t **colp, uint8_t **wp, int64_t *nnz, cudaStream_t s);
// transpose of a directed CSR (in-neighbours, rows sorted), for pull steps
cudaError_t build_csc(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int64_t **rpt, int32_t **colt,
                      cudaStream_t s);
// pull block: rows [lo, hi) (CSR over all n rows, rows outside empty)
cudaError_t part_pull_block(const int64_t *rp, const int32_t *col, int64_t n, int64_t lo, int64_t hi, int64_t **rpl,
                            int32_t **coll, int64_t *nnz, cudaStream_t s);
void launch_list_all(uint32_t *offsets, DevStats *st_all, const DevStats *st_src, int64_t nw1, cudaStream_t s);

// bcb.cu — source-batched BC (32 sources per batch): init, cooperative forward and backward
// kernels (grid-wide barriers between supersteps), reset
struct BcbLaunch {
    GraphView g;
    uint32_t *F, *V, *M;
    uint64_t *VB, *VS;
    double *s, *delta;
    int32_t *lv;
    uint32_t *lm;
    unsigned long long *loff, *maxb;
    BcbCtrl *c;
    int32_t cap;
    int64_t lcap;
    double *bc;
};
cudaError_t bcb_run_batch(const BcbLaunch &L, cudaStream_t s);

// bc.cu — Brandes helpers
void launch_bc_level_max(const double *sigma, const uint64_t *bits, const uint32_t *offsets, const DevStats *st,
                         int64_t max_words, unsigned long long *max_bits, cudaStream_t s);
void launch_bc_level_scale_and_stack(double *sigma, const uint64_t *bits, const uint32_t *offsets,
                                     const DevStats *st, int64_t max_words, const unsigned long long *max_bits,
                                     int32_t *exp_of_level, uint32_t level_idx, int32_t *stack,
                                     unsigned long long *stack_top, unsigned long long *underflow, cudaStream_t s);
void launch_bc_backward_level(const GraphView &g, const int32_t *stack, int64_t lo, int64_t hi, const uint32_t *level,
                              const double *sigma, double *delta, const int32_t *exp_of_level, uint32_t d,
                              double *bc, int32_t src, cudaStream_t s);

}  // namespace sg
