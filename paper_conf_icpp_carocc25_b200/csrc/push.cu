// push.cu — instantiations + launchers of the push advance for the four functors
// (§3.4: BFS, SSSP, CC, BC).  Design: push.cuh header comment, DESIGN.md §5.
#include "kernels.h"
#include "push.cuh"

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
    return p;
}

template <class F>
static void launch_push(const PushLaunch &L, const F &f, cudaStream_t s) {
    static bool attr_done = false;
    if (!attr_done) {
        cudaFuncSetAttribute(k_push_heavy<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)HEAVY_SMEM);
        attr_done = true;
    }
    const PushParams p = make_params(L);
    note_launch();
    k_push_words<F><<<L.grid_words, PUSH_THREADS, 0, s>>>(p, f);
    note_launch();
    k_push_heavy<F><<<L.grid_heavy, HEAVY_THREADS, HEAVY_SMEM, s>>>(p, f);
}

int push_max_grid_words() { return 148 * 4; }   // 64 regs x 256 threads: 4 CTAs per SM resident
int push_max_grid_heavy() { return 148 * 3; }

void launch_push_bfs(const PushLaunch &L, const BfsArgs &a, cudaStream_t s) {
    FnBfs f;
    f.visited = a.visited;
    f.level = a.level;
    f.next = a.next;
    f.next_ptr = a.next_ptr;
    f.out = OutSink{a.out_bits, a.out_summ};
    launch_push(L, f, s);
}
void launch_push_sssp(const PushLaunch &L, const SsspArgs &a, cudaStream_t s) {
    FnSssp f;
    f.dist = a.dist;
    f.out = OutSink{a.out_bits, a.out_summ};
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

}  // namespace sg
