// xchg.cuh — the exchange step of the 1-D destination partition, fused into the kernels that
// produce a superstep's output (§6 "static graph partitioning
// ... each GPU handles a local subgraph").
//
// Rank r owns destinations [lo_r, hi_r) (4,096-aligned: whole layer-1 and layer-2 words).  The
// output kernel of a superstep computes r's owned slice of the next frontier and, as it writes
// each owned word / layer-2 word / word-list entry / changed value locally, stores the same value
// into every peer's replica through peer memory (CUDA IPC mappings: NVLink P2P stores across
// GPUs, plain stores when two ranks share a GPU).  No NCCL call and no host round trip: the
// all-gather of the owned slices is the output kernel's own epilogue, overlapped with its compute
// tile by tile.  Its last CTA then runs the superstep barrier: it publishes this rank's n_f / m_f /
// arcs into every peer's control block (release, system scope), waits until every peer's
// contribution of the same epoch has arrived (acquire), and replaces the local partial
// statistics by the global sums, so every rank takes the same direction / termination decision.
#pragma once
#include "common.cuh"

namespace sg {

template <class T>
__device__ __forceinline__ T *xpeer(const Xchg &x, T *p, int j) {
    return reinterpret_cast<T *>(reinterpret_cast<char *>(p) + x.delta[j]);
}

// store v at p locally and in every peer replica (P = false: single-GPU instantiation, local only)
template <bool P = true, class T, class V>
__device__ __forceinline__ void xstore(const Xchg &x, T *p, V vv) {
    const T v = (T)vv;
    *p = v;
    if (P && x.nranks > 1) {
#pragma unroll
        for (int j = 0; j < SG_MAX_RANKS; j++)
            if (j < x.nranks && j != x.rank) *xpeer(x, p, j) = v;
    }
}

__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

#ifndef SG_XBARRIER_TIMEOUT_S
#define SG_XBARRIER_TIMEOUT_S 60
#endif

// Superstep barrier across ranks (one thread).  Publishes (nf, mf, arcs) and returns the sums
// over all ranks in *sum.  All of this rank's earlier global / peer stores (of every CTA that ran
// __threadfence_system() before the caller learnt it was last) are visible to a peer once it sees
// this rank's epoch.  A peer that does not arrive within SG_XBARRIER_TIMEOUT_S seconds sets
// ctl->error (the host turns it into SG_ERR_NCCL) instead of hanging the GPU.
__device__ __forceinline__ void xbarrier(const Xchg &x, unsigned long long nf, unsigned long long mf,
                                         unsigned long long arcs, XSlot *sum) {
    XCtl *c = x.ctl;
    const unsigned long long e = c->epoch + 1;
    c->epoch = e;
    const int par = (int)(e & 1ull);
    __threadfence_system();
    for (int j = 0; j < x.nranks; j++) {
        XSlot *s = xpeer(x, &c->slots[par][x.rank], j);
        s->nf = nf;
        s->mf = mf;
        s->arcs = arcs;
    }
    __threadfence_system();
    for (int j = 0; j < x.nranks; j++) st_release_sys(&xpeer(x, &c->slots[par][x.rank], j)->epoch, e);
    XSlot t{e, 0ull, 0ull, 0ull};
    const unsigned long long t0 = global_ns();
    for (int j = 0; j < x.nranks; j++) {
        XSlot *s = &c->slots[par][j];
        while (ld_acquire_sys(&s->epoch) < e) {
            if (global_ns() - t0 > (unsigned long long)SG_XBARRIER_TIMEOUT_S * 1000000000ull) {
                c->error = 1ull;
                break;
            }
            __nanosleep(200);
        }
        const volatile XSlot *vs = s;
        t.nf += vs->nf;
        t.mf += vs->mf;
        t.arcs += vs->arcs;
    }
    __threadfence_system();
    if (sum) *sum = t;
}

}  // namespace sg
