// bfsstep.cuh — end of a BFS superstep on the device, shared by k_bfs_diff (after push / sweep)
// and the pull step: block-aggregated emission of the output frontier's layer-2 words and word
// list, statistics, and the direction decision taken by the last CTA to finish (so a superstep
// is its advance kernels + one output kernel, no compaction / clear / decide launches).
#pragma once
#include "common.cuh"
#include "kernels.h"
#include "xchg.cuh"

namespace sg {

// m_f of a quad of 4 vertices: degree codes `codes` (4 bytes), vertices `mask` (4 bits), decoded
// through a 256-entry table in shared memory (filled by deg8_lut_init; 1 LDS per vertex instead
// of the ~10-op decode)
__device__ __forceinline__ void deg8_lut_init(uint32_t *lut) {
    for (int i = threadIdx.x; i < 256; i += blockDim.x) lut[i] = deg8_decode((uint32_t)i);
}
__device__ __forceinline__ unsigned long long quad_mf(const uint32_t *lut, uint32_t codes, uint32_t mask) {
    // common case: every selected vertex has degree < 32, whose code is the degree itself: one
    // byte mask (4 bits -> 4 bytes) and one dp4a (the table path was ~35 % of k_bfs_diff's
    // instructions, profiles/r02k)
    const uint32_t sel = codes & (((mask * 0x00204081u) & 0x01010101u) * 0xFFu);
    if ((sel & 0xE0E0E0E0u) == 0u) return (unsigned long long)__dp4a(sel, 0x01010101u, 0u);
    unsigned long long m = 0;
#pragma unroll
    for (int k = 0; k < 4; k++)
        if ((mask >> k) & 1u) m += lut[(codes >> (8 * k)) & 0xffu];
    return m;
}

__device__ __forceinline__ void bfs_set_cond(unsigned long long h, unsigned v) {
    if (h) cudaGraphSetConditional((cudaGraphConditionalHandle)h, v);
}

// Superstep kinds (decisions)
enum : uint32_t { SK_STOP = 0, SK_PUSH = 1, SK_PULL = 2, SK_SWEEP = 3, SK_SPARSE = 4 };

// Beamer direction policy (R2) + loop control, from the freshly built output frontier's
// control block `st`; `prev_arcs` = arcs inspected by the superstep just run (folded into the
// per-direction totals); `zero_prev` (nullable) = the control block of the frontier just advanced,
// zeroed here (it is the next superstep's output).  `next_in` = the buffer holding the next
// superstep's input: the IF nodes of that buffer's half get the decision, the other half's are
// switched off (the fused sparse loop may end on either parity; its half is then skipped and the
// WHILE loop comes back to the right one).  Returns the decision (SK_*).  One thread.
__device__ __forceinline__ uint32_t bfs_decide(BfsCtrl *c, const DevStats *st, unsigned long long prev_arcs,
                                               DevStats *zero_prev, int next_in, int first, bool defer_sparse = false,
                                               bool dead_end = false) {
    // control blocks were filled by atomics of other CTAs / kernels: volatile (L2) reads
    const volatile DevStats *vst = st;
    if (!first) {
        if (c->pull) c->arcs_pulled += prev_arcs;
        else c->arcs_pushed += prev_arcs;
    }
    const unsigned long long count = vst->count;
    bool go = count > 0;
    if (go) {
        if (!first) c->reached += vst->nf;
        // every vertex is visited (the reached ones + the never-reachable ones): expanding this
        // frontier cannot find a new vertex, so the BFS ends here instead of one empty superstep later
        if ((long long)c->reached + c->n_iso - c->src_iso >= c->n) go = false;
        if (dead_end) go = false;   // lookahead: no arc of this frontier leads to an unvisited vertex
    }
    if (go && c->iters >= (unsigned long long)c->max_iters) {
        c->overflow = 1;
        go = false;
    }
    if (go) {
        const long long nf = (long long)vst->nf, mf = (long long)vst->mf;
        c->mu -= mf;
        if (c->auto_dir) {
            if (!c->pull && nf > c->nf_prev && (double)mf > (double)c->mu / c->alpha) c->pull = 1;
            else if (c->pull && nf < c->nf_prev && (double)nf < (double)c->n / c->beta) c->pull = 0;
        }
        c->nf_prev = nf;
        c->next = first ? 1u : c->next + 1u;
        if (c->pull) c->pull_steps++;
        else c->push_steps++;
        c->iters++;
    }
    const bool push = go && !c->pull;
    const bool sweep = push && (c->sweep_mode == 2 || (c->sweep_mode == 1 && vst->mf >= c->sweep_thr));
    if (sweep) c->sweep_steps++;
    const bool sparse = push && !sweep && c->hsparse[next_in] && c->sparse_mode && count <= c->sparse_words &&
                        vst->mf <= c->sparse_arcs;
    if (sparse) c->sparse_steps++;
    {
        const unsigned long long i = c->tr_n++;
        if (i < (unsigned long long)SG_TRACE_STEPS) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
            c->t_ns[i] = t;
            c->kind[i] = !go ? SK_STOP : (c->pull ? SK_PULL : (sweep ? SK_SWEEP : (sparse ? SK_SPARSE : SK_PUSH)));
            c->tr_count[i] = count;
            c->tr_nf[i] = vst->nf;
            c->tr_mf[i] = vst->mf;
        }
    }
    // late pulls run warp-owned layer-2 words (pull.cu k_pull_bfs_w): few unvisited vertices left
    c->pull_warp[next_in] = c->pull_warp_frac &&
                   (unsigned long long)(c->n - c->n_iso - (long long)c->reached) * c->pull_warp_frac <
                       (unsigned long long)(c->n - c->n_iso);
    // handle values wanted: only the next input buffer's half has a taken IF; set the changed ones
    if (!(defer_sparse && sparse)) {   // (the fused sparse loop continues without touching them)
        const uint32_t kinds = (push && !sweep && !sparse ? 1u : 0u) | (go && c->pull ? 2u : 0u) |
                               (sweep ? 4u : 0u) | (sparse ? 8u : 0u);
        uint32_t want = go ? 0x100u : 0u;
        for (int k = 0; k < 4; k++)
            if ((kinds >> k) & 1u) want |= 1u << (2 * k + next_in);
        const uint32_t diff = want ^ c->hmask;
        const unsigned long long *hs[4] = {c->hpush, c->hpull, c->hsweep, c->hsparse};
        for (int k = 0; k < 4; k++)
            for (int b = 0; b < 2; b++)
                if ((diff >> (2 * k + b)) & 1u) bfs_set_cond(hs[k][b], (want >> (2 * k + b)) & 1u);
        if (diff & 0x100u) bfs_set_cond(c->hl, go);
        c->hmask = want;
    }
    if (zero_prev) *zero_prev = DevStats{};
    if (!go && c->res) {   // the run's counters to the host (mapped memory; read after the graph)
        volatile BfsResult *r = c->res;
        r->iters = c->iters;
        r->push_steps = c->push_steps;
        r->pull_steps = c->pull_steps;
        r->arcs_pushed = c->arcs_pushed;
        r->arcs_pulled = c->arcs_pulled;
        r->reached = c->reached;
        r->sweep_steps = c->sweep_steps;
        r->sparse_steps = c->sparse_steps;
        r->overflow = c->overflow;
        __threadfence_system();
        r->done = 1u;
    }
    return !go ? SK_STOP : (c->pull ? SK_PULL : (sweep ? SK_SWEEP : (sparse ? SK_SPARSE : SK_PUSH)));
}

// Decision of a graph-driven SSSP / CC superstep: stop on an empty frontier (or the cap), else
// the next superstep's direction (CC AUTO: pull when m_f > nnz/4, the host loop's rule); the IF
// handles of the next input buffer's half get it, only changed handles are set.  One thread.
__device__ __forceinline__ void val_decide(ValCtrl *c, const DevStats *st, unsigned long long prev_arcs,
                                           DevStats *zero_prev, int next_in, int first) {
    const volatile DevStats *vst = st;
    if (!first) {
        if (c->pull) c->arcs_pulled += prev_arcs;
        else c->arcs_pushed += prev_arcs;
    }
    const unsigned long long count = vst->count;
    bool go = count > 0;
    if (go && c->iters >= (unsigned long long)c->max_iters) {
        c->overflow = 1;
        go = false;
    }
    bool pull = false;
    if (go) {
        pull = c->cc && (c->direction == 2 || (c->direction == 0 && (double)vst->mf * 4.0 > (double)c->nnz));
        c->pull = pull;
        if (pull) c->pull_steps++;
        else c->push_steps++;
        c->iters++;
    }
    uint32_t want = go ? 0x100u : 0u;
    if (go) want |= 1u << (2 * (pull ? 1 : 0) + next_in);
    const uint32_t diff = want ^ c->hmask;
    const unsigned long long *hs[2] = {c->hpush, c->hpull};
    for (int k = 0; k < 2; k++)
        for (int b = 0; b < 2; b++)
            if ((diff >> (2 * k + b)) & 1u) bfs_set_cond(hs[k][b], (want >> (2 * k + b)) & 1u);
    if (diff & 0x100u) bfs_set_cond(c->hl, go);
    c->hmask = want;
    if (zero_prev) *zero_prev = DevStats{};
}

// Emit a block's slice of the output frontier: `S` = the block's layer-2 words (in shared
// memory, nS of them, the first = layer-2 word sw0; words at or past w2_hi are not this rank's
// and are skipped), written as is; their set bits are appended to the word list with one atomic
// per block (ascending within the block).  Partitioned: the same layer-2 words and list entries
// go to every peer's replica (one remote atomic per block and peer).  Call with the whole block;
// ends with __syncthreads.
template <bool P = true>
__device__ __forceinline__ void bfs_emit_words(const BfsOut &o, int64_t w2_hi, int64_t sw0, const uint64_t *S, int nS,
                                               uint32_t *s_base) {
    const Xchg &x = o.x;
    if ((int)threadIdx.x < nS && sw0 + threadIdx.x < w2_hi) xstore<P>(x, o.out_summ + sw0 + threadIdx.x, S[threadIdx.x]);
    if (threadIdx.x == 0) {
        uint32_t tot = 0;
        for (int i = 0; i < nS; i++) tot += (uint32_t)__popcll(S[i]);
        s_base[0] = tot ? (uint32_t)atomicAdd(&o.st->count, (unsigned long long)tot) : 0u;
        if (P && x.nranks > 1 && tot) {
            unsigned long long b[SG_MAX_RANKS];
#pragma unroll
            for (int j = 0; j < SG_MAX_RANKS; j++)   // all remote atomics in flight together
                b[j] = (j < x.nranks && j != x.rank) ? atomicAdd(&xpeer(x, o.st, j)->count, (unsigned long long)tot)
                                                       : 0ull;
#pragma unroll
            for (int j = 0; j < SG_MAX_RANKS; j++) s_base[1 + j] = (uint32_t)b[j];
        }
    }
    __syncthreads();
    for (int t = threadIdx.x; t < nS * 64; t += blockDim.x) {
        const int i = t >> 6, b = t & 63;
        const uint64_t xw = S[i];
        if ((xw >> b) & 1ull) {
            uint32_t pos = (uint32_t)__popcll(xw & ((1ull << b) - 1ull));
            for (int j = 0; j < i; j++) pos += (uint32_t)__popcll(S[j]);
            const uint32_t val = (uint32_t)((sw0 + i) * 64 + b);
            o.out_offsets[s_base[0] + pos] = val;
            if (P && x.nranks > 1) {
                for (int j = 0; j < x.nranks; j++)
                    if (j != x.rank) xpeer(x, o.out_offsets, j)[s_base[1 + j] + pos] = val;
            }
        }
    }
    __syncthreads();
}

// Dead-end lookahead (single GPU, the last CTA of a BFS output kernel, whole CTA): when the
// output frontier is tiny (<= 64 listed words, m_f <= 64) test its arcs against the final visited
// bitmap; if none leads to an unvisited vertex, the next superstep would produce an empty frontier,
// so the BFS ends now (st->pad2 = 1; bfs_decide) instead of one ~20 us superstep later - the last
// superstep of every config-4 BFS (2-22 leaves whose neighbours are all visited).  Five dependent
// loads (list, word, row bounds, arcs, visited) in one CTA.  Returns the verdict (CTA-uniform).
__device__ __forceinline__ bool bfs_lookahead(const BfsOut &o) {
    constexpr int LV = 64, LA = 256;
    __shared__ int64_t s_start[LV];
    __shared__ uint32_t s_pre[LV + 1];
    __shared__ int32_t s_v[LV];
    __shared__ uint32_t s_nv;
    __shared__ int s_dead;
    const volatile DevStats *vst = o.st;
    const unsigned long long count = vst->count, mf = vst->mf;
    if (!o.rp || count == 0 || count > (unsigned long long)LV || mf > (unsigned long long)LV) return false;
    if (threadIdx.x == 0) {
        s_nv = 0u;
        s_dead = 1;
    }
    __syncthreads();
    if (threadIdx.x < count) {
        const uint32_t w = o.out_offsets[threadIdx.x];
        for (uint64_t b = o.out_bits[w]; b; b &= b - 1) {
            const uint32_t i = atomicAdd(&s_nv, 1u);
            if (i < (uint32_t)LV) s_v[i] = (int32_t)(w * 64u + (uint32_t)(__ffsll((long long)b) - 1));
        }
    }
    __syncthreads();
    const uint32_t nv = s_nv;
    if (nv > (uint32_t)LV) return false;   // (uniform) cannot happen: every frontier vertex has an arc
    if (threadIdx.x < nv) {
        const int32_t v = s_v[threadIdx.x];
        const int64_t a = o.rp[v];
        s_start[threadIdx.x] = a;
        s_pre[threadIdx.x + 1] = (uint32_t)min(o.rp[v + 1] - a, (int64_t)LA + 1);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        s_pre[0] = 0u;
        for (uint32_t i = 0; i < nv; i++) s_pre[i + 1] += s_pre[i];
    }
    __syncthreads();
    const uint32_t total = s_pre[nv];
    if (total > (uint32_t)LA) return false;   // (uniform) degree codes under-estimated a row
    for (uint32_t t = threadIdx.x; t < total; t += blockDim.x) {
        uint32_t k = 0;
        while (s_pre[k + 1] <= t) k++;
        const int32_t u = o.col[s_start[k] + (t - s_pre[k])];
        if (!((o.visited[u >> 6] >> (u & 63)) & 1ull)) s_dead = 0;
    }
    __syncthreads();
    return s_dead != 0;
}

// End of the output kernel: block sums of n_f / m_f (and `arcs` into the input's control block),
// then the last CTA to finish takes the direction decision (graph mode).  Partitioned: the last
// CTA first runs the superstep barrier (xchg.cuh) and replaces st's n_f / m_f by the global sums;
// it zeroes the input's control block BEFORE publishing (peers add their word-list counts into it
// as soon as they pass this barrier: it is the next superstep's output).  Whole block.
template <bool P = true>
__device__ __forceinline__ void bfs_finish(const BfsOut &o, unsigned long long nf, unsigned long long mf,
                                           unsigned long long arcs, DevStats *in_st, unsigned long long scans = 0) {
    __shared__ unsigned long long s_r[4][32];
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const bool part = P && o.x.nranks > 1;
    nf = warp_sum(nf);
    mf = warp_sum(mf);
    arcs = warp_sum(arcs);
    scans = warp_sum(scans);
    if (lane == 0) {
        s_r[0][wid] = nf;
        s_r[1][wid] = mf;
        s_r[2][wid] = arcs;
        s_r[3][wid] = scans;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long a = 0, b = 0, c = 0, d = 0;
        for (int i = 0; i < (int)(blockDim.x >> 5); i++) {
            a += s_r[0][i];
            b += s_r[1][i];
            c += s_r[2][i];
            d += s_r[3][i];
        }
        if (d && in_st) atomicAdd(&in_st->scans, d);
        if (a) {
            atomicAdd(&o.st->nf, a);
            atomicAdd(&o.st->mf, b);
        }
        if (c && in_st) atomicAdd(&in_st->arcs, c);
        s_last = false;
        if (o.ctrl || o.vctrl || part || o.rp) {
            if (part) __threadfence_system();   // this CTA's peer stores before the barrier's epoch
            else __threadfence();
            s_last = atomicAdd(o.done, 1u) == gridDim.x - 1;
        }
    }
    __syncthreads();
    bool dead = false;
    if (s_last && !part && o.rp) {   // (uniform across the last CTA)
        __threadfence();
        dead = bfs_lookahead(o);
        if (dead && threadIdx.x == 0) o.st->pad2 = 1ull;   // the host loop reads the verdict here
    }
    if (s_last && threadIdx.x == 0) {
        if (part) __threadfence_system();
        else __threadfence();
        *o.done = 0u;
        DevStats *prev = o.prev ? o.prev : in_st;
        unsigned long long prev_arcs = prev ? reinterpret_cast<const volatile DevStats *>(prev)->arcs : 0ull;
        if (o.ctrl && prev) {   // retire the input buffer: the sparse kernel needs to know what it holds
            o.ctrl->saved_count[o.half] = reinterpret_cast<const volatile DevStats *>(prev)->count;
            o.ctrl->dirty[o.half] = o.sparse ? 0u : 1u;
        }
        if (part) {
            volatile DevStats *vst = o.st;
            const unsigned long long my_nf = vst->nf, my_mf = vst->mf;
            if (o.prev) *o.prev = DevStats{};   // zero before peers may add into it (next output)
            XSlot tot;
            xbarrier(o.x, my_nf, my_mf, prev_arcs, &tot);
            vst->nf = tot.nf;
            vst->mf = tot.mf;
            prev_arcs = tot.arcs;
            vst->pad = tot.arcs;   // host loops read the superstep's global arcs here
            if (o.ctrl) bfs_decide(o.ctrl, o.st, prev_arcs, nullptr, o.half ^ 1, 0);
        } else if (o.ctrl) {
            bfs_decide(o.ctrl, o.st, prev_arcs, o.prev, o.half ^ 1, 0, false, dead);
        } else if (o.vctrl) {
            val_decide(o.vctrl, o.st, prev_arcs, o.prev, o.half ^ 1, 0);
        }
    }
}

}  // namespace sg
