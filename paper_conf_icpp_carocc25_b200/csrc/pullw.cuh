// pullw.cuh — the warp-owned layer-2 word of the pull step (included by pull.cu) (§3.4 "possible to
// use both push and pull techniques as per Beamer et al. [5]").
//
// Same result as pull.cu (every unvisited vertex with a neighbour in the input frontier enters
// the output, level[v] = next; symmetric CSR: N(v) = in-neighbours, reading C8), redesigned after
// the round-1 profile of k_pull_bfs (profiles/r01g_ncu_full.txt: barrier stalls 22.4 on late
// pulls, long sequential list scans on early ones):
//   * one WARP owns one layer-2 word (64 layer-1 words, 4,096 vertices) end to end: its 64
//     visited words (2 per lane), the candidate tests, the output words, the layer-2 word and its
//     word-list entries — no CTA barrier anywhere in the loop;
//   * dense layer-2 words: 32 quad rounds (lanes 0-15 / 16-31 = the 16 quads of two layer-1
//     words), one 16-B candidate load (fnbr) and 4 bit probes per lane; sparse ones (<= 16
//     unvisited per word): word mode, a lane per layer-1 word walking its unvisited vertices;
//   * a vertex whose candidate misses is not scanned by its lane (a lane scanning a 90-arc row
//     stalls its warp for 45 dependent rounds) but queued in shared memory; the warp drains the
//     queue cooperatively: first every queued vertex on its own lane for up to PULL2_SHORT arcs
//     (most hits come early), then each still-open row by the whole warp, 32 arcs per round;
//   * found bits gather in a per-warp copy of the 64 output words (shared memory), written out
//     once with the visited / vis_old updates, the layer-2 word and one list append per warp.
// Level stores: candidate hits strided over the half-warp (64-B runs), queue hits scattered.
#pragma once
#include "common.cuh"
#include "kernels.h"
#include "bfsstep.cuh"
#include "xchg.cuh"

namespace sg {

constexpr int P2_THREADS = 256;
constexpr int P2_WARPS = P2_THREADS / 32;
constexpr int P2_QCAP = 256;     // queued vertices per warp (a quad round adds <= 128)
#ifndef SG_PULL2_SHORT
#define SG_PULL2_SHORT 8         // arcs a queued vertex scans on its own lane before the warp takes it
#endif
#ifndef SG_PULL2_WORD_MAX
#define SG_PULL2_WORD_MAX 16     // word mode when no layer-1 word has more unvisited vertices
#endif

struct P2Warp {
    uint64_t found[64];          // new bits of the layer-2 word's 64 layer-1 words
    int32_t q[P2_QCAP];          // queued vertices (candidate missed)
    int32_t q2[32];              // rows still open after the lane stage
};

__device__ __forceinline__ bool bit_in(const uint32_t *__restrict__ in32, int32_t u) {
    return (__ldg(in32 + (u >> 5)) >> (u & 31)) & 1u;
}

// Drain the warp's queue (n entries, warp-uniform): found vertices -> found bits, level, n_f / m_f.
__device__ __forceinline__ void p2_drain(const GraphView &g, const uint32_t *__restrict__ in32, P2Warp &W, int n,
                                         uint32_t *lvl, uint32_t nx, const uint32_t *lut, unsigned long long &nf,
                                         unsigned long long &mf, unsigned long long &arcs) {
    const int lane = lane_id();
    int n2 = 0;
    // stage A: one queued vertex per lane, up to SG_PULL2_SHORT arcs, 2 in flight
    for (int base = 0; base < n; base += 32) {
        const int i = base + lane;
        bool open = false;
        int32_t v = -1;
        if (i < n) {
            v = W.q[i];
            int64_t r = __ldg(g.rp + v);
            const int64_t e = __ldg(g.rp + v + 1);
            const int64_t ea = min(e, r + SG_PULL2_SHORT);
            bool hit = false;
            while (r < ea && !hit) {
                const int32_t u0 = __ldg(g.col + r);
                const int32_t u1 = r + 1 < ea ? __ldg(g.col + r + 1) : -1;
                const bool h0 = bit_in(in32, u0);
                const bool h1 = u1 >= 0 && bit_in(in32, u1);
                arcs += u1 >= 0 && !h0 ? 2 : 1;
                hit = h0 || h1;
                r += 2;
            }
            if (hit) {
                atomicOr(reinterpret_cast<unsigned long long *>(&W.found[(v >> 6) & 63]), 1ull << (v & 63));
                lvl[v] = nx;
                nf++;
                mf += lut[__ldg(g.deg8 + v)];
            } else {
                open = ea < e;
            }
        }
        const uint32_t ob = __ballot_sync(0xffffffffu, open);
        if (open) W.q2[n2 + __popc(ob & ((1u << lane) - 1u))] = v;
        n2 += __popc(ob);
        __syncwarp();
        // stage B: the open rows, the whole warp per row, 32 arcs per round from arc SHORT on
        for (int j = 0; j < n2; j++) {
            const int32_t w = W.q2[j];
            const int64_t s = __ldg(g.rp + w) + SG_PULL2_SHORT, e = __ldg(g.rp + w + 1);
            bool hit = false;
            for (int64_t r = s; r < e && !hit; r += 32) {
                const int64_t k = r + lane;
                const bool h = k < e && bit_in(in32, __ldg(g.col + k));
                const uint32_t hb = __ballot_sync(0xffffffffu, h);
                arcs += (lane == 0) ? (uint64_t)(hb ? __ffs(hb) : min((int64_t)32, e - r)) : 0ull;
                hit = hb != 0u;
            }
            if (hit && lane == 0) {
                W.found[(w >> 6) & 63] |= 1ull << (w & 63);
                lvl[w] = nx;
                nf++;
                mf += lut[__ldg(g.deg8 + w)];
            }
        }
        n2 = 0;
        __syncwarp();
    }
}

// One layer-2 word `sw` on one warp (visited words, candidates, queue drain, output words, layer-2
// word, list append).  Warp-synchronous; no CTA barrier.
template <bool P>
__device__ __forceinline__ void pull_l2_warp(const GraphView &g, int64_t sw, const uint32_t *__restrict__ in32,
                                             uint64_t *__restrict__ visited, const BfsOut &o, P2Warp &W,
                                             const uint32_t *s_lut, uint32_t *lvl, uint32_t nx, unsigned long long &nf,
                                             unsigned long long &mf, unsigned long long &arcs,
                                             unsigned long long &scans) {
    const int lane = lane_id();
    // ---- the layer-2 word's 64 visited words: lane owns wa = 64 sw + lane and wb = wa + 32 ----
    const int64_t wa = sw * 64 + lane, wb = wa + 32;
    auto valid = [&](int64_t w) -> uint64_t {
        if (w >= g.nw1) return 0ull;
        const int64_t rem = g.n - w * 64;
        return rem >= 64 ? ~0ull : ((1ull << rem) - 1ull);
    };
    const uint64_t va = wa < g.nw1 ? visited[wa] : ~0ull, vb = wb < g.nw1 ? visited[wb] : ~0ull;
    const uint64_t ua = ~va & valid(wa), ub = ~vb & valid(wb);
    const uint32_t fa = __ballot_sync(0xffffffffu, ua == 0ull), fb = __ballot_sync(0xffffffffu, ub == 0ull);
    if ((fa & fb) == 0xffffffffu) {   // no unvisited vertex: 64 zero output words
        if (wa < g.nw1) xstore<P>(o.x, o.out_bits + wa, 0ull);
        if (wb < g.nw1) xstore<P>(o.x, o.out_bits + wb, 0ull);
        if (lane == 0) xstore<P>(o.x, o.out_summ + sw, 0ull);
        return;
    }
    W.found[lane] = 0ull;
    W.found[lane + 32] = 0ull;
    const uint32_t mx = __reduce_max_sync(0xffffffffu, (uint32_t)max(__popcll(ua), __popcll(ub)));
    int nq = 0;   // warp-uniform queue length
    if (mx <= SG_PULL2_WORD_MAX) {
        // ---- word mode: lane walks the unvisited vertices of wa, then of wb, 4 tests in flight ----
#pragma unroll 1
        for (int h = 0; h < 2; h++) {
            const int64_t w = h ? wb : wa;
            uint64_t m = h ? ub : ua;
            uint64_t nb = 0;
            while (__any_sync(0xffffffffu, m != 0ull)) {
                int b[4];
                int32_t c[4];
                uint32_t x[4];
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    b[k] = m ? __ffsll((long long)m) - 1 : -1;
                    m &= m - 1;
                }
#pragma unroll
                for (int k = 0; k < 4; k++) c[k] = b[k] >= 0 ? __ldg(g.fnbr + w * 64 + b[k]) : -1;
#pragma unroll
                for (int k = 0; k < 4; k++) x[k] = c[k] >= 0 ? __ldg(in32 + (c[k] >> 5)) : 0u;
                uint32_t miss = 0;
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (b[k] < 0) continue;
                    bool hit = false;
                    if (c[k] >= 0) {
                        arcs++;
                        hit = (x[k] >> (c[k] & 31)) & 1u;
                    }
                    if (hit) nb |= 1ull << b[k];
                    else miss |= 1u << k;   // candidate missed (or none): the queue scans the row
                }
                // queue the misses (a vertex whose candidate missed, or that has none)
                const int cnt = __popc(miss);
                const int incl = warp_inclusive_scan(cnt);
                const int tot = __shfl_sync(0xffffffffu, incl, 31);
                if (nq + tot > P2_QCAP) {   // (cannot happen in word mode: <= 128 per pass) drain first
                    p2_drain(g, in32, W, nq, lvl, nx, s_lut, nf, mf, arcs);
                    nq = 0;
                }
                int pos = nq + incl - cnt;
#pragma unroll
                for (int k = 0; k < 4; k++)
                    if ((miss >> k) & 1u) W.q[pos++] = (int32_t)(w * 64 + b[k]);
                scans += (unsigned)cnt;
                nq += tot;
                __syncwarp();
            }
            if (nb) {
                const int64_t v0 = w * 64;
                nf += __popcll(nb);
                for (uint64_t t = nb; t; t &= t - 1) {
                    const int b0 = __ffsll((long long)t) - 1;
                    lvl[v0 + b0] = nx;
                    mf += s_lut[__ldg(g.deg8 + v0 + b0)];
                }
            }
            // (w & 63) = lane or lane + 32: this lane's own word; OR, because a mid-loop drain may
            // already have set bits of it (drains run warp-synchronously, never concurrently)
            W.found[(w & 63)] |= nb;
        }
        __syncwarp();
    } else {
        // ---- quad mode: round r covers layer-1 words 2r (lanes 0-15) and 2r+1 (lanes 16-31) ----
        const int hw = lane >> 4, q = lane & 15, sh = q * 4;
        const uint32_t half = hw ? 0xffff0000u : 0x0000ffffu;
#pragma unroll 1
        for (int r = 0; r < 32; r++) {
            const int wi = 2 * r + hw;                         // layer-1 word within the layer-2 word
            const uint32_t full2 = (r < 16) ? (fa >> (2 * r)) & 3u : (fb >> (2 * (r - 16))) & 3u;
            if (full2 == 3u) continue;                          // both words fully visited
            const uint64_t vis = __shfl_sync(0xffffffffu, wi < 32 ? va : vb, wi & 31);
            const int64_t w = sw * 64 + wi;
            const int64_t v0 = w * 64 + sh;
            const uint64_t vmask = valid(w);
            const uint32_t unv = (uint32_t)((~vis & vmask) >> sh) & 0xfu;
            uint32_t found = 0, codes = 0, miss = 0;
            if (unv) {
                const int4 c4 = __ldg(reinterpret_cast<const int4 *>(g.fnbr + v0));
                codes = __ldg(reinterpret_cast<const uint32_t *>(g.deg8 + v0));
                const int32_t c[4] = {c4.x, c4.y, c4.z, c4.w};
                uint32_t x[4];
#pragma unroll
                for (int k = 0; k < 4; k++) x[k] = ((unv >> k) & 1u) && c[k] >= 0 ? __ldg(in32 + (c[k] >> 5)) : 0u;
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (!((unv >> k) & 1u)) continue;
                    if (c[k] >= 0) {
                        arcs++;
                        if ((x[k] >> (c[k] & 31)) & 1u) {
                            found |= 1u << k;
                            continue;
                        }
                    }
                    miss |= 1u << k;
                }
            }
            const uint64_t mine = (uint64_t)found << sh;
            const uint64_t nb = (uint64_t)__reduce_or_sync(half, (uint32_t)mine) |
                                ((uint64_t)__reduce_or_sync(half, (uint32_t)(mine >> 32)) << 32);
            if (found) {
                nf += __popc(found);
                mf += quad_mf(s_lut, codes, found);
            }
            if (nb) {   // level stores strided over the half-warp (64-B runs)
                const uint64_t t = nb >> q;
                uint32_t *lw = lvl + w * 64 + q;
#pragma unroll
                for (int i = 0; i < 4; i++)
                    if ((t >> (16 * i)) & 1u) lw[16 * i] = nx;
            }
            if (q == 0) W.found[wi] = nb;
            // queue the misses
            const int cnt = __popc(miss);
            const int incl = warp_inclusive_scan(cnt);
            const int tot = __shfl_sync(0xffffffffu, incl, 31);
            if (tot) {
                if (nq + tot > P2_QCAP) {
                    __syncwarp();
                    p2_drain(g, in32, W, nq, lvl, nx, s_lut, nf, mf, arcs);
                    nq = 0;
                }
                int pos = nq + incl - cnt;
#pragma unroll
                for (int k = 0; k < 4; k++)
                    if ((miss >> k) & 1u) W.q[pos++] = (int32_t)(v0 + k);
                scans += (unsigned)cnt;
                nq += tot;
            }
            __syncwarp();
        }
    }
    if (nq) p2_drain(g, in32, W, nq, lvl, nx, s_lut, nf, mf, arcs);
    __syncwarp();
    // ---- output: 64 words, visited / vis_old, layer-2 word, list entries ----
    const uint64_t na = W.found[lane], nbw = W.found[lane + 32];
    if (wa < g.nw1) {
        xstore<P>(o.x, o.out_bits + wa, na);
        if (na) {
            visited[wa] = va | na;
            o.vis_old[wa] = va | na;
        }
    }
    if (wb < g.nw1) {
        xstore<P>(o.x, o.out_bits + wb, nbw);
        if (nbw) {
            visited[wb] = vb | nbw;
            o.vis_old[wb] = vb | nbw;
        }
    }
    const uint64_t S = (uint64_t)__ballot_sync(0xffffffffu, na != 0ull) |
                       ((uint64_t)__ballot_sync(0xffffffffu, nbw != 0ull) << 32);
    const int tot = __popcll(S);
    unsigned long long base[SG_MAX_RANKS + 1] = {};
    if (lane == 0) {
        xstore<P>(o.x, o.out_summ + sw, S);
        if (tot) {
            base[0] = atomicAdd(&o.st->count, (unsigned long long)tot);
            if (P)
                for (int j = 0; j < o.x.nranks; j++)
                    if (j != o.x.rank) base[1 + j] = atomicAdd(&xpeer(o.x, o.st, j)->count, (unsigned long long)tot);
        }
    }
    if (tot) {
        const uint32_t pa = (uint32_t)__popcll(S & ((1ull << lane) - 1ull));
        const uint32_t pb = (uint32_t)__popcll(S & ((1ull << (lane + 32)) - 1ull));
        const unsigned long long b0 = __shfl_sync(0xffffffffu, base[0], 0);
        if (na) o.out_offsets[b0 + pa] = (uint32_t)wa;
        if (nbw) o.out_offsets[b0 + pb] = (uint32_t)wb;
        for (int j = 0; P && j < o.x.nranks; j++) {
            if (j == o.x.rank) continue;
            const unsigned long long bj = __shfl_sync(0xffffffffu, base[1 + j], 0);
            if (na) xpeer(o.x, o.out_offsets, j)[bj + pa] = (uint32_t)wa;
            if (nbw) xpeer(o.x, o.out_offsets, j)[bj + pb] = (uint32_t)wb;
        }
    }
    __syncwarp();
}

}  // namespace sg
