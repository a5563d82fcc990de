// seg.cuh — destination-segmented hub tier of the BFS push advance.
//
// The per-arc visited probe of a push step is one random 8-B load into a 2 MB bitmap: one L1
// wavefront and one L2 sector per arc, which caps the top-down advance far below HBM bandwidth
// (ncu: profiles/r01_ncu_full_push_pull_level3.txt).  For hub rows (deg >= SEG_MIN) this tier
// instead walks the destination space in segments of SEG_V vertices: each CTA (one per SM,
// 192 KB of shared memory) copies the segment's visited slice into shared memory, streams the
// part of every queued hub chunk that falls in the segment (per-hub segment offsets computed at
// graph load; rows are sorted, so each part is contiguous), probes and marks bits in shared
// memory, then flushes: for each slice word, bits it set that are not yet set globally go to
// one global atomicOr; the CTA whose atomic flips a bit writes the level and the output
// frontier.  Same result set as the probe path (advance semantics PAPER.md:116/123; tested).
//
// Per warp, 32 chunk parts are packed into one arc list (prefix sum of their lengths) and
// streamed in 32-arc windows, 4 windows in flight per iteration: short parts (a mid hub has
// ~deg/11 arcs per segment) do not idle lanes.
#pragma once
#include "common.cuh"
#include "functors.cuh"
#include "push.cuh"

namespace sg {

constexpr int SEG_THREADS = 1024;
constexpr size_t SEG_SMEM = (size_t)SEG_WORDS * sizeof(uint64_t);
#ifndef SG_SEG_OWNER
#define SG_SEG_OWNER 1   // 1: a CTA owns one segment (one slice load / flush); 0: every CTA walks all
#endif
#ifndef SG_SEG_UNROLL
#define SG_SEG_UNROLL 8
#endif
#ifndef SG_SEG_LQ
#define SG_SEG_LQ 4   // long parts: int4 loads per lane in flight per iteration (2 / 4 / 8 measured: 4)
#endif
#ifndef SG_SEG_LONG
#define SG_SEG_LONG 192
#endif
#ifndef SG_SEG_CHECK
#define SG_SEG_CHECK 0   // 1: test the slice bit before the shared-memory atomic (0: atomic on every arc;
                         // measured faster: the level-2 hub pushes mark mostly fresh bits, so the test
                         // was an extra LDS per arc - 283 -> 264 us on a 133 M-arc level)
#endif
constexpr int SEG_UNROLL = SG_SEG_UNROLL;
// mark a destination in the shared-memory slice (32-bit ATOMS.OR is native; 64-bit is a CAS loop)
__device__ __forceinline__ void seg_mark(uint32_t *s_vis32, int i, uint32_t m) {
    if (!SG_SEG_CHECK || !(s_vis32[i] & m)) atomicOr(s_vis32 + i, m);
}
constexpr uint32_t SEG_LONG = SG_SEG_LONG;   // parts at least this long are streamed with int4 loads

__global__ void __launch_bounds__(SEG_THREADS, 1) k_push_seg(PushParams p, FnBfs f) {
    extern __shared__ __align__(16) uint64_t s_vis[];
    __shared__ __align__(8) uint64_t s_bar;   // slice load: cp.async.bulk completion
    __shared__ uint32_t s_next;                 // next item batch (dynamic deal to warps)
    const unsigned long long cnt = p.st->seg_count;
    const uint32_t nitems = (uint32_t)(cnt < p.seg_cap ? cnt : p.seg_cap);
    if (nitems == 0) return;
    const int nseg = p.g.nseg, S1 = nseg + 1;
#if SG_SEG_OWNER
    // each CTA owns one destination segment and a share of the items: the CTAs are dealt to the
    // segments in contiguous groups (gridDim.x >= nseg), so every slice is loaded and flushed by
    // its group only (gridDim.x slices in total instead of gridDim.x * nseg)
    const int G = (int)gridDim.x;
    const int b_own = (int)((int64_t)blockIdx.x * nseg / G);
    const int c_lo = (int)(((int64_t)b_own * G + nseg - 1) / nseg);       // first CTA of the group
    const int c_hi = (int)(((int64_t)(b_own + 1) * G + nseg - 1) / nseg);  // one past its last
    const uint32_t i0 = (uint32_t)((uint64_t)nitems * (blockIdx.x - c_lo) / (c_hi - c_lo));
    const uint32_t i1 = (uint32_t)((uint64_t)nitems * (blockIdx.x - c_lo + 1) / (c_hi - c_lo));
    if (i0 == i1) return;
#else
    const uint32_t i0 = (uint32_t)((uint64_t)nitems * blockIdx.x / gridDim.x);
    const uint32_t i1 = (uint32_t)((uint64_t)nitems * (blockIdx.x + 1) / gridDim.x);
    if (i0 == i1) return;
#endif
    const int warp = threadIdx.x >> 5, lane = lane_id();
    constexpr int NW = SEG_THREADS / 32;
    uint32_t bar_phase = 0u;
    bool bar_ready = false;
    uint32_t *level = f.level_pp ? *f.level_pp : f.level;
    const uint32_t next = f.next_ptr ? *f.next_ptr : f.next;
#if SG_SEG_OWNER
    for (int b = b_own; b == b_own; b++) {
#else
    for (int b = 0; b < nseg; b++) {
#endif
        const int64_t w0 = (int64_t)b * SEG_WORDS;
        const int nw = (int)min((int64_t)SEG_WORDS, p.g.nw1 - w0);
        // the slice (up to 192 KB) arrives by TMA bulk copies (one mbarrier, copies of <= 48 KB):
        // a thread-per-word copy loop was latency-bound (24 dependent load/store rounds per thread,
        // 28 % of the kernel's stall samples in ncu); visited carries 8 words of tail padding
        if (threadIdx.x == 0) {
            s_next = 0u;
            if (bar_phase == 0u && !bar_ready) {
                mbar_init(&s_bar, 1);
                asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
            }
            // the previous segment's shared-memory atomics (generic proxy) before the async copy
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            const uint32_t bytes = (uint32_t)((((int64_t)nw * 8) + 15) & ~15ll);
            mbar_expect_tx(&s_bar, bytes);
            constexpr uint32_t PIECE = 48 * 1024;
            for (uint32_t o = 0; o < bytes; o += PIECE)
                bulk_g2s(reinterpret_cast<char *>(s_vis) + o, reinterpret_cast<const char *>(f.visited + w0) + o,
                         min(PIECE, bytes - o), &s_bar);
        }
        bar_ready = true;
        __syncthreads();
        mbar_wait(&s_bar, bar_phase);
        bar_phase ^= 1u;
        const int32_t vbase = (int32_t)(w0 * 64);
        uint32_t *s_vis32 = reinterpret_cast<uint32_t *>(s_vis);   // 32-bit ATOMS.OR is native (64-bit is a CAS loop)
        // items are dealt to warps with stride NW: consecutive chunks of one hub (which fall into
        // the same segment) spread over all warps instead of piling onto one
        // batches (r, slot) = the items i0 + (r*32 + k)*NW + slot, k = lane (consecutive chunks of
        // one hub spread over batches), taken dynamically by the warps: part lengths vary 0..4096,
        // a static deal left warps idle at the flush barrier (ncu: barrier stalls 5.1)
        const uint32_t nbatch = ((i1 - i0 + 32 * NW - 1) / (32 * NW)) * NW;
        for (;;) {
            uint32_t q = 0;
            if (lane == 0) q = atomicAdd(&s_next, 1u);
            q = __shfl_sync(0xffffffffu, q, 0);
            if (q >= nbatch) break;
            const uint32_t r = q / NW, slot = q % NW;
            if (i0 + r * 32 * NW + slot >= i1) continue;
            // lane k: the part of item i0 + (r*32 + k)*NW + slot inside segment b
            const uint32_t item = i0 + (r * 32 + lane) * NW + slot;
            int64_t lo = 0;
            uint32_t len = 0;
            if (item < i1) {
                const SegItem x = p.seg[item];
                const uint32_t *off = p.g.hub_off + (size_t)x.h * S1;
                int64_t a = x.row + __ldg(off + b), e = x.row + __ldg(off + b + 1);
                a = max(a, x.begin);
                e = min(e, x.begin + (int64_t)x.len);
                if (e > a) {
                    lo = a;
                    len = (uint32_t)(e - a);
                }
            }
            // long parts: the whole warp streams each with 16-B loads (no per-arc owner search).
            // Each lane first handles the ragged head / tail (< 4 arcs each) of its own part; the
            // aligned bodies are then walked as one sequence of 128*LQ-arc windows over the
            // warp's long parts, the next window's loads issued before the current one's
            // shared-memory updates (software pipelining across windows and parts).
            const bool is_long = len >= SEG_LONG;
            const uint32_t longm = __ballot_sync(0xffffffffu, is_long);
            int64_t la = 0, lb = 0;
            if (is_long) {
                const int64_t e = lo + len;
                la = (lo + 3) & ~3ll;
                lb = la + ((e - la) & ~3ll);
                for (int64_t i = lo; i < la; i++) {
                    const int32_t vv = __ldg(p.g.col + i) - vbase;
                    const uint32_t m = 1u << (vv & 31);
                    seg_mark(s_vis32, vv >> 5, m);
                }
                for (int64_t i = lb; i < e; i++) {
                    const int32_t vv = __ldg(p.g.col + i) - vbase;
                    const uint32_t m = 1u << (vv & 31);
                    seg_mark(s_vis32, vv >> 5, m);
                }
            }
            if (longm) {
                constexpr int64_t WIN = 128 * SG_SEG_LQ;
                auto load_win = [&](int4 (&q)[SG_SEG_LQ], int64_t i, int64_t pb) {
#pragma unroll
                    for (int u = 0; u < SG_SEG_LQ; u++) {
                        const int64_t iu = i + 4 * lane + 128 * u;
                        q[u] = iu < pb ? __ldg(reinterpret_cast<const int4 *>(p.g.col + iu))
                                       : make_int4(vbase - 1, vbase - 1, vbase - 1, vbase - 1);
                    }
                };
                int src = __ffs(longm) - 1;
                int64_t i = __shfl_sync(0xffffffffu, la, src), pb = __shfl_sync(0xffffffffu, lb, src);
                int4 cur[SG_SEG_LQ];
                load_win(cur, i, pb);
                while (src >= 0) {
                    int nsrc = src;
                    int64_t ni = i + WIN, npb = pb;
                    if (ni >= pb) {   // next part in the mask
                        const uint32_t rest = longm & ~((2u << src) - 1u);
                        nsrc = rest ? __ffs(rest) - 1 : -1;
                        if (nsrc >= 0) {
                            ni = __shfl_sync(0xffffffffu, la, nsrc);
                            npb = __shfl_sync(0xffffffffu, lb, nsrc);
                        }
                    }
                    int4 nxt[SG_SEG_LQ];
                    if (nsrc >= 0) load_win(nxt, ni, npb);
#pragma unroll
                    for (int u = 0; u < SG_SEG_LQ; u++) {
                        const int32_t vv[4] = {cur[u].x - vbase, cur[u].y - vbase, cur[u].z - vbase, cur[u].w - vbase};
#pragma unroll
                        for (int k = 0; k < 4; k++) {
                            if (vv[k] < 0) continue;
                            const uint32_t m = 1u << (vv[k] & 31);
                            seg_mark(s_vis32, vv[k] >> 5, m);
                        }
                    }
                    if (nsrc < 0) break;
#pragma unroll
                    for (int u = 0; u < SG_SEG_LQ; u++) cur[u] = nxt[u];
                    src = nsrc;
                    i = ni;
                    pb = npb;
                }
            }
            if (len >= SEG_LONG) len = 0;
            // short parts: packed into one arc list, 32-arc windows
            const uint32_t incl = warp_inclusive_scan(len);
            const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
            const uint32_t pre = incl - len;
            for (uint32_t win = 0; win < total; win += 32 * SEG_UNROLL) {
                int32_t v[SEG_UNROLL];
#pragma unroll
                for (int j = 0; j < SEG_UNROLL; j++) {
                    // owner of arc t = the last lane whose part starts at or before t (pre is
                    // sorted over lanes; an empty lane is never the last such lane): 5-step
                    // binary search with shuffles
                    const uint32_t t = win + 32 * j + lane;
                    int own = 0;
#pragma unroll
                    for (int step = 16; step > 0; step >>= 1) {
                        const uint32_t pc = __shfl_sync(0xffffffffu, pre, own + step);
                        if (pc <= t) own += step;
                    }
                    const int64_t lo_k = __shfl_sync(0xffffffffu, lo, own);
                    const uint32_t pre_k = __shfl_sync(0xffffffffu, pre, own);
                    v[j] = (t < total) ? __ldg(p.g.col + lo_k + (t - pre_k)) - vbase : -1;
                }
#pragma unroll
                for (int j = 0; j < SEG_UNROLL; j++) {
                    if (v[j] < 0) continue;
                    const uint32_t m = 1u << (v[j] & 31);
                    seg_mark(s_vis32, v[j] >> 5, m);
                }
            }
        }
        __syncthreads();
        // flush: bits this CTA set that are not set globally yet -> one atomicOr per word
        for (int i = threadIdx.x; i < nw; i += SEG_THREADS) {
            const int64_t w = w0 + i;
            const uint64_t nb = s_vis[i] & ~f.visited[w];
            if (!nb) continue;
            if (f.diff) {   // k_bfs_diff builds the output
                atomic_or_u64(f.visited + w, nb);
                continue;
            }
            const uint64_t old = atomic_or_u64(f.visited + w, nb);
            const uint64_t flips = nb & ~old;
            if (!flips) continue;
            if (f.out.bits) {
                const uint64_t oo = atomic_or_u64(f.out.bits + w, flips);
                if (oo == 0ull) atomic_or_u64(f.out.summ + (w >> 6), 1ull << (w & 63));
            }
            uint64_t y = flips;
            while (y) {
                const int j = __ffsll((long long)y) - 1;
                y &= y - 1;
                level[w * 64 + j] = next;
            }
        }
        __syncthreads();
    }
}

}  // namespace sg
