// scsr.cu — destination-segmented sweep: the push advance of dense BFS supersteps (PAPER.md:116/123
// Table 2 advance::frontier with the BFS functor of Listing 1; 2LB input frontier P:249-262).
//
// Why: a top-down step probes the visited bitmap once per arc, a random 8-B access into a 2 MB
// array that lives in L2.  On the heavy Kronecker level (~0.95 G arcs) those probes and the
// atomics that follow them are bound by the L2 slices' request rate, not by HBM
// (profiles/r01b_launches_push.csv: the push-only level 3 takes ~3.1 ms for ~3.8 GB of col_idx).
//
// What: at the first BFS on a graph, a second copy of the arcs is built in destination-segment-
// major order (the "SCSR"): the vertex range is cut into segments of sv = 64*sw <= 2^20 vertices
// whose visited slice (sw 64-bit words, <= 128 KB) fits in shared memory next to a copy ring, and
// segment b's block holds, for u = 0..n-1 in order, the arcs of u into segment b.  Since rows are
// sorted each row splits into one contiguous part per segment.  An arc is stored as one u32:
// (u mod 4096) << 20 | (v - b*sv), the source relative to its *unit* (64 layer-1 words = one
// layer-2 summary bit... word) and the destination relative to its segment.  Index: per (segment,
// word) the block offset of the word's first arc (u32 `base`); a unit's arcs in a segment are the
// contiguous range base[b][64k] .. base[b][64k+64].
//
// The advance (k_push_sweep), for supersteps whose frontier holds a large share of the arcs:
// one 1,024-thread CTA per SM, warp 0 producing, warps 1..31 consuming.  Work items = (segment,
// group of units); a CTA starts on a home segment and steals items from the next segments when
// its own run dry.  The producer skips units whose layer-2 summary word is zero (no active
// vertex) and streams the others' arc ranges into a SW_STAGES-deep shared-memory ring with
// cp.async.bulk (TMA bulk copies, mbarrier complete_tx).  Consumers test each arc's source in
// the input frontier's layer 1 (its word is shared by the arc's neighbours: L1 broadcast) and
// probe / set the destination's bit in the shared-memory visited slice (ATOMS.OR only for unset
// bits).  On a segment switch the consumers OR the bits they set that are not yet global into
// `visited` (one RED per changed word) and load the next slice.  Diff mode: k_bfs_diff then
// derives the output frontier, levels and statistics from visited & ~vis_old, exactly as after
// the word-path push — the same result set (tested bit-exact against it and the oracle).
#include <vector>
#include "common.cuh"
#include "kernels.h"

namespace sg {

#ifndef SG_SW_CWARPS
#define SG_SW_CWARPS 30
#endif
#ifndef SG_SW_QPT
#define SG_SW_QPT 2
#endif
#ifndef SG_SW_STAGES
#define SG_SW_STAGES 3
#endif
constexpr int SW_CONSUMERS = SG_SW_CWARPS * 32;  // consumer threads (warps 2 .. 2 + SG_SW_CWARPS)
constexpr int SW_THREADS = SW_CONSUMERS + 64;    // + warp 0 = copy producer, warp 1 = work scheduler
constexpr int SW_TASKS = 64;                     // scheduler -> producer queue of active (segment, unit) ranges
constexpr int SW_QPT = SG_SW_QPT;                // 16-B quads per consumer thread per slot
constexpr int SW_QUADS = SW_CONSUMERS * SW_QPT;  // quads per ring slot
constexpr int SW_ACT_BYTES = 512;                // the unit's 64 input-frontier words, copied with the arcs
constexpr int SW_SLOT_BYTES = SW_ACT_BYTES + SW_QUADS * 16;

#ifndef SG_SW_NOPROBE
#define SG_SW_NOPROBE 1   // 1: OR every active arc's bit without probing it first (measured faster: ATOMS beat LDS + branch)
#endif
#ifndef SG_SW_UNITS
#define SG_SW_UNITS 16
#endif
constexpr int SW_STAGES = SG_SW_STAGES;          // ring depth
constexpr int SW_UNITS = SG_SW_UNITS;            // units (64 layer-1 words each) per work item
constexpr int SCSR_UNIT_SHIFT = 12;              // a unit = 4096 source vertices = one summary word
constexpr int SCSR_DST_BITS = 20;                // segment-relative destination id bits
constexpr int SCSR_MAX_SW = 1 << (SCSR_DST_BITS - 6);   // 16,384 words = 128 KB slice

// ---------------------------------------------------------------------------------------
// build (graph side; runs once per graph, not on the timed path)

// Part lengths of every vertex: cnt[b][u] (saturated at 255), word sums wsum[b][w], and the
// list of vertices with a part >= 255 arcs (escapes).  Rows are sorted: short rows are walked,
// long rows find each segment boundary by binary search.
__global__ void k_scsr_count(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n, int64_t npad,
                             int64_t nw1, int nseg, int64_t sv, uint8_t *__restrict__ cnt,
                             unsigned long long *__restrict__ wsum, int32_t *__restrict__ xidx,
                             int32_t *__restrict__ xvert, unsigned int *nx) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += stride) {
        const int64_t r0 = rp[u], r1 = rp[u + 1], d = r1 - r0;
        const int64_t w = u >> 6;
        bool esc = false;
        if (d <= 64 || d <= 4 * (int64_t)nseg) {
            int64_t r = r0;
            while (r < r1) {
                const int b = (int)(col[r] / sv);
                if (col[r] < 0 || b >= nseg) {   // unvalidated input: the build then fails (sum != nnz)
                    r++;
                    continue;
                }
                const int64_t lim = (int64_t)(b + 1) * sv;
                int64_t e = r + 1;
                while (e < r1 && col[e] < lim) e++;
                const int64_t len = e - r;
                cnt[(size_t)b * npad + u] = (uint8_t)(len >= 255 ? 255 : len);
                atomicAdd(wsum + (size_t)b * nw1 + w, (unsigned long long)len);
                esc |= len >= 255;
                r = e;
            }
        } else {
            int64_t lo_prev = 0;   // offset of segment b within the row
            for (int b = 0; b < nseg; b++) {
                const int64_t key = (int64_t)(b + 1) * sv;
                int64_t lo = lo_prev, hi = d;
                while (lo < hi) {
                    const int64_t mid = (lo + hi) >> 1;
                    if ((int64_t)col[r0 + mid] < key) lo = mid + 1;
                    else hi = mid;
                }
                const int64_t len = lo - lo_prev;
                if (len) {
                    cnt[(size_t)b * npad + u] = (uint8_t)(len >= 255 ? 255 : len);
                    atomicAdd(wsum + (size_t)b * nw1 + w, (unsigned long long)len);
                    esc |= len >= 255;
                }
                lo_prev = lo;
                if (lo == d) break;
            }
        }
        int32_t k = -1;
        if (esc) {
            k = (int32_t)atomicAdd(nx, 1u);
            xvert[k] = (int32_t)u;
        }
        xidx[u] = k;
    }
}

// xoff[k][b] = number of arcs of escape vertex xvert[k] into segments < b (lower bound of b*sv)
__global__ void k_scsr_xoff(const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                            const int32_t *__restrict__ xvert, int64_t nx, int nseg, int64_t sv,
                            uint32_t *__restrict__ xoff) {
    const int64_t S1 = nseg + 1;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nx * S1; t += stride) {
        const int64_t k = t / S1;
        const int b = (int)(t % S1);
        const int32_t u = xvert[k];
        const int64_t r0 = rp[u], d = rp[u + 1] - r0;
        int64_t lo = 0, hi = d;
        const int64_t key = (int64_t)b * sv;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if ((int64_t)col[r0 + mid] < key) lo = mid + 1;
            else hi = mid;
        }
        xoff[t] = (uint32_t)lo;
    }
}

// Every (segment, unit) range is padded to a multiple of 4 arcs (16 B) so that ranges start and
// end on 16-B boundaries: the sweep's slots then hold whole quads.  The pad is added to the
// unit's last word; k_scsr_padfill fills it with copies of the range's first arc (idempotent).
__global__ void k_scsr_pad(unsigned long long *__restrict__ wsum, int64_t nw1, int64_t nw2, int nseg,
                           uint8_t *__restrict__ upad, unsigned long long *total_pad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nw2 * nseg; t += stride) {
        const int64_t b = t / nw2, u = t % nw2;
        unsigned long long *ws = wsum + (size_t)b * nw1;
        const int64_t w0 = u * 64, w1 = min(nw1, w0 + 64);
        unsigned long long real = 0;
        for (int64_t w = w0; w < w1; w++) real += ws[w];
        const uint32_t pad = (uint32_t)((4u - (uint32_t)(real & 3u)) & 3u);
        upad[t] = (uint8_t)pad;
        if (pad) {
            ws[w1 - 1] += pad;
            atomicAdd(total_pad, (unsigned long long)pad);
        }
    }
}
__global__ void k_scsr_padfill(const uint8_t *__restrict__ upad, ScsrView s, int64_t nw2, uint32_t *__restrict__ scol) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nw2 * s.nseg; t += stride) {
        const uint32_t pad = upad[t];
        if (!pad) continue;
        const int64_t b = t / nw2, u = t % nw2;
        const uint32_t *base = s.base + (size_t)b * (s.nw1 + 1);
        const int64_t lo = s.start[b] + base[u * 64], hi = s.start[b] + base[min(u * 64 + 64, s.nw1)];
        const uint32_t first = scol[lo];
        for (uint32_t i = 1; i <= pad; i++) scol[hi - i] = first;
    }
}

// One CTA per segment: base[b][w] = exclusive prefix of wsum[b][*] (u32), base[b][nw1] = the
// block size, total[b] = the same in 64 bits (the host rejects blocks >= 2^32 arcs).
__global__ void __launch_bounds__(1024) k_scsr_scan(const unsigned long long *__restrict__ wsum, int64_t nw1,
                                                    uint32_t *__restrict__ base,
                                                    unsigned long long *__restrict__ total) {
    __shared__ unsigned long long s_w[32];
    const int b = blockIdx.x;
    const unsigned long long *ws = wsum + (size_t)b * nw1;
    uint32_t *bs = base + (size_t)b * (nw1 + 1);
    const int64_t per = (nw1 + 1023) / 1024;
    const int64_t a = threadIdx.x * per, e = min(nw1, a + per);
    unsigned long long loc = 0;
    for (int64_t i = a; i < e; i++) loc += ws[i];
    const int lane = lane_id(), warp = threadIdx.x >> 5;
    const unsigned long long incl = warp_inclusive_scan(loc);
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    if (warp == 0) {
        const unsigned long long x = s_w[lane];
        const unsigned long long xi = warp_inclusive_scan(x);
        s_w[lane] = xi - x;
        if (lane == 31) {
            total[b] = xi;
            bs[nw1] = (uint32_t)xi;
        }
    }
    __syncthreads();
    unsigned long long run = s_w[warp] + incl - loc;
    for (int64_t i = a; i < e; i++) {
        bs[i] = (uint32_t)run;
        run += ws[i];
    }
}

// Code of a stored arc (32 bits), laid out so the sweep decodes it with the fewest ALU ops:
//   [31:25] source word in its unit's 128 32-bit activity words (src >> 5)   - one shift
//   [24:10] destination word in the segment slice (dst >> 5)                 - shift + and
//   [9:5]   destination bit (dst & 31)  - a wrapping funnel shift reads it after one shift
//   [4:0]   source bit (src & 31)       - a wrapping funnel shift reads it directly
// with src = u mod 4096 (u's position in its 4096-vertex unit) and dst = v - b*sv < 2^20.
__host__ __device__ __forceinline__ uint32_t scsr_code(uint32_t src, uint32_t dst) {
    return ((src >> 5) << 25) | (((dst >> 5) & 0x7fffu) << 10) | ((dst & 31u) << 5) | (src & 31u);
}

struct ScsrBuild {
    const uint8_t *cnt;     // [nseg][nw1*64] part lengths, 255 = escape
    const int32_t *xidx;    // [n] escape row or -1
    const uint32_t *xoff;   // [nx][nseg+1]
};

__device__ __forceinline__ uint32_t scsr_exact(const ScsrBuild &B, int nseg, uint32_t c, int64_t u, int b) {
    if (c != 255u) return c;
    const int32_t k = __ldg(B.xidx + u);
    const uint32_t *o = B.xoff + (size_t)k * (nseg + 1);
    return __ldg(o + b + 1) - __ldg(o + b);
}

// Warp per word: scatter each vertex's parts into the segment blocks as tagged arcs.  Every
// destination is checked to lie in its segment (rows must be sorted): *bad != 0 fails the build.
__global__ void k_scsr_fill(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                            ScsrView s, ScsrBuild B, uint32_t *__restrict__ scol, unsigned int *bad) {
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t npad = s.nw1 * 64;
    const uint32_t svu = (uint32_t)s.sv;
    for (int64_t w = gw; w < s.nw1; w += nwarps) {
        const int64_t u0 = w * 64 + 2 * lane, u1 = u0 + 1;
        const uint32_t tag0 = (uint32_t)(u0 & ((1 << SCSR_UNIT_SHIFT) - 1));
        const uint32_t tag1 = tag0 + 1u;
        int64_t off0 = u0 < n ? rp[u0] : 0, off1 = u1 < n ? rp[u1] : 0;   // next arc of the row to place
        bool oob = false;
        for (int b = 0; b < s.nseg; b++) {
            const uint16_t cc = *reinterpret_cast<const uint16_t *>(B.cnt + (size_t)b * npad + u0);
            const uint32_t c0 = u0 < n ? scsr_exact(B, s.nseg, cc & 0xffu, u0, b) : 0u;
            const uint32_t c1 = u1 < n ? scsr_exact(B, s.nseg, cc >> 8, u1, b) : 0u;
            const uint32_t tot = c0 + c1;
            if (!__any_sync(0xffffffffu, tot != 0)) continue;
            const uint32_t incl = warp_inclusive_scan(tot);
            const int64_t dst = s.start[b] + s.base[(size_t)b * (s.nw1 + 1) + w] + (incl - tot);
            const int32_t rel = (int32_t)((int64_t)b * s.sv);
            // long parts: the whole warp copies them
            for (int h = 0; h < 2; h++) {
                const int64_t src = h ? off1 : off0, len = h ? c1 : c0, d0 = h ? dst + c0 : dst;
                const uint32_t tg = h ? tag1 : tag0;
                uint32_t big = __ballot_sync(0xffffffffu, len >= 64);
                while (big) {
                    const int l = __ffs(big) - 1;
                    big &= big - 1;
                    const int64_t sa = __shfl_sync(0xffffffffu, src, l), la = __shfl_sync(0xffffffffu, len, l);
                    const int64_t da = __shfl_sync(0xffffffffu, d0, l);
                    const uint32_t ta = __shfl_sync(0xffffffffu, tg, l);
                    for (int64_t i = lane; i < la; i += 32) {
                        const int32_t r = col[sa + i] - rel;
                        oob |= (uint32_t)r >= svu;
                        scol[da + i] = scsr_code(ta, (uint32_t)r);
                    }
                }
                if (len < 64)
                    for (int64_t i = 0; i < len; i++) {
                        const int32_t r = col[src + i] - rel;
                        oob |= (uint32_t)r >= svu;
                        scol[d0 + i] = scsr_code(tg, (uint32_t)r);
                    }
            }
            off0 += c0;
            off1 += c1;
        }
        if (oob) atomicOr(bad, 1u);
    }
}

// ---------------------------------------------------------------------------------------
// the sweep

struct SweepParams {
    ScsrView s;
    const uint64_t *in_bits;        // input frontier, layer 1
    const uint64_t *in_summ;        // input frontier, layer 2: unit k active <=> in_summ[k] != 0
    DevStats *st;                   // arcs (accumulated)
    uint64_t *visited;
    int64_t nw2;                    // units
    unsigned long long min_mf;      // graph mode: run only if the frontier's m_f >= min_mf (0: always)
};

struct SwRec {
    uint32_t n;       // arcs in the slot
    uint32_t skew;    // first arc's offset inside the slot (0..3)
    int32_t unit;     // source unit of the arcs; DATA only
    int32_t kind;     // SW_DATA, SW_SWITCH (unit = new segment), SW_STOP
};
enum { SW_DATA = 0, SW_SWITCH = 1, SW_STOP = 2 };
struct SwTask {
    int64_t lo, hi;   // arc range of one active unit in segment b's block (absolute)
    int32_t u, b;     // unit; segment (-1: no more work)
};

__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void sw_mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void sw_mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void sw_mbar_arrive_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void sw_mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_addr(bar)), "r"(parity)
            : "memory");
    } while (!done);
}
// waiting consumers: try_wait with a suspend-time hint (the thread sleeps until the phase
// completes or the hint expires instead of spinning on issue slots)
__device__ __forceinline__ void sw_mbar_wait_sleep(uint64_t *bar, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_addr(bar)), "r"(parity), "r"(20000u)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void sw_bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_addr(dst)),
        "l"(src), "r"(bytes), "r"(smem_addr(bar))
        : "memory");
}
__device__ __forceinline__ void consumer_sync() { asm volatile("bar.sync 1, %0;" ::"n"(SW_CONSUMERS) : "memory"); }

__device__ __forceinline__ void sw_mark(uint32_t *s_vis32, uint32_t v) {
    const uint32_t m = 1u << (v & 31);
    if (!(s_vis32[v >> 5] & m)) atomicOr(s_vis32 + (v >> 5), m);
}

__global__ void __launch_bounds__(SW_THREADS, 1) k_push_sweep(SweepParams p) {
    extern __shared__ __align__(128) unsigned char sw_smem[];
    uint64_t *s_vis = reinterpret_cast<uint64_t *>(sw_smem + (size_t)SW_STAGES * SW_SLOT_BYTES);
    __shared__ SwRec s_rec[SW_STAGES];
    __shared__ __align__(8) uint64_t s_full[SW_STAGES], s_empty[SW_STAGES];
    __shared__ SwTask s_task[SW_TASKS];
    __shared__ uint32_t s_thead, s_ttail;
    if (p.min_mf && p.st->mf < p.min_mf) return;
    const ScsrView &S = p.s;
    const int nseg = S.nseg;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    if (threadIdx.x == 0) {
        for (int i = 0; i < SW_STAGES; i++) {
            sw_mbar_init(s_full + i, 1);
            sw_mbar_init(s_empty + i, SW_CONSUMERS / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        s_thead = s_ttail = 0;
    }
    __syncthreads();
    if (warp == 1) {
        // ---------------- scheduler: items -> active unit ranges ----------------
        // grabs work items (segment, SW_UNITS units), loads their summary words and block
        // offsets with one warp-wide round of loads, and queues the active units' arc ranges
        // for the producer, which therefore never waits on an atomic or a metadata load
        const uint32_t nitems = (uint32_t)((p.nw2 + SW_UNITS - 1) / SW_UNITS);
        int home = (int)(blockIdx.x % (unsigned)nseg);
        uint32_t tail = 0;
        auto push = [&](const SwTask &t) {   // lane 0 only
            while (tail - *(volatile uint32_t *)&s_thead >= (uint32_t)SW_TASKS) __nanosleep(64);
            s_task[tail % SW_TASKS] = t;
            __threadfence_block();
            *(volatile uint32_t *)&s_ttail = ++tail;
        };
        for (;;) {
            uint32_t it = 0xffffffffu;
            int b = home;
            if (lane == 0) {
                for (int t = 0; t < nseg; t++) {
                    if (*(volatile uint32_t *)(S.qc + b) < nitems) {
                        it = atomicAdd(S.qc + b, 1u);
                        if (it < nitems) break;
                        it = 0xffffffffu;
                    }
                    b = b + 1 == nseg ? 0 : b + 1;
                }
            }
            it = __shfl_sync(0xffffffffu, it, 0);
            b = __shfl_sync(0xffffffffu, b, 0);
            if (it == 0xffffffffu) break;
            home = b;
            const int64_t sb = S.start[b];
            const uint32_t *base = S.base + (size_t)b * (S.nw1 + 1);
            const int64_t u = (int64_t)it * SW_UNITS + lane;
            int64_t lo = 0, hi = 0;
            bool act = false;
            if (lane < SW_UNITS && u < p.nw2) {
                const uint64_t sm = __ldg(p.in_summ + u);
                lo = sb + __ldg(base + u * 64);
                hi = sb + __ldg(base + min(u * 64 + 64, S.nw1));
                act = sm != 0ull && hi > lo;
            }
            uint32_t am = __ballot_sync(0xffffffffu, act);
            while (am) {
                const int j = __ffs(am) - 1;
                am &= am - 1;
                const int64_t l = __shfl_sync(0xffffffffu, lo, j), h = __shfl_sync(0xffffffffu, hi, j);
                if (lane == 0) push(SwTask{l, h, (int32_t)(it * SW_UNITS + j), b});
            }
        }
        if (lane == 0) push(SwTask{0, 0, 0, -1});
    } else if (warp == 0) {
        // ---------------- producer (lane 0): unit ranges -> ring slots ----------------
        if (lane == 0) {
            uint32_t k = 0, head = 0;   // ring position, task queue position
            int announced = -1;
            auto slot = [&](int kind, uint32_t n, uint32_t skew, int32_t unit) -> int {
                const int s = (int)(k % SW_STAGES);
                sw_mbar_wait(s_empty + s, ((k / SW_STAGES) & 1u) ^ 1u);
                s_rec[s] = SwRec{n, skew, unit, kind};
                k++;
                return s;
            };
            for (;;) {
                while (*(volatile uint32_t *)&s_ttail == head) __nanosleep(32);
                __threadfence_block();
                const SwTask t = s_task[head % SW_TASKS];
                *(volatile uint32_t *)&s_thead = ++head;
                if (t.b < 0) break;
                if (t.b != announced) {
                    const int s = slot(SW_SWITCH, 0u, 0u, t.b);
                    sw_mbar_arrive(s_full + s);
                    announced = t.b;
                }
                // the unit's layer-1 words (16-B multiple; frontier buffers carry 8 words of padding)
                const uint32_t act_bytes = (uint32_t)(((min((int64_t)64, S.nw1 - (int64_t)t.u * 64) + 1) & ~1ll) * 8);
                // ranges are padded to whole quads and start 16-B aligned (k_scsr_pad): every slot
                // but a range's last is full
                for (int64_t c = t.lo; c < t.hi;) {
                    const int64_t nx = min(t.hi, c + (int64_t)SW_QUADS * 4);
                    const uint32_t n = (uint32_t)(nx - c);
                    const uint32_t bytes = n * 4u;
                    const int s = slot(SW_DATA, n, 0u, t.u);
                    unsigned char *dst = sw_smem + (size_t)s * SW_SLOT_BYTES;
                    sw_mbar_arrive_tx(s_full + s, bytes + act_bytes);
                    sw_bulk_g2s(dst, p.in_bits + (int64_t)t.u * 64, act_bytes, s_full + s);
                    sw_bulk_g2s(dst + SW_ACT_BYTES, S.col + c, bytes, s_full + s);
                    c = nx;
                }
            }
            const int s = slot(SW_STOP, 0u, 0u, 0);
            sw_mbar_arrive(s_full + s);
        }
    } else {
        // ---------------- consumers ----------------
        const int ct = threadIdx.x - 64;
        uint32_t *s_vis32 = reinterpret_cast<uint32_t *>(s_vis);
        int loaded = -1, nwl = 0;
        auto flush = [&]() {
            const int64_t w0 = (int64_t)loaded * S.sw;
            for (int i = ct; i < nwl; i += SW_CONSUMERS) {
                const uint64_t x = s_vis[i];
                if (!x) continue;
                const uint64_t nb = x & ~p.visited[w0 + i];
                if (nb) atomic_or_u64(p.visited + w0 + i, nb);
            }
        };
        for (uint32_t k = 0;; k++) {
            const int s = (int)(k % SW_STAGES);
            sw_mbar_wait_sleep(s_full + s, (k / SW_STAGES) & 1u);
            const SwRec r = s_rec[s];
            if (r.kind == SW_STOP) break;
            if (r.kind == SW_SWITCH) {
                consumer_sync();   // every consumer is done with the previous segment's slots
                if (loaded >= 0) flush();
                loaded = r.unit;
                const int64_t w0 = (int64_t)loaded * S.sw;
                nwl = (int)(S.nw1 - w0 < S.sw ? S.nw1 - w0 : S.sw);
                for (int i = ct; i < nwl; i += SW_CONSUMERS) s_vis[i] = p.visited[w0 + i];
                consumer_sync();
            } else {
                const unsigned char *slot_p = sw_smem + (size_t)s * SW_SLOT_BYTES;
                const uint32_t *act32 = reinterpret_cast<const uint32_t *>(slot_p);
                const uint4 *qs = reinterpret_cast<const uint4 *>(slot_p + SW_ACT_BYTES);
                uint4 q[SW_QPT];
#pragma unroll
                for (int h = 0; h < SW_QPT; h++) {
                    const uint32_t qi = (uint32_t)(h * SW_CONSUMERS + ct);
                    q[h] = qs[qi];   // stale data past `end` is masked below
                }
                // all SW_QPT*4 arcs of the thread at once: activity words and probes first, then
                // the decisions, then the shared-memory ORs for active arcs to unset bits
                constexpr int NA = SW_QPT * 4;
                uint32_t v[NA];
#pragma unroll
                for (int h = 0; h < SW_QPT; h++) {
                    v[4 * h + 0] = q[h].x;
                    v[4 * h + 1] = q[h].y;
                    v[4 * h + 2] = q[h].z;
                    v[4 * h + 3] = q[h].w;
                }
                uint32_t aw[NA], vw[NA];
#pragma unroll
                for (int j = 0; j < NA; j++) {
                    aw[j] = act32[v[j] >> 25];
#if !SG_SW_NOPROBE
                    vw[j] = s_vis32[(v[j] >> 10) & 0x7fffu];
#endif
                }
                // ranges are padded to whole quads: only quads past the slot's end are masked
#pragma unroll
                for (int h = 0; h < SW_QPT; h++)
                    if ((uint32_t)(h * SW_CONSUMERS + ct) * 4 >= r.n)
#pragma unroll
                        for (int j = 0; j < 4; j++) aw[4 * h + j] = 0u;
#pragma unroll
                for (int j = 0; j < NA; j++) {
                    const uint32_t a = __funnelshift_r(aw[j], 0u, v[j]);          // bit 0: source active
                    const uint32_t db = v[j] >> 5;                                 // low 5 bits: destination bit
#if SG_SW_NOPROBE
                    if (a & 1u) atomicOr(s_vis32 + ((v[j] >> 10) & 0x7fffu), __funnelshift_l(0u, 1u, db));
#else
                    const uint32_t d = __funnelshift_r(vw[j], 0u, db);             // bit 0: destination visited
                    if ((a & ~d) & 1u) atomicOr(s_vis32 + ((v[j] >> 10) & 0x7fffu), __funnelshift_l(0u, 1u, db));
#endif
                }
            }
            __syncwarp();
            if (lane == 0) sw_mbar_arrive(s_empty + s);
        }
        consumer_sync();
        if (loaded >= 0) flush();
    }
}

// The statistics of a sweep step: the exact sum of the input frontier's degrees (the arcs a push
// step inspects, as the word path counts them), one thread per listed word, 4 row_ptr pairs in
// flight per iteration.
__global__ void __launch_bounds__(256) k_frontier_arcs(const int64_t *__restrict__ rp, const uint64_t *__restrict__ in_bits,
                                                       const uint32_t *__restrict__ offsets, DevStats *st,
                                                       unsigned long long min_mf) {
    __shared__ unsigned long long s_a[8];
    if (min_mf && st->mf < min_mf) return;
    const uint32_t count = (uint32_t)st->count;
    unsigned long long acc = 0;
    const uint32_t stride = gridDim.x * blockDim.x;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
        const int64_t w = offsets[i];
        uint64_t x = __ldg(in_bits + w);
        while (x) {
            int64_t v[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                v[k] = x ? w * 64 + (__ffsll((long long)x) - 1) : -1;
                x &= x - 1;
            }
#pragma unroll
            for (int k = 0; k < 4; k++)
                if (v[k] >= 0) acc += (unsigned long long)(__ldg(rp + v[k] + 1) - __ldg(rp + v[k]));
        }
    }
    acc = warp_sum(acc);
    if (lane_id() == 0) s_a[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int i = 0; i < 8; i++) t += s_a[i];
        if (t) atomicAdd(&st->arcs, t);
    }
}

// ---------------------------------------------------------------------------------------
// host side

static int sm_count() { return num_sms(); }

cudaError_t scsr_build(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int32_t sw, ScsrStore *out,
                       cudaStream_t s) {
    ScsrStore &S = *out;
    S = ScsrStore{};
    if (sw < 1 || sw > SCSR_MAX_SW) sw = SCSR_MAX_SW;
    const int64_t nw1 = (n + 63) / 64, npad = nw1 * 64;
    const int64_t sv = (int64_t)sw * 64;
    const int nseg = (int)((n + sv - 1) / sv);
    S.v.nw1 = nw1;
    S.v.sw = sw;
    S.v.sv = sv;
    S.v.nseg = nseg;
    cudaError_t e = cudaSuccess;
    uint8_t *cnt = nullptr;
    int32_t *xidx = nullptr, *xvert = nullptr;
    uint32_t *xoff = nullptr;
    unsigned long long *wsum = nullptr, *tot = nullptr;
    unsigned int *nx_d = nullptr;
    std::vector<unsigned long long> h(nseg + 1);
    std::vector<int64_t> start(nseg);
    unsigned int nx = 0, bad = 0;
    unsigned long long tpad = 0;
    uint8_t *upad = nullptr;
    const int64_t nw2 = (nw1 + 63) / 64;
    int64_t acc = 0;
    bool too_big = false;
    const int64_t max_x = nnz / 255 + 1;
#define SCK(x) do { e = (x); if (e != cudaSuccess) goto done; } while (0)
    SCK(cudaMalloc(&cnt, (size_t)nseg * npad + 16));
    SCK(cudaMemsetAsync(cnt, 0, (size_t)nseg * npad + 16, s));
    SCK(cudaMalloc(&wsum, sizeof(unsigned long long) * (size_t)nseg * nw1));
    SCK(cudaMemsetAsync(wsum, 0, sizeof(unsigned long long) * (size_t)nseg * nw1, s));
    SCK(cudaMalloc(&xidx, sizeof(int32_t) * (size_t)n));
    SCK(cudaMalloc(&xvert, sizeof(int32_t) * (size_t)max_x));
    SCK(cudaMalloc(&nx_d, 16 + sizeof(unsigned long long) * (size_t)(nseg + 1)));
    SCK(cudaMemsetAsync(nx_d, 0, 16, s));
    tot = reinterpret_cast<unsigned long long *>(nx_d + 4);
    {
        int64_t blocks = (n + 255) / 256;
        if (blocks > sm_count() * 8) blocks = sm_count() * 8;
        note_launch();
        k_scsr_count<<<(int)(blocks < 1 ? 1 : blocks), 256, 0, s>>>(rp, col, n, npad, nw1, nseg, sv, cnt, wsum, xidx,
                                                                    xvert, nx_d);
    }
    SCK(cudaMalloc(&upad, (size_t)nseg * nw2));
    {
        int64_t bl = (nseg * nw2 + 255) / 256;
        if (bl > sm_count() * 8) bl = sm_count() * 8;
        note_launch();
        k_scsr_pad<<<(int)(bl < 1 ? 1 : bl), 256, 0, s>>>(wsum, nw1, nw2, nseg, upad,
                                                           reinterpret_cast<unsigned long long *>(nx_d + 2));
    }
    SCK(dev_alloc(&S.base, sizeof(uint32_t) * (size_t)nseg * (nw1 + 1), s));
    note_launch();
    k_scsr_scan<<<nseg, 1024, 0, s>>>(wsum, nw1, S.base, tot);
    SCK(cudaMemcpyAsync(&nx, nx_d, sizeof(unsigned int), cudaMemcpyDeviceToHost, s));
    SCK(cudaMemcpyAsync(&tpad, nx_d + 2, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    SCK(cudaMemcpyAsync(h.data(), tot, sizeof(unsigned long long) * nseg, cudaMemcpyDeviceToHost, s));
    SCK(cudaStreamSynchronize(s));
    SCK(cudaGetLastError());
    for (int b = 0; b < nseg; b++) {
        start[b] = acc;
        acc += (int64_t)h[b];
        too_big |= h[b] >= 0xffffffffull;
    }
    if (too_big || acc != nnz + (int64_t)tpad) {   // segment block >= 2^32 arcs, or ids outside [0, n)
        e = cudaErrorInvalidValue;
        goto done;
    }
    S.nx = nx;
    SCK(dev_alloc(&S.start, sizeof(int64_t) * (size_t)nseg, s));
    SCK(cudaMemcpyAsync(S.start, start.data(), sizeof(int64_t) * nseg, cudaMemcpyHostToDevice, s));
    SCK(cudaMalloc(&xoff, sizeof(uint32_t) * (size_t)(nx ? nx : 1) * (nseg + 1)));
    if (nx) {
        const int64_t items = (int64_t)nx * (nseg + 1);
        int64_t bl = (items + 255) / 256;
        if (bl > sm_count() * 8) bl = sm_count() * 8;
        note_launch();
        k_scsr_xoff<<<(int)bl, 256, 0, s>>>(rp, col, xvert, nx, nseg, sv, xoff);
    }
    SCK(dev_alloc(&S.col, sizeof(uint32_t) * (size_t)acc + 64, s));
    SCK(cudaMemsetAsync((char *)S.col + sizeof(uint32_t) * (size_t)acc, 0, 64, s));
    SCK(dev_alloc(&S.qc, sizeof(uint32_t) * (size_t)nseg, s));
    S.v.col = S.col;
    S.v.base = S.base;
    S.v.start = S.start;
    S.v.qc = S.qc;
    {
        int64_t bl = (nw1 * 32 + 255) / 256;
        if (bl > sm_count() * 8) bl = sm_count() * 8;
        SCK(cudaMemsetAsync(nx_d, 0, sizeof(unsigned int), s));
        note_launch();
        k_scsr_fill<<<(int)(bl < 1 ? 1 : bl), 256, 0, s>>>(rp, col, n, S.v, ScsrBuild{cnt, xidx, xoff}, S.col, nx_d);
        int64_t bp = (nseg * nw2 + 255) / 256;
        if (bp > sm_count() * 8) bp = sm_count() * 8;
        note_launch();
        k_scsr_padfill<<<(int)(bp < 1 ? 1 : bp), 256, 0, s>>>(upad, S.v, nw2, S.col);
    }
    SCK(cudaMemcpyAsync(&bad, nx_d, sizeof(unsigned int), cudaMemcpyDeviceToHost, s));
    SCK(cudaStreamSynchronize(s));
    SCK(cudaGetLastError());
    if (bad) e = cudaErrorInvalidValue;   // unsorted rows: keep the word path
    S.bytes = sizeof(uint32_t) * (size_t)acc + sizeof(uint32_t) * (size_t)nseg * (nw1 + 1);
done:
#undef SCK
    cudaFree(cnt);
    cudaFree(wsum);
    cudaFree(xidx);
    cudaFree(xvert);
    cudaFree(xoff);
    cudaFree(nx_d);
    cudaFree(upad);
    if (e != cudaSuccess) {
        cudaDeviceSynchronize();
        scsr_free(out);
    }
    return e;
}

void scsr_free(ScsrStore *S) {
    dev_free(S->col);   // (callers synchronise first: graph_free)
    dev_free(S->base);
    dev_free(S->start);
    dev_free(S->qc);
    *S = ScsrStore{};
}

void launch_push_sweep(const ScsrView &v, const int64_t *rp, const uint64_t *in_bits, const uint64_t *in_summ,
                       const uint32_t *offsets, int64_t nw2, DevStats *st, uint64_t *visited,
                       unsigned long long min_mf, cudaStream_t s) {
    static bool attr = false;
    // the whole 128 KB slice is always allocated: masked lanes may probe any 15-bit word index
    const size_t smem = (size_t)SW_STAGES * SW_SLOT_BYTES + (size_t)SCSR_MAX_SW * sizeof(uint64_t);
    if (!attr) {
        cudaFuncSetAttribute(k_push_sweep, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)((size_t)SW_STAGES * SW_SLOT_BYTES + (size_t)SCSR_MAX_SW * 8));
        attr = true;
    }
    SweepParams p;
    p.s = v;
    p.in_bits = in_bits;
    p.in_summ = in_summ;
    p.st = st;
    p.visited = visited;
    p.nw2 = nw2;
    p.min_mf = min_mf;
    cudaMemsetAsync(v.qc, 0, sizeof(uint32_t) * (size_t)v.nseg, s);
    note_launch();
    k_push_sweep<<<sm_count(), SW_THREADS, smem, s>>>(p);
    note_launch();
    k_frontier_arcs<<<sm_count() * 8, 256, 0, s>>>(rp, in_bits, offsets, st, min_mf);
}

}  // namespace sg
