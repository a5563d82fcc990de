// bcb.cu — source-batched Brandes BC (algorithm PAPER.md:161 §3.4).
//
// Up to 32 sources advance in lock-step, one bit per source in a per-vertex 32-bit mask (lane j
// of a warp = source j): the frontier of level d is a list L_d of (vertex, mask) entries, the
// per-source path counts sigma live in [n][32] doubles.  A high-diameter graph (config 5: ~10^4
// levels of a few thousand vertices each) then does 32 sources' work per superstep, and each
// direction (forward / backward) is ONE persistent cooperative kernel whose supersteps are
// separated by grid-wide barriers (two per level) instead of kernel launches.
//
// Forward level d -> d+1 (k_j(d) = exponent of the max of level d's stored sigma for source j):
//   A  expand (QUAD threads per entry): for (v, m) in L_d, w in N(v): nm = m & ~V[w]; if nm:
//      F_{d+1}[w] |= nm and w into a vertex-level 2LB (VB / VS);  clear F_{d-1}      | grid sync
//   A2 extract L_{d+1} from the 2LB in ascending vertex order (summary compaction), clear it
//                                                                                  | grid sync
//   B  sigma (QUAD threads per new entry, loop over its sources j; fixed-order gather):
//        s[w][j] = 2^-k_j(d) * sum_{v in N(w), j in F_d[v]} s[v][j];  V[w] |= F_{d+1}[w]
//      per-source max -> k_j(d+1); control step                                    | grid sync
//   (three frontier-mask buffers rotate: F_{d-1} is cleared while F_d / F_{d+1} are live)
// Stored s is sigma scaled by 2^-G_j(level) with G_j(L+1) = G_j(L) + k_j(L): exact power-of-two
// scaling (reading C20 / R5), every level's max in [1, 2).  (Pushing sigma with fp64 atomics in
// A instead was measured slower on config 5: 302 vs 284 ms of forward time per batch.)
// Backward, one pass per level d = D-1 .. 1 (three rotating level-mask buffers M):
//   for (v, m) in L_d, j in m: delta[v][j] = 2^-k_j(d) * s[v][j] * acc[v][j], where acc (the
//   `delta` array) holds sum_{w succ} (1 + delta[w][j]) / s[w][j] pushed by the pass of d+1;
//   bc[v] += delta[v][j] (j ascending); push (1 + delta[v][j]) / s[v][j] to predecessors u with
//   j in M_{d-1}[u] (fp64 atomics, as the paper's functors; one barrier per level instead of
//   the gather's two); lay out M_{d-2}, clear M_d                                  | grid sync
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sg {

constexpr int BCB_B = 32;   // sources per batch
#ifndef SG_BCB_THREADS
#define SG_BCB_THREADS 1024
#endif
#ifndef SG_BCB_PER_SM
#define SG_BCB_PER_SM 1
#endif
constexpr int BCB_THREADS = SG_BCB_THREADS;   // few large CTAs: a grid barrier over 148 CTAs is cheap
#ifndef SG_BCB_QUAD
#define SG_BCB_QUAD 2
#endif
constexpr int QUAD = SG_BCB_QUAD;             // threads per level entry (arcs strided by QUAD)

struct BcbView {
    GraphView g;
    uint32_t *F;          // [3][n] frontier masks (rotating)
    uint32_t *V;          // [n] visited masks
    uint32_t *M;          // [2][n] backward: masks of level d+1
    uint64_t *VB, *VS;    // vertex-level 2LB of the level being built (layer 1 / layer 2)
    double *s;            // [n][32] scaled sigma
    double *delta;        // [n][32]
    int32_t *lv;          // list vertices (all levels, concatenated)
    uint32_t *lm;         // list masks
    unsigned long long *loff;   // [cap+2] level start offsets
    unsigned long long *maxb;   // [cap+1][32] per level, per source: 4096 + max exponent of s (0: none)
    BcbCtrl *c;
    int32_t cap;          // level capacity
    int64_t lcap;         // list capacity
    double *bc;
};

constexpr int EXP_BIAS = 4096;
__device__ __forceinline__ int kexp(unsigned long long mb) { return mb ? (int)mb - EXP_BIAS : 0; }
__device__ __forceinline__ int exp_of(double x) {   // floor(log2 x) for a positive normal double
    return (int)((__double_as_longlong(x) >> 52) & 0x7ff) - 1023;
}
template <typename T>
__device__ __forceinline__ T vload(const T *p) { return *reinterpret_cast<const volatile T *>(p); }
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// F_{d+1}[w] |= nm and w into the level's vertex 2LB (fire-and-forget ORs)
__device__ __forceinline__ void bcb_mark(const BcbView &b, uint32_t *Fn, int32_t w, uint32_t nm) {
    if (nm) {
        atomicOr(Fn + w, nm);
        atomic_or_u64(b.VB + (w >> 6), 1ull << (w & 63));
        atomic_or_u64(b.VS + (w >> 12), 1ull << ((w >> 6) & 63));
    }
}

// L_0: masks of the batch's sources (duplicates merge into one entry)
__global__ void k_bcb_init(BcbView b) {
    BcbCtrl *c = b.c;
    const int j = threadIdx.x;
    if (j < c->nsrc) {
        const int32_t s = c->src[j];
        const uint32_t old = atomicOr(b.F + s, 1u << j);
        atomicOr(b.V + s, 1u << j);
        b.s[(int64_t)s * BCB_B + j] = 1.0;
        if (old == 0u) {
            const unsigned long long pos = atomicAdd(&c->ltop, 1ull);
            b.lv[pos] = s;
        }
    }
    __syncthreads();
    if (j == 0) {
        b.loff[0] = 0;
        b.loff[1] = c->ltop;
        c->d = 0;
        c->par = 0;
        c->depth = 1;
        c->overflow = 0;
    }
    __syncthreads();
    for (unsigned long long i = j; i < c->ltop; i += blockDim.x) b.lm[i] = b.F[b.lv[i]];
    if (j < BCB_B) b.maxb[j] = EXP_BIAS;   // level 0: every sigma is 1.0 (exponent 0)
}

__global__ void __launch_bounds__(BCB_THREADS) k_bcb_forward(BcbView b) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_maxe[BCB_B], s_kexp[BCB_B];
    // control words are read by one thread per CTA and broadcast through shared memory (151K
    // threads loading one address would queue ~5K requests on one L2 slice per phase)
    __shared__ unsigned long long s_ctl[6];
    BcbCtrl *c = b.c;
    const int64_t n = b.g.n;
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    unsigned long long t_mark = gtimer();
    for (;;) {
        if (threadIdx.x == 0) {
            const int dd = vload(&c->d);
            s_ctl[0] = (unsigned long long)dd;
            s_ctl[1] = vload(&b.loff[dd]);
            s_ctl[2] = vload(&b.loff[dd + 1]);
            s_ctl[3] = dd >= 1 ? vload(&b.loff[dd - 1]) : 0ull;
        }
        __syncthreads();
        const int d = (int)s_ctl[0];
        uint32_t *Fc = b.F + (int64_t)(d % 3) * n;            // masks of L_d
        uint32_t *Fn = b.F + (int64_t)((d + 1) % 3) * n;      // masks of L_{d+1} (being built)
        uint32_t *Fo = b.F + (int64_t)((d + 2) % 3) * n;      // masks of L_{d-1} (to clear)
        // ---- A: expand L_d into the next level's masks and a vertex-level 2LB; clear L_{d-1}
        {
            // QUAD threads per entry (thread k: arcs k, k+QUAD, ...): short dependent chains; all
            // updates are idempotent ORs issued without waiting for a result (RED)
            const unsigned long long a = s_ctl[1], e = s_ctl[2];
            const int k = (int)(tid & (QUAD - 1));
            for (unsigned long long i = a + tid / QUAD; i < e; i += nthr / QUAD) {
                const int32_t v = b.lv[i];
                const uint32_t m = b.lm[i];
                const int64_t r1 = __ldg(b.g.rp + v + 1);
                const int64_t ra = __ldg(b.g.rp + v) + k;
                // the thread's first two arcs are loaded side by side (two independent chains)
                const int32_t w0 = ra < r1 ? __ldg(b.g.col + ra) : 0;
                const int32_t w1 = ra + QUAD < r1 ? __ldg(b.g.col + ra + QUAD) : 0;
                const uint32_t n0 = ra < r1 ? m & ~vload(b.V + w0) : 0u;
                const uint32_t n1 = ra + QUAD < r1 ? m & ~vload(b.V + w1) : 0u;
                bcb_mark(b, Fn, w0, n0);
                bcb_mark(b, Fn, w1, n1);
                for (int64_t r = ra + 2 * QUAD; r < r1; r += QUAD) {
                    const int32_t w = __ldg(b.g.col + r);
                    bcb_mark(b, Fn, w, m & ~vload(b.V + w));
                }
            }
            if (d >= 1) {
                const unsigned long long a0 = s_ctl[3], e0 = s_ctl[1];
                for (unsigned long long i = a0 + tid; i < e0; i += nthr) Fo[b.lv[i]] = 0u;
            }
        }
        if (threadIdx.x < BCB_B) s_maxe[threadIdx.x] = -1000000;
        grid.sync();
        if (tid == 0) { const unsigned long long t1 = gtimer(); c->t_ns[0] += t1 - t_mark; t_mark = t1; }
        // ---- A2: the new level's entries in ascending vertex order (summary-layer compaction:
        // warp per summary word, lane l owns layer-1 words 64s+2l, 64s+2l+1), clearing the 2LB;
        // id order gives the sigma / delta passes spatial locality on sigma rows and masks
        // (one list reservation per CTA and round: a same-address atomic per summary word
        // serialises thousands of requests per level)
        {
            __shared__ uint32_t s_wofs[BCB_THREADS / 32];
            __shared__ unsigned long long s_base;
            const int lane = lane_id(), wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
            for (int64_t sw0 = (int64_t)blockIdx.x * nwb; sw0 < b.g.nw2; sw0 += (int64_t)gridDim.x * nwb) {
                const int64_t sw = sw0 + wib;
                const uint64_t x = sw < b.g.nw2 ? vload(b.VS + sw) : 0ull;
                const int64_t w0 = sw * 64 + 2 * lane;
                uint64_t y0 = 0, y1 = 0;
                if ((x >> (2 * lane)) & 1ull) y0 = vload(b.VB + w0);
                if ((x >> (2 * lane + 1)) & 1ull) y1 = vload(b.VB + w0 + 1);
                const uint32_t cnt = __popcll(y0) + __popcll(y1);
                const uint32_t incl = warp_inclusive_scan(cnt);
                if (lane == 31) s_wofs[wib] = incl;
                __syncthreads();
                if (wib == 0) {
                    const uint32_t t = lane < nwb ? s_wofs[lane] : 0u;
                    const uint32_t ti = warp_inclusive_scan(t);
                    if (lane < nwb) s_wofs[lane] = ti - t;
                    if (lane == 31) s_base = ti ? atomicAdd(&c->ltop, (unsigned long long)ti) : 0ull;
                }
                __syncthreads();
                unsigned long long base = s_base + s_wofs[wib] + (incl - cnt);
                __syncthreads();   // s_wofs / s_base are rewritten next round
                if (!x) continue;
                for (int q = 0; q < 2; q++) {
                    uint64_t y = q ? y1 : y0;
                    const int64_t w = w0 + q;
                    if (y) b.VB[w] = 0ull;
                    while (y) {
                        const int bit = __ffsll((long long)y) - 1;
                        y &= y - 1;
                        const int32_t v = (int32_t)(w * 64 + bit);
                        // stores only (a load whose result is stored would stall every bit);
                        // the mask lm is filled by phase B, which reads F_{d+1}[w] anyway
                        if (base < (unsigned long long)b.lcap) b.lv[base] = v;
                        base++;
                    }
                }
                if (lane == 0) b.VS[sw] = 0ull;
            }
        }
        grid.sync();
        if (tid == 0) { const unsigned long long t1 = gtimer(); c->t_ns[1] += t1 - t_mark; t_mark = t1; }
        // ---- B: sigma of the new level (thread per entry, loop over its sources); control step
        if (threadIdx.x == 0) s_ctl[4] = vload(&c->ltop);
        if (threadIdx.x < BCB_B) s_kexp[threadIdx.x] = kexp(vload(&b.maxb[(int64_t)d * BCB_B + threadIdx.x]));
        __syncthreads();
        const unsigned long long top0 = s_ctl[4];
        const bool over = top0 > (unsigned long long)b.lcap || d + 2 > b.cap;
        {
            const unsigned long long a = s_ctl[2];
            const unsigned long long e = over ? a : top0;
            // QUAD threads per entry: thread k sums arcs k, k+QUAD, ...; quad shuffle reduction in a
            // fixed order (deterministic)
            const int k = (int)(tid & (QUAD - 1));
            // warp-uniform trip count (the loop body uses warp shuffles / votes)
            const unsigned long long ncap = ((e - a) * QUAD + 31) / 32 * 32;
            for (unsigned long long ii = tid; ii < ncap; ii += nthr) {
                const unsigned long long i = a + ii / QUAD;
                const bool valid = i < e;
                const int32_t w = valid ? b.lv[i] : 0;
                uint32_t m = 0u;
                int64_t r0 = 0, r1 = 0;
                if (valid) {
                    m = vload(Fn + w);
                    r0 = __ldg(b.g.rp + w);
                    r1 = __ldg(b.g.rp + w + 1);
                    if (k == 0) b.lm[i] = m;
                }
                // the thread's first two arcs and their frontier masks are loaded once, outside
                // the loop over sources (each source then costs one dependent load of sigma)
                const int64_t ra = r0 + k;
                const int32_t v0 = ra < r1 ? __ldg(b.g.col + ra) : 0;
                const int32_t v1 = ra + QUAD < r1 ? __ldg(b.g.col + ra + QUAD) : 0;
                const uint32_t f0 = ra < r1 ? vload(Fc + v0) & m : 0u;
                const uint32_t f1 = ra + QUAD < r1 ? vload(Fc + v1) & m : 0u;
                uint32_t mm = m;
                while (__any_sync(0xffffffffu, mm != 0u)) {
                    const int j = mm ? __ffs(mm) - 1 : 0;
                    double acc = 0.0;
                    if (mm) {
                        if ((f0 >> j) & 1u) acc += b.s[(int64_t)v0 * BCB_B + j];
                        if ((f1 >> j) & 1u) acc += b.s[(int64_t)v1 * BCB_B + j];
                        for (int64_t r = ra + 2 * QUAD; r < r1; r += QUAD) {
                            const int32_t v = __ldg(b.g.col + r);
                            if ((vload(Fc + v) >> j) & 1u) acc += b.s[(int64_t)v * BCB_B + j];
                        }
                    }
#pragma unroll
                    for (int o = 1; o < QUAD; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
                    if (mm && k == 0) {
                        const double sv = ldexp(acc, -s_kexp[j]);
                        b.s[(int64_t)w * BCB_B + j] = sv;
                        atomicMax(&s_maxe[j], exp_of(sv));
                    }
                    if (mm) mm &= mm - 1;
                }
                if (valid && k == 0) b.V[w] |= m;
            }
            __syncthreads();
            if (threadIdx.x < BCB_B && s_maxe[threadIdx.x] > -100000)
                atomicMax(&b.maxb[(int64_t)(d + 1) * BCB_B + threadIdx.x],
                          (unsigned long long)(s_maxe[threadIdx.x] + EXP_BIAS));
        }
        if (tid == 0) {
            const bool more = !over && top0 > s_ctl[2];
            if (over) c->overflow = 1;
            if (more) {
                c->d = d + 1;
                b.loff[d + 2] = top0;
                c->depth = d + 2;
            } else if (d + 2 <= b.cap + 1) {
                b.loff[d + 2] = b.loff[d + 1];   // empty level `depth` closes the list
            }
            c->par = more ? 1 : 0;               // loop flag
        }
        grid.sync();
        if (tid == 0) { const unsigned long long t1 = gtimer(); c->t_ns[2] += t1 - t_mark; t_mark = t1; }
        if (threadIdx.x == 0) s_ctl[5] = vload(&c->par);
        __syncthreads();
        if (!s_ctl[5]) break;
    }
}

// M_x: masks of level x (three rotating buffers)
__device__ __forceinline__ uint32_t *bcb_M(const BcbView &b, int x) { return b.M + (int64_t)(x % 3) * b.g.n; }

__global__ void __launch_bounds__(BCB_THREADS) k_bcb_backward(BcbView b) {
    cg::grid_group grid = cg::this_grid();
    BcbCtrl *c = b.c;
    __shared__ int s_kexp[BCB_B], s_src[BCB_B];
    __shared__ unsigned long long s_off[5];   // loff[d], loff[d+1], loff[d-2], loff[d-1]; depth
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    if (threadIdx.x < BCB_B) s_src[threadIdx.x] = threadIdx.x < c->nsrc ? c->src[threadIdx.x] : -1;
    if (threadIdx.x == 0) s_off[4] = (unsigned long long)vload(&c->depth);
    __syncthreads();
    const int depth = (int)s_off[4];
    unsigned long long t_mark = gtimer();
    // pre-pass: masks of the level below the deepest
    if (depth - 2 >= 1) {
        uint32_t *Mp = bcb_M(b, depth - 2);
        for (unsigned long long i = b.loff[depth - 2] + tid; i < b.loff[depth - 1]; i += nthr) Mp[b.lv[i]] = b.lm[i];
    }
    grid.sync();
    if (tid == 0) { const unsigned long long t1 = gtimer(); c->t_ns[3] += t1 - t_mark; t_mark = t1; }
    // level d (deepest first): delta_j(v) = 2^-k_j(d) s_j(v) acc_j(v) with acc_j(v) the sum of
    // (1 + delta_j(w)) / s_j(w) over successors w, pushed by level d+1 (zero for the deepest);
    // v pushes (1 + delta_j(v)) / s_j(v) to its predecessors u (j in M_{d-1}(u)); the masks of
    // level d-2 are laid out for the next pass and those of level d cleared
    for (int d = depth - 1; d >= 1; d--) {
        if (threadIdx.x < BCB_B) s_kexp[threadIdx.x] = kexp(b.maxb[(int64_t)d * BCB_B + threadIdx.x]);
        if (threadIdx.x == 0) {
            s_off[0] = b.loff[d];
            s_off[1] = b.loff[d + 1];
            s_off[2] = d >= 3 ? b.loff[d - 2] : 0ull;
            s_off[3] = d >= 3 ? b.loff[d - 1] : 0ull;
        }
        __syncthreads();
        uint32_t *Mp = bcb_M(b, d - 1);   // predecessors' masks
        uint32_t *Mc = bcb_M(b, d);       // this level's masks (read by the pass of d+1): cleared
        uint32_t *Mq = bcb_M(b, d + 1);   // == M_{d-2}: set for the next pass
        {
            const unsigned long long a = s_off[0], e = s_off[1];
            const int k = (int)(tid & (QUAD - 1));
            const bool push = d >= 2;     // level-0 vertices are sources: their delta is not used
            for (unsigned long long i = a + tid / QUAD; i < e; i += nthr / QUAD) {
                const int32_t v = b.lv[i];
                const uint32_t m = b.lm[i];
                const int64_t r1 = __ldg(b.g.rp + v + 1);
                const int64_t ra = __ldg(b.g.rp + v) + k;
                const int32_t u0 = push && ra < r1 ? __ldg(b.g.col + ra) : 0;
                const int32_t u1 = push && ra + QUAD < r1 ? __ldg(b.g.col + ra + QUAD) : 0;
                const uint32_t g0 = push && ra < r1 ? vload(Mp + u0) & m : 0u;
                const uint32_t g1 = push && ra + QUAD < r1 ? vload(Mp + u1) & m : 0u;
                double contrib = 0.0;
                for (uint32_t mm = m; mm; mm &= mm - 1) {   // sources ascending: fixed order
                    const int j = __ffs(mm) - 1;
                    const int64_t q = (int64_t)v * BCB_B + j;
                    const double sv = __ldcg(b.s + q);
                    const double dv = ldexp(sv * __ldcg(b.delta + q), -s_kexp[j]);
                    if (v != s_src[j]) contrib += dv;
                    if (push) {
                        const double t = (1.0 + dv) / sv;
                        if ((g0 >> j) & 1u) atomicAdd(b.delta + (int64_t)u0 * BCB_B + j, t);
                        if ((g1 >> j) & 1u) atomicAdd(b.delta + (int64_t)u1 * BCB_B + j, t);
                        for (int64_t r = ra + 2 * QUAD; r < r1; r += QUAD) {
                            const int32_t u = __ldg(b.g.col + r);
                            if ((vload(Mp + u) >> j) & 1u) atomicAdd(b.delta + (int64_t)u * BCB_B + j, t);
                        }
                    }
                }
                if (k == 0) {
                    b.bc[v] += contrib;
                    Mc[v] = 0u;
                }
            }
            const unsigned long long a2 = s_off[2], e2 = s_off[3];
            for (unsigned long long i = a2 + tid; i < e2; i += nthr) Mq[b.lv[i]] = b.lm[i];
        }
        grid.sync();
        if (tid == 0) { const unsigned long long t1 = gtimer(); c->t_ns[4] += t1 - t_mark; t_mark = t1; }
    }
}

// reset the per-batch masks and delta accumulators for the next batch (entries of every level;
// whole arrays when the entries outnumber the vertices; full 32-B sectors either way: a partial
// sector store would make L2 fetch the sector from HBM first)
__global__ void k_bcb_reset(BcbView b) {
    BcbCtrl *c = b.c;
    unsigned long long top = c->ltop;
    if (top > (unsigned long long)b.lcap) top = b.lcap;
    const int64_t n = b.g.n;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (top > (unsigned long long)n / 2) {
        // many entries (a vertex recurs once per source): zeroing the arrays whole is cheaper
        // than scattering per entry
        uint32_t *arr[3] = {b.V, b.F, b.M};
        const int64_t len[3] = {n, 3 * n, 3 * n};
        for (int a = 0; a < 3; a++) {
            uint32_t *p = arr[a];
            const int64_t nv = len[a] / 4;   // cudaMalloc'd: 256-B aligned
            for (int64_t i = t0; i < nv; i += stride) reinterpret_cast<uint4 *>(p)[i] = make_uint4(0, 0, 0, 0);
            for (int64_t i = nv * 4 + t0; i < len[a]; i += stride) p[i] = 0u;
        }
        const int64_t nd = n * (BCB_B / 2);   // delta accumulators: 16 B per store
        for (int64_t i = t0; i < nd; i += stride) reinterpret_cast<uint4 *>(b.delta)[i] = make_uint4(0, 0, 0, 0);
        top = 0;
    }
    for (unsigned long long i = t0; i < top; i += stride) {
        const int32_t v = b.lv[i];
        b.V[v] = 0u;
        b.F[v] = 0u;
        b.F[n + v] = 0u;
        b.F[2 * n + v] = 0u;
        b.M[v] = 0u;
        b.M[n + v] = 0u;
        b.M[2 * n + v] = 0u;
        uint4 *row = reinterpret_cast<uint4 *>(b.delta + (int64_t)v * BCB_B);   // delta accumulators
#pragma unroll
        for (int q = 0; q < BCB_B / 2; q++) row[q] = make_uint4(0, 0, 0, 0);
    }
    int64_t levels = (int64_t)c->depth + 1;
    if (levels > b.cap + 1) levels = b.cap + 1;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < levels * BCB_B; i += stride) b.maxb[i] = 0ull;
}

static BcbView view_of(const BcbLaunch &L) {
    BcbView b;
    b.g = L.g;
    b.F = L.F;
    b.V = L.V;
    b.M = L.M;
    b.VB = L.VB;
    b.VS = L.VS;
    b.s = L.s;
    b.delta = L.delta;
    b.lv = L.lv;
    b.lm = L.lm;
    b.loff = L.loff;
    b.maxb = L.maxb;
    b.c = L.c;
    b.cap = L.cap;
    b.lcap = L.lcap;
    b.bc = L.bc;
    return b;
}

// One batch: init, cooperative forward, cooperative backward, reset (stream-ordered).
cudaError_t bcb_run_batch(const BcbLaunch &L, cudaStream_t s) {
    static int coop_blocks = 0;
    if (!coop_blocks) {
        int per_sm = 0, nsm = 0, dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_bcb_forward, BCB_THREADS, 0);
        int per_sm_b = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm_b, k_bcb_backward, BCB_THREADS, 0);
        per_sm = per_sm < per_sm_b ? per_sm : per_sm_b;
        if (per_sm > SG_BCB_PER_SM) per_sm = SG_BCB_PER_SM;
        coop_blocks = nsm * (per_sm > 0 ? per_sm : 1);
    }
    BcbView b = view_of(L);
    note_launch();
    k_bcb_init<<<1, 256, 0, s>>>(b);
    void *args[] = {&b};
    note_launch();
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_bcb_forward, coop_blocks, BCB_THREADS, args, 0, s);
    if (e != cudaSuccess) return e;
    note_launch();
    e = cudaLaunchCooperativeKernel((const void *)k_bcb_backward, coop_blocks, BCB_THREADS, args, 0, s);
    if (e != cudaSuccess) return e;
    note_launch();
    k_bcb_reset<<<num_sms() * 8, 256, 0, s>>>(b);
    return cudaGetLastError();
}

}  // namespace sg
