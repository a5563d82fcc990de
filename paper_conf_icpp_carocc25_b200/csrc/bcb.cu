// bcb.cu — source-batched Brandes BC (algorithm PAPER.md:161 §3.4).
//
// Up to 32 sources advance in lock-step, one bit per source in a per-vertex 32-bit mask (lane j
// of a warp = source j): the frontier of level d is a list L_d of (vertex, mask) entries, the
// per-source path counts sigma live in [n][32] doubles.  A high-diameter graph (config 5: ~10^4
// levels of a few thousand vertices each) then does 32 sources' work per superstep, and each
// direction (forward / backward) is ONE persistent cooperative kernel whose supersteps are
// separated by grid-wide barriers (two per level) instead of kernel launches.
//
// Forward level d -> d+1:
//   A  expand: for (v, m) in L_d, w in N(v): nm = m & ~V[w]; if nm: F_{d+1}[w] |= nm (first
//      setter appends w to L_{d+1});  clear F_{d-1} for the entries of L_{d-1}    | grid sync
//   B  sigma (warp per new entry, lane j): if j in F_{d+1}[w]:
//        s[w][j] = 2^-k_j(d) * sum_{v in N(w), j in F_d[v]} s[v][j];  V[w] |= F_{d+1}[w]
//      per-source max of the level -> k_j(d+1) = floor(log2 max); control step   | grid sync
//   (three frontier-mask buffers rotate: F_{d-1} is cleared while F_d / F_{d+1} are live)
// Stored s is sigma scaled by 2^-G_j(level) with G_j(L+1) = G_j(L) + k_j(L): exact power-of-two
// scaling (reading C20 / R5), every level's max in [1, 2).
// Backward level d = D-1 .. 1:
//   A  M_{(d+1)%2}[w] = mask of w in L_{d+1}                                      | grid sync
//   B  for (v, m) in L_d (warp; lane j in m):
//        delta[v][j] = 2^-k_j(d) * s[v][j] * sum_{w in N(v), j in M[w]} (1 + delta[w][j]) / s[w][j]
//      bc[v] += sum over lanes (fixed shuffle order: deterministic); clear M_{d%2} of L_{d+2}
//                                                                                  | grid sync
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

struct BcbView {
    GraphView g;
    uint32_t *F;          // [3][n] frontier masks (rotating)
    uint32_t *V;          // [n] visited masks
    uint32_t *M;          // [2][n] backward: masks of level d+1
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
    BcbCtrl *c = b.c;
    const int64_t n = b.g.n;
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    for (;;) {
        const int d = vload(&c->d);
        uint32_t *Fc = b.F + (int64_t)(d % 3) * n;            // masks of L_d
        uint32_t *Fn = b.F + (int64_t)((d + 1) % 3) * n;      // masks of L_{d+1} (being built)
        uint32_t *Fo = b.F + (int64_t)((d + 2) % 3) * n;      // masks of L_{d-1} (to clear)
        // ---- A: expand L_d; clear L_{d-1}'s masks
        {
            const unsigned long long a = vload(&b.loff[d]), e = vload(&b.loff[d + 1]);
            // warp-uniform loop bounds so list appends can be aggregated: one atomicAdd on the
            // list tail per warp and neighbour step (a per-vertex atomic on one address
            // serialises ~10^5 operations per level in L2)
            const int lane = lane_id();
            for (unsigned long long i0 = a + (tid & ~31ll); i0 < e; i0 += nthr) {
                const unsigned long long i = i0 + lane;
                int32_t v = 0;
                uint32_t m = 0;
                int64_t r0 = 0, r1 = 0;
                if (i < e) {
                    v = b.lv[i];
                    m = b.lm[i];
                    r0 = __ldg(b.g.rp + v);
                    r1 = __ldg(b.g.rp + v + 1);
                }
                int64_t dmax = r1 - r0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    const int64_t y = __shfl_xor_sync(0xffffffffu, dmax, o);
                    dmax = y > dmax ? y : dmax;
                }
                for (int64_t k = 0; k < dmax; k++) {
                    bool app = false;
                    int32_t w = 0;
                    if (r0 + k < r1) {
                        w = __ldg(b.g.col + r0 + k);
                        const uint32_t nm = m & ~vload(b.V + w);
                        if (nm) app = atomicOr(Fn + w, nm) == 0u;
                    }
                    const uint32_t am = __ballot_sync(0xffffffffu, app);
                    if (am) {
                        unsigned long long base = 0;
                        if (lane == __ffs(am) - 1) base = atomicAdd(&c->ltop, (unsigned long long)__popc(am));
                        base = __shfl_sync(0xffffffffu, base, __ffs(am) - 1);
                        if (app) {
                            const unsigned long long pos = base + __popc(am & ((1u << lane) - 1u));
                            if (pos < (unsigned long long)b.lcap) b.lv[pos] = w;
                        }
                    }
                }
            }
            if (d >= 1) {
                const unsigned long long a0 = vload(&b.loff[d - 1]), e0 = vload(&b.loff[d]);
                for (unsigned long long i = a0 + tid; i < e0; i += nthr) Fo[b.lv[i]] = 0u;
            }
        }
        if (threadIdx.x < BCB_B) s_maxe[threadIdx.x] = -1000000;
        grid.sync();
        // ---- B: sigma of the new level (thread per entry, loop over its sources); control step
        const unsigned long long top0 = vload(&c->ltop);
        const bool over = top0 > (unsigned long long)b.lcap || d + 2 > b.cap;
        {
            const unsigned long long a = vload(&b.loff[d + 1]);
            const unsigned long long e = over ? a : top0;
            if (threadIdx.x < BCB_B) s_kexp[threadIdx.x] = kexp(vload(&b.maxb[(int64_t)d * BCB_B + threadIdx.x]));
            __syncthreads();
            for (unsigned long long i = a + tid; i < e; i += nthr) {
                const int32_t w = b.lv[i];
                const uint32_t m = vload(Fn + w);
                const int64_t r0 = __ldg(b.g.rp + w), r1 = __ldg(b.g.rp + w + 1);
                uint32_t mm = m;
                while (mm) {
                    const int j = __ffs(mm) - 1;
                    mm &= mm - 1;
                    double acc = 0.0;
                    for (int64_t r = r0; r < r1; r++) {
                        const int32_t v = __ldg(b.g.col + r);
                        if ((vload(Fc + v) >> j) & 1u) acc += b.s[(int64_t)v * BCB_B + j];
                    }
                    const double sv = ldexp(acc, -s_kexp[j]);
                    b.s[(int64_t)w * BCB_B + j] = sv;
                    atomicMax(&s_maxe[j], exp_of(sv));
                }
                b.lm[i] = m;
                b.V[w] |= m;
            }
            __syncthreads();
            if (threadIdx.x < BCB_B && s_maxe[threadIdx.x] > -100000)
                atomicMax(&b.maxb[(int64_t)(d + 1) * BCB_B + threadIdx.x],
                          (unsigned long long)(s_maxe[threadIdx.x] + EXP_BIAS));
        }
        if (tid == 0) {
            const bool more = !over && top0 > b.loff[d + 1];
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
        if (!vload(&c->par)) break;
    }
}

__global__ void __launch_bounds__(BCB_THREADS) k_bcb_backward(BcbView b) {
    cg::grid_group grid = cg::this_grid();
    BcbCtrl *c = b.c;
    const int64_t n = b.g.n;
    __shared__ int s_kexp[BCB_B], s_src[BCB_B];
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    if (threadIdx.x < BCB_B) s_src[threadIdx.x] = threadIdx.x < c->nsrc ? c->src[threadIdx.x] : -1;
    __syncthreads();
    // the deepest level has no successors: delta = 0 there, written by its own pass
    for (int d = vload(&c->depth) - 1; d >= 1; d--) {
        uint32_t *Mn = b.M + (int64_t)((d + 1) & 1) * n;   // masks of L_{d+1}
        uint32_t *Mo = b.M + (int64_t)(d & 1) * n;         // held L_{d+2}: cleared below
        {
            const unsigned long long a = b.loff[d + 1], e = b.loff[d + 2];
            for (unsigned long long i = a + tid; i < e; i += nthr) Mn[b.lv[i]] = b.lm[i];
        }
        grid.sync();
        {
            const unsigned long long a = b.loff[d], e = b.loff[d + 1];
            if (threadIdx.x < BCB_B) s_kexp[threadIdx.x] = kexp(b.maxb[(int64_t)d * BCB_B + threadIdx.x]);
            __syncthreads();
            for (unsigned long long i = a + tid; i < e; i += nthr) {
                const int32_t v = b.lv[i];
                const uint32_t m = b.lm[i];
                const int64_t r0 = __ldg(b.g.rp + v), r1 = __ldg(b.g.rp + v + 1);
                double contrib = 0.0;
                uint32_t mm = m;
                while (mm) {   // sources in ascending order: deterministic sum
                    const int j = __ffs(mm) - 1;
                    mm &= mm - 1;
                    double acc = 0.0;
                    for (int64_t r = r0; r < r1; r++) {
                        const int32_t w = __ldg(b.g.col + r);
                        if ((vload(Mn + w) >> j) & 1u) {
                            const int64_t q = (int64_t)w * BCB_B + j;
                            acc += (1.0 + b.delta[q]) / b.s[q];
                        }
                    }
                    const double dv = ldexp(b.s[(int64_t)v * BCB_B + j] * acc, -s_kexp[j]);
                    b.delta[(int64_t)v * BCB_B + j] = dv;
                    if (v != s_src[j]) contrib += dv;
                }
                if (m) b.bc[v] += contrib;
            }
            if (d + 2 <= vload(&c->depth)) {
                const unsigned long long a2 = b.loff[d + 2], e2 = b.loff[d + 3];
                for (unsigned long long i = a2 + tid; i < e2; i += nthr) Mo[b.lv[i]] = 0u;
            }
        }
        grid.sync();
    }
}

// reset the per-batch state for the next batch (entries of every level)
__global__ void k_bcb_reset(BcbView b) {
    BcbCtrl *c = b.c;
    unsigned long long top = c->ltop;
    if (top > (unsigned long long)b.lcap) top = b.lcap;
    const int64_t n = b.g.n;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (unsigned long long i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < top; i += stride) {
        const int32_t v = b.lv[i];
        b.V[v] = 0u;
        b.F[v] = 0u;
        b.F[n + v] = 0u;
        b.F[2 * n + v] = 0u;
        b.M[v] = 0u;
        b.M[n + v] = 0u;
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
    k_bcb_reset<<<148 * 8, 256, 0, s>>>(b);
    return cudaGetLastError();
}

}  // namespace sg
