// filter.cu — filter::inplace / filter::external and compute::execute over a 2LB frontier
// (Table 2; §3.1; layer-2 maintenance on removal P:253 §4.3).
//
// The paper's functors are user C++ lambdas; across a C ABI they become a predicate / operation
// code plus parameters (sygraph.h SG_PRED_* / SG_OP_*).  One thread per layer-1 word: the word's
// active bits are tested, the result word is written and its layer-2 bit is set or reset
// (a word that becomes 0 clears its summary bit).
#include "common.cuh"
#include "kernels.h"

namespace sg {

struct PredArgs {
    int pred;
    const void *array;      // per-vertex values (uint32 / int32 / double) or bitmap
    double a, b;            // scalar parameters
};

__device__ __forceinline__ bool eval_pred(const GraphView &g, const PredArgs &p, int64_t v) {
    switch (p.pred) {
        case 0: {   // SG_PRED_DEGREE_RANGE: a <= deg(v) < b
            const double d = (double)(g.rp[v + 1] - g.rp[v]);
            return d >= p.a && d < p.b;
        }
        case 1: {   // SG_PRED_U32_RANGE: a <= array_u32[v] < b
            const double x = (double)reinterpret_cast<const uint32_t *>(p.array)[v];
            return x >= p.a && x < p.b;
        }
        case 2: {   // SG_PRED_I32_RANGE
            const double x = (double)reinterpret_cast<const int32_t *>(p.array)[v];
            return x >= p.a && x < p.b;
        }
        case 3: {   // SG_PRED_F64_RANGE
            const double x = reinterpret_cast<const double *>(p.array)[v];
            return x >= p.a && x < p.b;
        }
        case 4:     // SG_PRED_IN_BITMAP: bit v of a layer-1-shaped bitmap
            return (reinterpret_cast<const uint64_t *>(p.array)[v >> 6] >> (v & 63)) & 1ull;
        default:
            return false;
    }
}

// out_bits/out_summ == in: in place (removal).  Otherwise external: out |= passing elements.
__global__ void k_filter(GraphView g, const uint64_t *__restrict__ in_bits, uint64_t *out_bits, uint64_t *out_summ,
                         PredArgs p, int inplace) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < g.nw1; w += stride) {
        const uint64_t x = in_bits[w];
        uint64_t keep = 0;
        uint64_t y = x;
        while (y) {
            const int b = __ffsll((long long)y) - 1;
            y &= y - 1;
            if (eval_pred(g, p, w * 64 + b)) keep |= 1ull << b;
        }
        if (inplace) {
            if (keep != x) {
                out_bits[w] = keep;
                if (keep == 0ull) atomicAnd(reinterpret_cast<unsigned long long *>(out_summ + (w >> 6)),
                                            ~(1ull << (w & 63)));
            }
        } else if (keep) {
            const unsigned long long old = atomic_or_u64(out_bits + w, keep);
            if (old == 0ull) atomic_or_u64(out_summ + (w >> 6), 1ull << (w & 63));
        }
    }
}

struct OpArgs {
    int op;
    void *array;
    double value;
};

// compute::execute: apply an operation to every active vertex
__global__ void k_compute(GraphView g, const uint64_t *__restrict__ bits, OpArgs o) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < g.nw1; w += stride) {
        uint64_t y = bits[w];
        while (y) {
            const int b = __ffsll((long long)y) - 1;
            y &= y - 1;
            const int64_t v = w * 64 + b;
            switch (o.op) {
                case 0: reinterpret_cast<uint32_t *>(o.array)[v] = (uint32_t)o.value; break;   // SG_OP_SET_U32
                case 1: reinterpret_cast<int32_t *>(o.array)[v] = (int32_t)o.value; break;     // SG_OP_SET_I32
                case 2: reinterpret_cast<double *>(o.array)[v] = o.value; break;               // SG_OP_SET_F64
                case 3: reinterpret_cast<uint32_t *>(o.array)[v] += (uint32_t)o.value; break;  // SG_OP_ADD_U32
                case 4: reinterpret_cast<double *>(o.array)[v] += o.value; break;              // SG_OP_ADD_F64
                default: break;
            }
        }
    }
}

// min over the active vertices of a uint32 array (delta-stepping: far pile's smallest distance)
__global__ void k_min_over_bits(GraphView g, const uint64_t *__restrict__ bits, const uint32_t *__restrict__ a,
                                unsigned int *out) {
    unsigned int m = 0xFFFFFFFFu;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < g.nw1; w += stride) {
        uint64_t y = bits[w];
        while (y) {
            const int b = __ffsll((long long)y) - 1;
            y &= y - 1;
            m = min(m, a[w * 64 + b]);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
    if (lane_id() == 0 && m != 0xFFFFFFFFu) atomicMin(out, m);
}

static int grid_for(int64_t items) {
    int64_t b = (items + 255) / 256;
    if (b > num_sms() * 8) b = num_sms() * 8;
    return (int)(b < 1 ? 1 : b);
}

void launch_filter(const GraphView &g, const uint64_t *in_bits, uint64_t *out_bits, uint64_t *out_summ, int pred,
                   const void *array, double a, double b, int inplace, cudaStream_t s) {
    PredArgs p{pred, array, a, b};
    note_launch();
    k_filter<<<grid_for(g.nw1), 256, 0, s>>>(g, in_bits, out_bits, out_summ, p, inplace);
}

void launch_min_over_bits(const GraphView &g, const uint64_t *bits, const uint32_t *a, unsigned int *out,
                          cudaStream_t s) {
    note_launch();
    k_min_over_bits<<<grid_for(g.nw1), 256, 0, s>>>(g, bits, a, out);
}

void launch_compute(const GraphView &g, const uint64_t *bits, int op, void *array, double value, cudaStream_t s) {
    OpArgs o{op, array, value};
    note_launch();
    k_compute<<<grid_for(g.nw1), 256, 0, s>>>(g, bits, o);
}

}  // namespace sg
