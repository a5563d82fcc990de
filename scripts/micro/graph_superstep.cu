// graph_superstep.cu — per-superstep cost of the BFS graph's control structure, isolated:
// WHILE { half 0: IF_0..IF_{F-1} | half 1: IF_0..IF_{F-1} }, one IF per half taken; its body is
// KB kernels of G CTAs, the last of which (last CTA to finish, atomic counter) sets the next
// half's handles and the loop handle — as bfs_finish / bfs_decide do.  Prints us per superstep.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o graph_superstep.bin graph_superstep.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s (line %d)\n", #x, cudaGetErrorString(e), __LINE__); return 1; } } while (0)

struct Ctl {
    int iter, n;
    unsigned int done;
    unsigned long long hl;
    unsigned long long h[2][4];
    int fence_sys;
};

__global__ void k_plain(Ctl *) {}
__global__ void k_last(Ctl *c, int half) {
    __shared__ bool last;
    if (threadIdx.x == 0) {
        if (c->fence_sys) __threadfence_system(); else __threadfence();
        last = atomicAdd(&c->done, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (last && threadIdx.x == 0) {
        c->done = 0;
        const int i = ++c->iter;
        const bool go = i < c->n;
        const int nh = half ^ 1;
        for (int k = 0; k < 4; k++)
            if (c->h[nh][k]) cudaGraphSetConditional((cudaGraphConditionalHandle)c->h[nh][k], go && k == 0);
        cudaGraphSetConditional((cudaGraphConditionalHandle)c->hl, go);
    }
}

int run(int F, int KB, int G, int fsys, int iters) {
    Ctl *c;
    CK(cudaMallocManaged(&c, sizeof(Ctl)));
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle hl, h[2][4];
    CK(cudaGraphConditionalHandleCreate(&hl, g, 1, cudaGraphCondAssignDefault));
    for (int b = 0; b < 2; b++)
        for (int k = 0; k < F; k++) CK(cudaGraphConditionalHandleCreate(&h[b][k], g, b == 0 && k == 0, cudaGraphCondAssignDefault));
    memset(c, 0, sizeof(Ctl));
    c->n = iters;
    c->hl = (unsigned long long)hl;
    c->fence_sys = fsys;
    for (int b = 0; b < 2; b++)
        for (int k = 0; k < F; k++) c->h[b][k] = (unsigned long long)h[b][k];
    cudaGraphNodeParams wp = {};
    wp.type = cudaGraphNodeTypeConditional;
    wp.conditional.handle = hl;
    wp.conditional.type = cudaGraphCondTypeWhile;
    wp.conditional.size = 1;
    cudaGraphNode_t wn;
    CK(cudaGraphAddNode(&wn, g, nullptr, 0, &wp));
    cudaGraph_t body = wp.conditional.phGraph_out[0];
    std::vector<cudaGraphNode_t> deps;
    for (int half = 0; half < 2; half++) {
        std::vector<cudaGraphNode_t> nd;
        for (int k = 0; k < F; k++) {
            cudaGraphNodeParams ip = {};
            ip.type = cudaGraphNodeTypeConditional;
            ip.conditional.handle = h[half][k];
            ip.conditional.type = cudaGraphCondTypeIf;
            ip.conditional.size = 1;
            cudaGraphNode_t n;
            CK(cudaGraphAddNode(&n, body, deps.data(), deps.size(), &ip));
            cudaGraph_t bb = ip.conditional.phGraph_out[0];
            cudaGraphNode_t prev = nullptr;
            int hh = half;
            for (int j = 0; j < KB; j++) {
                void *args[] = {&c, &hh};
                cudaKernelNodeParams kp = {};
                kp.func = j == KB - 1 ? (void *)k_last : (void *)k_plain;
                kp.gridDim = dim3(G);
                kp.blockDim = dim3(256);
                kp.kernelParams = args;
                cudaGraphNode_t kn;
                CK(cudaGraphAddKernelNode(&kn, bb, prev ? &prev : nullptr, prev ? 1 : 0, &kp));
                prev = kn;
            }
            nd.push_back(n);
        }
        deps = nd;
    }
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    cudaStream_t s;
    CK(cudaStreamCreate(&s));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < 4; r++) {
        c->iter = 0;
        CK(cudaDeviceSynchronize());
        cudaEventRecord(a, s);
        CK(cudaGraphLaunch(ex, s));
        cudaEventRecord(b, s);
        CK(cudaStreamSynchronize(s));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r && ms < best) best = ms;
    }
    printf("IFs/half %d, kernels/body %d, grid %4d, fence %s: %.2f us per superstep\n", F, KB, G, fsys ? "sys" : "gpu",
           1000.f * best / iters);
    cudaGraphExecDestroy(ex);
    cudaGraphDestroy(g);
    cudaFree(c);
    return 0;
}

int main() {
    for (int F : {1, 3})
        for (int KB : {1, 4})
            for (int G : {1, 148, 592}) run(F, KB, G, 0, 400);
    run(3, 1, 148, 1, 400);
    return 0;
}
