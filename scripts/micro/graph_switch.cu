// graph_switch.cu — per-superstep cost of the BFS graph's control structure with KB kernels of G
// CTAs per superstep body (the last one's last CTA sets the next superstep's conditionals, as
// bfs_finish / bfs_decide do), for: (0) WHILE { Q parts x [IF push, IF pull] } (Q = 2: the current
// graph, Q = 4: unrolled), (1) WHILE { Q parts x SWITCH(push, pull) }, (2) a straight line of KB
// kernels per superstep (no conditional: the floor).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o graph_switch graph_switch.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s (line %d)\n", #x, cudaGetErrorString(e), __LINE__); return 1; } } while (0)

struct Ctl {
    int iter, n, mode, Q;
    unsigned int done;
    unsigned long long hl;
    unsigned long long h[4][2];   // per part: IF push / IF pull handles, or h[q][0] = SWITCH handle
};
__global__ void k_plain(Ctl *) {}
__global__ void k_last(Ctl *c, int part) {
    __shared__ bool last;
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(&c->done, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (last && threadIdx.x == 0) {
        c->done = 0;
        const int i = ++c->iter;
        const bool go = i < c->n;
        const int np = (part + 1) % c->Q;
        const int kind = i & 1;   // alternate push / pull
        if (c->mode == 0) {
            for (int k = 0; k < 2; k++) cudaGraphSetConditional((cudaGraphConditionalHandle)c->h[np][k], go && k == kind);
            for (int k = 0; k < 2; k++) cudaGraphSetConditional((cudaGraphConditionalHandle)c->h[part][k], 0);
        } else {
            cudaGraphSetConditional((cudaGraphConditionalHandle)c->h[np][0], go ? kind : 2);
            cudaGraphSetConditional((cudaGraphConditionalHandle)c->h[part][0], 2);
        }
        if (np == 0 || !go) cudaGraphSetConditional((cudaGraphConditionalHandle)c->hl, go);
    }
}
static cudaError_t add_body(cudaGraph_t bb, Ctl *c, int part, int KB, int G) {
    cudaGraphNode_t prev = nullptr;
    for (int j = 0; j < KB; j++) {
        int hp = part;
        void *args[] = {&c, &hp};
        cudaKernelNodeParams kp = {};
        kp.func = j == KB - 1 ? (void *)k_last : (void *)k_plain;
        kp.gridDim = dim3(G);
        kp.blockDim = dim3(256);
        kp.kernelParams = args;
        cudaGraphNode_t kn;
        cudaError_t e = cudaGraphAddKernelNode(&kn, bb, prev ? &prev : nullptr, prev ? 1 : 0, &kp);
        if (e != cudaSuccess) return e;
        prev = kn;
    }
    return cudaSuccess;
}
int run(int mode, int Q, int KB, int G, int iters) {
    Ctl *c;
    CK(cudaMallocManaged(&c, sizeof(Ctl)));
    memset(c, 0, sizeof(Ctl));
    c->n = iters;
    c->mode = mode;
    c->Q = Q;
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaStream_t s;
    CK(cudaStreamCreate(&s));
    if (mode == 2) {
        for (int i = 0; i < iters; i++) CK(add_body(g, c, 0, KB, G));   // (independent chains: serialised below)
        cudaGraphDestroy(g);
        CK(cudaGraphCreate(&g, 0));
        CK(cudaStreamBeginCaptureToGraph(s, g, nullptr, nullptr, 0, cudaStreamCaptureModeGlobal));
        for (int i = 0; i < iters; i++)
            for (int j = 0; j < KB; j++) k_plain<<<G, 256, 0, s>>>(c);
        CK(cudaStreamEndCapture(s, &g));
    } else {
        cudaGraphConditionalHandle hl;
        CK(cudaGraphConditionalHandleCreate(&hl, g, 1, cudaGraphCondAssignDefault));
        c->hl = (unsigned long long)hl;
        for (int q = 0; q < Q; q++)
            for (int k = 0; k < (mode == 0 ? 2 : 1); k++) {
                cudaGraphConditionalHandle h;
                const unsigned dflt = mode == 0 ? (q == 0 && k == 0) : (q == 0 ? 0 : 2);
                CK(cudaGraphConditionalHandleCreate(&h, g, dflt, cudaGraphCondAssignDefault));
                c->h[q][k] = (unsigned long long)h;
            }
        cudaGraphNodeParams wp = {};
        wp.type = cudaGraphNodeTypeConditional;
        wp.conditional.handle = hl;
        wp.conditional.type = cudaGraphCondTypeWhile;
        wp.conditional.size = 1;
        cudaGraphNode_t wn;
        CK(cudaGraphAddNode(&wn, g, nullptr, 0, &wp));
        cudaGraph_t body = wp.conditional.phGraph_out[0];
        std::vector<cudaGraphNode_t> deps;
        for (int q = 0; q < Q; q++) {
            std::vector<cudaGraphNode_t> nd;
            if (mode == 0) {
                for (int k = 0; k < 2; k++) {
                    cudaGraphNodeParams ip = {};
                    ip.type = cudaGraphNodeTypeConditional;
                    ip.conditional.handle = (cudaGraphConditionalHandle)c->h[q][k];
                    ip.conditional.type = cudaGraphCondTypeIf;
                    ip.conditional.size = 1;
                    cudaGraphNode_t n;
                    CK(cudaGraphAddNode(&n, body, deps.data(), deps.size(), &ip));
                    CK(add_body(ip.conditional.phGraph_out[0], c, q, KB, G));
                    nd.push_back(n);
                }
            } else {
                cudaGraphNodeParams ip = {};
                ip.type = cudaGraphNodeTypeConditional;
                ip.conditional.handle = (cudaGraphConditionalHandle)c->h[q][0];
                ip.conditional.type = cudaGraphCondTypeSwitch;
                ip.conditional.size = 2;
                cudaGraphNode_t n;
                CK(cudaGraphAddNode(&n, body, deps.data(), deps.size(), &ip));
                for (int k = 0; k < 2; k++) CK(add_body(ip.conditional.phGraph_out[k], c, q, KB, G));
                nd.push_back(n);
            }
            deps = nd;
        }
    }
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
        c->iter = 0;
        c->done = 0;
        CK(cudaDeviceSynchronize());
        cudaEventRecord(a, s);
        CK(cudaGraphLaunch(ex, s));
        cudaEventRecord(b, s);
        CK(cudaStreamSynchronize(s));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r && ms < best) best = ms;
    }
    const char *nm[] = {"WHILE + IF pairs", "WHILE + SWITCH", "straight line"};
    printf("%-18s parts %d, kernels/superstep %d, grid %4d: %6.2f us per superstep (iter %d)\n", nm[mode], Q, KB, G,
           1000.f * best / iters, c->iter);
    cudaGraphExecDestroy(ex);
    cudaGraphDestroy(g);
    cudaFree(c);
    return 0;
}
int main() {
    for (int KB : {1, 4}) {
        run(2, 1, KB, 592, 96);
        run(0, 2, KB, 592, 96);
        run(0, 4, KB, 592, 96);
        run(1, 2, KB, 592, 96);
        run(1, 4, KB, 592, 96);
    }
    return 0;
}
