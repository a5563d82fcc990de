// Cost of CUDA-graph control structures on this GPU: per-iteration time of a WHILE loop whose
// body holds (A) K plain kernel nodes, (B) K IF nodes each holding one kernel (condition true),
// (C) K IF nodes with condition false + one kernel.  Build: nvcc -gencode arch=compute_100a,code=sm_100a
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__global__ void k_work(int *p, int blocks_work) { if (threadIdx.x == 0 && blocks_work) atomicAdd(p + 1, 1); }
__global__ void k_ctl(int *iter, int n, cudaGraphConditionalHandle hl, cudaGraphConditionalHandle *hs, int nh, int val) {
    if (threadIdx.x || blockIdx.x) return;
    int i = ++*iter;
    for (int k = 0; k < nh; k++) cudaGraphSetConditional(hs[k], val);
    cudaGraphSetConditional(hl, i < n);
}

int run(int mode, int K, int iters, int grid) {
    int *d; CK(cudaMalloc(&d, 64)); CK(cudaMemset(d, 0, 64));
    cudaGraphConditionalHandle *dh; CK(cudaMalloc(&dh, sizeof(cudaGraphConditionalHandle) * 16));
    cudaGraph_t g; CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle hl; CK(cudaGraphConditionalHandleCreate(&hl, g, 1, cudaGraphCondAssignDefault));
    std::vector<cudaGraphConditionalHandle> hs(K);
    if (mode) for (int k = 0; k < K; k++) CK(cudaGraphConditionalHandleCreate(&hs[k], g, 0, cudaGraphCondAssignDefault));
    if (mode) CK(cudaMemcpy(dh, hs.data(), sizeof(cudaGraphConditionalHandle) * K, cudaMemcpyHostToDevice));
    cudaGraphNodeParams wp = {}; wp.type = cudaGraphNodeTypeConditional; wp.conditional.handle = hl;
    wp.conditional.type = cudaGraphCondTypeWhile; wp.conditional.size = 1;
    cudaGraphNode_t wn; CK(cudaGraphAddNode(&wn, g, nullptr, 0, &wp));
    cudaGraph_t body = wp.conditional.phGraph_out[0];
    int nv = iters, one = 1;
    void *ka[] = {&d, &one};
    cudaKernelNodeParams kp = {}; kp.func = (void *)k_work; kp.gridDim = dim3(grid); kp.blockDim = dim3(256); kp.kernelParams = ka;
    int nh = mode ? K : 0, val = mode == 1 ? 1 : 0;
    int *dit = d;
    void *ca[] = {&dit, &nv, &hl, &dh, &nh, &val};
    cudaKernelNodeParams cp = {}; cp.func = (void *)k_ctl; cp.gridDim = dim3(1); cp.blockDim = dim3(32); cp.kernelParams = ca;
    cudaGraphNode_t prev; CK(cudaGraphAddKernelNode(&prev, body, nullptr, 0, &cp));
    for (int k = 0; k < K; k++) {
        cudaGraphNode_t n;
        if (mode == 0) { CK(cudaGraphAddKernelNode(&n, body, &prev, 1, &kp)); }
        else {
            cudaGraphNodeParams ip = {}; ip.type = cudaGraphNodeTypeConditional; ip.conditional.handle = hs[k];
            ip.conditional.type = cudaGraphCondTypeIf; ip.conditional.size = 1;
            CK(cudaGraphAddNode(&n, body, &prev, 1, &ip));
            cudaGraphNode_t kn; CK(cudaGraphAddKernelNode(&kn, ip.conditional.phGraph_out[0], nullptr, 0, &kp));
        }
        prev = n;
    }
    cudaGraphExec_t ex; CK(cudaGraphInstantiate(&ex, g, 0));
    cudaStream_t s; CK(cudaStreamCreate(&s));
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int r = 0; r < 3; r++) { CK(cudaMemsetAsync(d, 0, 4, s)); CK(cudaGraphLaunch(ex, s)); }
    CK(cudaStreamSynchronize(s));
    CK(cudaMemsetAsync(d, 0, 4, s));
    cudaEventRecord(a, s); CK(cudaGraphLaunch(ex, s)); cudaEventRecord(b, s); CK(cudaStreamSynchronize(s));
    float ms; cudaEventElapsedTime(&ms, a, b);
    const char *nm[] = {"K plain kernels", "K IF(true)+kernel", "K IF(false)"};
    printf("mode %-18s K=%d grid=%4d: %.2f us per iteration (%.2f us per node)\n", nm[mode], K, grid, 1000.f * ms / iters,
           1000.f * ms / iters / (K + 1));
    return 0;
}
int main() {
    for (int grid : {1, 592})
        for (int K : {1, 4})
            for (int m = 0; m < 3; m++) run(m, K, 2000, grid);
    return 0;
}
