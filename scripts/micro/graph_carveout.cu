// graph_carveout.cu — cost of a BFS push superstep's kernel sequence in a CUDA graph when the
// kernels do no work: words (592 x 256, no smem) -> heavy (444 x 256, 64 KB dynamic smem) ->
// seg (148 x 1024, 192 KB) -> diff (592 x 256), repeated R times in a straight-line graph.
// Variants: as above; heavy/seg without dynamic smem; every kernel with the max-smem carveout.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o graph_carveout graph_carveout.cu
#include <cuda_runtime.h>
#include <cstdio>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s (line %d)\n", #x, cudaGetErrorString(e), __LINE__); return 1; } } while (0)
__global__ void k_small(int *p) { if (p[0] == 12345) p[1] = threadIdx.x; }
// PDL variant: let the next kernel launch at once, wait for the previous grid before reading
__global__ void k_pdl(int *p) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    if (p[0] == 12345) p[1] = threadIdx.x;
}
__global__ void __launch_bounds__(1024, 1) k_pdl_big(int *p) {
    extern __shared__ int s[];
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    if (p[0] == 12345) { s[threadIdx.x] = 1; p[1] = s[threadIdx.x ^ 1]; }
}
static cudaError_t launch_pdl(void (*k)(int *), int grid, int block, int smem, cudaStream_t s, int *p) {
    cudaLaunchConfig_t c = {};
    c.gridDim = dim3(grid);
    c.blockDim = dim3(block);
    c.dynamicSmemBytes = smem;
    c.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    c.attrs = at;
    c.numAttrs = 1;
    return cudaLaunchKernelEx(&c, k, p);
}
__global__ void k_smem(int *p) { extern __shared__ int s[]; if (p[0] == 12345) { s[threadIdx.x] = 1; p[1] = s[threadIdx.x ^ 1]; } }
__global__ void __launch_bounds__(1024, 1) k_big(int *p) { extern __shared__ int s[]; if (p[0] == 12345) { s[threadIdx.x] = 1; p[1] = s[threadIdx.x ^ 1]; } }

int run(int variant, int R) {
    int *p;
    CK(cudaMalloc(&p, 64));
    CK(cudaMemset(p, 0, 64));
    const int sm_heavy = variant == 1 ? 0 : 64 * 1024, sm_seg = variant == 1 ? 0 : 192 * 1024;
    CK(cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024));
    CK(cudaFuncSetAttribute(k_big, cudaFuncAttributeMaxDynamicSharedMemorySize, 192 * 1024));
    CK(cudaFuncSetAttribute(k_pdl_big, cudaFuncAttributeMaxDynamicSharedMemorySize, 192 * 1024));
    const int carve = variant == 2 ? 100 : -1;
    CK(cudaFuncSetAttribute(k_small, cudaFuncAttributePreferredSharedMemoryCarveout, carve));
    CK(cudaFuncSetAttribute(k_smem, cudaFuncAttributePreferredSharedMemoryCarveout, carve));
    CK(cudaFuncSetAttribute(k_big, cudaFuncAttributePreferredSharedMemoryCarveout, carve));
    cudaStream_t s;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    cudaGraph_t g;
    CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
    for (int r = 0; r < R; r++) {
        if (variant == 4) {   // PDL chain
            CK(launch_pdl(k_pdl, 592, 256, 0, s, p));
            CK(launch_pdl(k_pdl, 444, 256, 0, s, p));
            CK(launch_pdl(k_pdl_big, 148, 1024, 192 * 1024, s, p));
            CK(launch_pdl(k_pdl, 592, 256, 0, s, p));
            continue;
        }
        if (variant == 3) {   // words + diff only
            k_small<<<592, 256, 0, s>>>(p);
            k_small<<<592, 256, 0, s>>>(p);
            continue;
        }
        k_small<<<592, 256, 0, s>>>(p);
        k_smem<<<444, 256, sm_heavy, s>>>(p);
        k_big<<<148, 1024, sm_seg, s>>>(p);
        k_small<<<592, 256, 0, s>>>(p);
    }
    CK(cudaStreamEndCapture(s, &g));
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int i = 0; i < 5; i++) {
        cudaEventRecord(a, s);
        CK(cudaGraphLaunch(ex, s));
        cudaEventRecord(b, s);
        CK(cudaStreamSynchronize(s));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (i && ms < best) best = ms;
    }
    const char *nm[] = {"words/heavy(64K)/seg(192K)/diff", "same, no dynamic smem", "same, carveout max on all",
                        "words/diff only", "4 kernels, PDL chain (192K seg)"};
    printf("%-36s: %.2f us per superstep\n", nm[variant], 1000.f * best / R);
    return 0;
}
int main() {
    for (int v = 0; v < 5; v++) run(v, 200);
    return 0;
}
