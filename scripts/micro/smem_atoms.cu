// Microbenchmark: shared-memory random-access rates on one B200 (LDS / ATOMS.OR / STS.U8 / LDS+cond ATOMS).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/smem_atoms smem_atoms.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint32_t x) { x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16; return x; }
constexpr int WORDS = 48 * 1024;   // 192 KB
template <int MODE>
__global__ void __launch_bounds__(1024, 1) k(int iters, uint32_t *out, uint32_t density) {
    extern __shared__ uint32_t s[];
    for (int i = threadIdx.x; i < WORDS; i += 1024) s[i] = 0;
    __syncthreads();
    uint32_t acc = 0, x = hsh(blockIdx.x * 1024 + threadIdx.x);
    for (int it = 0; it < iters; it++) {
        x = hsh(x + it);
        const uint32_t v = x % (WORDS * 32);   // vertex in the slice
        const uint32_t m = 1u << (v & 31);
        if (MODE == 0) acc += s[v >> 5];
        else if (MODE == 1) atomicOr(s + (v >> 5), m);
        else if (MODE == 2) reinterpret_cast<volatile uint8_t *>(s)[v % (WORDS * 4)] = 1;
        else if (MODE == 3) { if (!(s[v >> 5] & m)) atomicOr(s + (v >> 5), m); }
        else if (MODE == 4) { if ((x >> 8) % 100 < density) atomicOr(s + (v >> 5), m); else acc += s[v >> 5]; }
    }
    __syncthreads();
    if (threadIdx.x == 0) out[blockIdx.x] = s[acc % WORDS] + acc;
}
int main() {
    uint32_t *out; cudaMalloc(&out, 4096 * 4);
    const char *names[] = {"LDS random u32", "ATOMS.OR random", "STS.U8 random", "LDS+cond ATOMS (fills)", "ATOMS frac"};
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    int iters = 4096;
    auto run = [&](auto kern, const char *nm, uint32_t dens) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, WORDS * 4);
        kern<<<148, 1024, WORDS * 4>>>(iters, out, dens);
        cudaEventRecord(a);
        kern<<<148, 1024, WORDS * 4>>>(iters, out, dens);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double ops = 148.0 * 1024 * iters;
        printf("%-28s dens %3u: %.3f ms  %.2f Gop/s  %.3f op/clk/SM @1.965GHz  err=%s\n", nm, dens, ms, ops / ms / 1e6,
               ops / 148 / (ms * 1e-3 * 1.965e9), cudaGetErrorString(cudaGetLastError()));
    };
    run(k<0>, names[0], 0); run(k<1>, names[1], 0); run(k<2>, names[2], 0); run(k<3>, names[3], 0);
    for (uint32_t d : {5u, 10u, 25u, 50u}) run(k<4>, names[4], d);
    return 0;
}
