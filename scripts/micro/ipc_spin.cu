// ipc_spin.cu — feasibility probe for the cross-process peer-memory exchange on ONE GPU:
// two processes (fork before CUDA init) share a cudaMalloc buffer through cudaIpcMemHandle; each
// launches a kernel that stores a flag into the shared buffer and spins until the other's flag
// appears (system-scope release/acquire).  Finishing proves that time-sliced contexts make
// progress while a kernel spins, so a device-side cross-rank barrier cannot deadlock on one GPU.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/ipc_spin ipc_spin.cu
#include <cstdio>
#include <cstring>
#include <sys/wait.h>
#include <unistd.h>
#include <cuda_runtime.h>

__global__ void k_meet(unsigned long long *flags, int me, int rounds, unsigned long long *out) {
    const int other = me ^ 1;
    unsigned long long spins = 0;
    for (int r = 1; r <= rounds; r++) {
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(flags + me), "l"((unsigned long long)r) : "memory");
        unsigned long long v = 0;
        do {
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(flags + other) : "memory");
            spins++;
        } while (v < (unsigned long long)r);
    }
    *out = spins;
}

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e)); _exit(2); } } while (0)

int main(int argc, char **argv) {
    const int rounds = argc > 1 ? atoi(argv[1]) : 100;
    int p2c[2];
    if (pipe(p2c)) return 1;
    pid_t pid = fork();
    const int me = pid == 0 ? 1 : 0;
    CK(cudaSetDevice(0));
    unsigned long long *flags = nullptr, *out = nullptr;
    CK(cudaMalloc(&out, 8));
    if (me == 0) {
        CK(cudaMalloc(&flags, 64));
        CK(cudaMemset(flags, 0, 64));
        CK(cudaDeviceSynchronize());
        cudaIpcMemHandle_t h;
        CK(cudaIpcGetMemHandle(&h, flags));
        if (write(p2c[1], &h, sizeof h) != sizeof h) return 1;
    } else {
        cudaIpcMemHandle_t h;
        if (read(p2c[0], &h, sizeof h) != sizeof h) return 1;
        CK(cudaIpcOpenMemHandle((void **)&flags, h, cudaIpcMemLazyEnablePeerAccess));
    }
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    k_meet<<<1, 1>>>(flags, me, rounds, out);
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    unsigned long long spins = 0;
    CK(cudaMemcpy(&spins, out, 8, cudaMemcpyDeviceToHost));
    printf("rank %d: %d rounds in %.3f ms (%.1f us/round), spins %llu\n", me, rounds, ms, ms * 1e3 / rounds, spins);
    if (me == 1) CK(cudaIpcCloseMemHandle(flags));
    if (me == 0) {
        int st = 0;
        waitpid(pid, &st, 0);
        printf("child exit %d\n", WEXITSTATUS(st));
    }
    return 0;
}
