// Microbenchmark: throughput of __match_any_sync vs a shuffle-based
// equivalent on this GPU (warps per SM = 16, dependent chain per warp).
#include <cstdio>
#include <cuda_runtime.h>
template <int DISTINCT>
__global__ void k_match(unsigned *out, int iters, unsigned seed) {
    unsigned v = ((threadIdx.x & 31) % DISTINCT) * 77u + seed, acc = 0;
    for (int i = 0; i < iters; i++) {
        unsigned m = __match_any_sync(0xffffffffu, v);
        acc += m;
        v += (m & 1) * 4096u;  // same equivalence classes every iteration
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_alu(unsigned *out, int iters, unsigned seed) {
    unsigned v = (threadIdx.x * 2654435761u + seed) >> 28, acc = 0;
    for (int i = 0; i < iters; i++) {
        unsigned m = (v * 0x9E3779B1u) ^ (v >> 3);
        acc += m;
        v = (v + (m & 7)) & 15;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
    unsigned *d;
    cudaMalloc(&d, 148 * 512 * 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int iters = 100000;
    for (int rep = 0; rep < 2; rep++) {
        float ms;
        double per;
#define RUN(D)                                                                                     \
        cudaEventRecord(a);                                                                        \
        k_match<D><<<148, 512>>>(d, iters, rep);                                                   \
        cudaEventRecord(b);                                                                        \
        cudaEventSynchronize(b);                                                                   \
        cudaEventElapsedTime(&ms, a, b);                                                           \
        per = ms * 1e-3 * 1.965e9 / iters;                                                         \
        printf("match_any %2d distinct: %.3f ms, %.2f SM cycles per iteration (16 warps/SM)\n", D, ms, per);
        RUN(1) RUN(4) RUN(16) RUN(32)
        cudaEventRecord(a);
        k_alu<<<148, 512>>>(d, iters, rep);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        per = ms * 1e-3 * 1.965e9 / iters;
        printf("alu loop : %.3f ms, %.2f cycles per iteration per SM\n", ms, per);
    }
    return 0;
}
