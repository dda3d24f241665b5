// L2 vs HBM read bandwidth microbenchmark: each CTA streams its slice of a buffer `iters` times.
#include <cuda_runtime.h>
#include <stdint.h>
__global__ void rd(const int4* __restrict__ p, size_t n16, int iters, int* sink) {
    int acc = 0;
    for (int it = 0; it < iters; ++it)
        for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
            int4 v;
            asm volatile("ld.global.cg.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i));
            acc += v.x ^ v.y ^ v.z ^ v.w;
        }
    if (acc == 0x12345678) *sink = acc;
}
extern "C" float run_rd(const void* p, size_t bytes, int iters, int* sink) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    rd<<<nsm * 8, 256>>>((const int4*)p, bytes / 16, 1, sink);
    cudaEventRecord(a);
    rd<<<nsm * 8, 256>>>((const int4*)p, bytes / 16, iters, sink);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    return ms;
}
