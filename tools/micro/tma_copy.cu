// TMA-bulk copy microbenchmark (developer tool): what the scan kernel's memory pattern can reach
// without its dependency chain.  Persistent CTAs (one per SM) claim tiles from an atomic counter,
// pull each tile from HBM with a 1-D cp.async.bulk into a ring of NB smem buffers and write it
// back with a bulk store.  Mode 1 ("reload") also parks each tile in L2 for LAGT tiles and re-reads
// it from L2 before the store, like the scan's carry application.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_copy tools/micro/tma_copy.cu
//   /tmp/tma_copy [log2 bytes=32]
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
    asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(sa(b)), "r"(par) : "memory");
}
__device__ __forceinline__ void g2s(void* d, const void* s, uint32_t n, uint64_t* b, uint64_t pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 ::"r"(sa(d)), "l"(s), "r"(n), "r"(sa(b)), "l"(pol) : "memory");
}
__device__ __forceinline__ void s2g(void* d, const void* s, uint32_t n, uint64_t pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(d), "r"(sa(s)), "r"(n), "l"(pol) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N> __device__ __forceinline__ void wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ uint64_t pol_last() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ uint64_t pol_first() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }

constexpr int NB = 6;
// mode 0: load -> store, NB buffers, NB-1 loads in flight.
// mode 1: every tile is read twice: from HBM (evict_last, ring A of NA buffers, data discarded)
// and LAGT tiles later from L2 (evict_first, ring B) before its store -- the scan's traffic pattern.
__global__ void copy_kernel(const unsigned char* in, unsigned char* out, uint64_t ntiles, uint32_t tb, int mode,
                            int lagt, unsigned long long* ctr) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* bar = (uint64_t*)(sm + NB * tb);
    __shared__ long long tiles[64];
    if (threadIdx.x != 0) return;
    for (int b = 0; b < NB; ++b) mbar_init(&bar[b], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    const uint64_t pl = pol_last(), pf = pol_first();
    if (mode == 0) {
        long long t[NB];
        auto issue = [&](int i) {
            const unsigned long long c = atomicAdd(ctr, 1ull);
            t[i % NB] = c < ntiles ? (long long)c : -1;
            if (t[i % NB] >= 0) {
                expect_tx(&bar[i % NB], tb);
                g2s(sm + (i % NB) * tb, in + (uint64_t)t[i % NB] * tb, tb, &bar[i % NB], pf);
            }
        };
        for (int i = 0; i < NB - 1; ++i) issue(i);
        for (int i = 0;; ++i) {
            if (t[i % NB] < 0) break;
            mbar_wait(&bar[i % NB], (i / NB) & 1);
            s2g(out + (uint64_t)t[i % NB] * tb, sm + (i % NB) * tb, tb, pf);
            wait_read<1>();  // store of slot i-1 has read its buffer, which slot i+NB-1 reuses
            issue(i + NB - 1);
        }
    } else {
        // ring A: buffers 0..2 (HBM reads), ring B: buffers 3..5 (L2 reloads + stores).  Step i:
        // (A) claim + HBM-load tile i, (B) L2-reload tile i-lagt, (C) store tile i-lagt-1.
        constexpr int NA = 3, NBB = 3;
        int nt = -1;  // tiles claimed (valid) once the counter ran out
        for (int i = 0;; ++i) {
            if (nt < 0) {
                const unsigned long long c = atomicAdd(ctr, 1ull);
                if (c < ntiles) {
                    if (i >= NA) mbar_wait(&bar[i % NA], ((i - NA) / NA) & 1);
                    expect_tx(&bar[i % NA], tb);
                    g2s(sm + (i % NA) * tb, in + c * tb, tb, &bar[i % NA], pl);
                    tiles[i % 64] = (long long)c;
                } else {
                    nt = i;
                }
            }
            const int q = i - lagt;
            if (q >= 0 && (nt < 0 || q < nt)) {
                const int b = NA + q % NBB;
                if (q >= NBB) wait_read<NBB - 2>();
                expect_tx(&bar[b], tb);
                g2s(sm + b * tb, in + (uint64_t)tiles[q % 64] * tb, tb, &bar[b], pf);
            }
            const int q2 = q - 1;
            if (q2 >= 0 && (nt < 0 || q2 < nt)) {
                const int b = NA + q2 % NBB;
                mbar_wait(&bar[b], (q2 / NBB) & 1);
                s2g(out + (uint64_t)tiles[q2 % 64] * tb, sm + b * tb, tb, pf);
            }
            if (nt >= 0 && q2 >= nt - 1) break;
        }
        for (int q = (nt > NA ? nt - NA : 0); q < nt; ++q) mbar_wait(&bar[q % NA], (q / NA) & 1);
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main(int argc, char** argv) {
    const int lg = argc > 1 ? atoi(argv[1]) : 32;
    const size_t bytes = (size_t)1 << lg;
    unsigned char *a, *b;
    unsigned long long* ctr;
    cudaMalloc(&a, bytes);
    cudaMalloc(&b, bytes);
    cudaMalloc(&ctr, 8);
    cudaMemset(a, 1, bytes);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms;
    for (int i = 0; i < 3; ++i) cudaMemcpy(b, a, bytes, cudaMemcpyDeviceToDevice);
    cudaEventRecord(e0);
    for (int i = 0; i < 10; ++i) cudaMemcpy(b, a, bytes, cudaMemcpyDeviceToDevice);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("cudaMemcpy D2D %.1f GiB: %.0f GB/s\n", bytes / 1073741824.0, 2.0 * bytes * 10 / ms / 1e6);
    const uint32_t tbs[] = {16384, 27648, 36864};
    for (int mode = 0; mode < 2; ++mode) {
        for (uint32_t tb : tbs) {
            const int lags[] = {1, 8, 16, 24, 40};
            for (int li = 0; li < (mode ? 5 : 1); ++li) {
                const int lagt = lags[li];
                const size_t smem = NB * (size_t)tb + NB * 8;
                if (smem > 227 * 1024) continue;
                cudaFuncSetAttribute(copy_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
                const uint64_t nt = bytes / tb;
                float best = 1e9;
                for (int r = 0; r < 6; ++r) {
                    cudaMemset(ctr, 0, 8);
                    cudaEventRecord(e0);
                    copy_kernel<<<sms, 32, smem>>>(a, b, nt, tb, mode, lagt, ctr);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    cudaEventElapsedTime(&ms, e0, e1);
                    if (r >= 2 && ms < best) best = ms;
                }
                cudaError_t err = cudaGetLastError();
                printf("mode %d tile %6u B lag %2d: %.0f GB/s (algorithmic 2x bytes) %s\n", mode, tb, lagt,
                       2.0 * nt * tb / best / 1e6, err == cudaSuccess ? "" : cudaGetErrorString(err));
            }
        }
    }
    return 0;
}
