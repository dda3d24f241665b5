/*
 * ORACLE PACKAGE -- TEST / MEASUREMENT INFRASTRUCTURE ONLY (bench.py's cpu_baseline context leg and
 * tests/ may load it; the product path never does).
 *
 * All-cores CPU context scan ("a context-only all-cores CPU scan"): the order-k,
 * tuple-s inclusive prefix sum computed as k passes of the order-1 operator, each
 * pass parallelised over `nthreads` contiguous chunks with the classic two-phase scheme:
 *   1. every chunk sums each tuple lane m of its elements (lane of a[i] = (phase + i) mod s,
 *      P:349-355);
 *   2. a serial exclusive prefix over the chunk sums gives each chunk's incoming per-lane sums;
 *   3. every chunk rescans its elements seeded with them.
 * Integers only (uint32/uint64, wraparound mod 2^w: the same results as sam_oracle.c, bit for bit,
 * checked in tests/test_oracle_pins.py).  Two sweeps of the array per pass; no blocking beyond
 * the chunks.  It exists to put the GPU number next to a multi-core CPU one, not as a reference.
 */
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>

#define ALLCORES_SCAN(T)                                                                      \
    if (k < 1 || k > 64 || s < 1 || s > 64 || nthreads < 1 || nthreads > 1024) return -2;     \
    T* sums = (T*)calloc((size_t)nthreads * (size_t)s, sizeof(T));                           \
    if (!sums) return -3;                                                                      \
    for (int t = 0; t < k; ++t) {                                                              \
        _Pragma("omp parallel num_threads(nthreads)")                                         \
        {                                                                                      \
            const int c = omp_get_thread_num();                                                \
            const uint64_t lo = n * (uint64_t)c / (uint64_t)nthreads;                          \
            const uint64_t hi = n * (uint64_t)(c + 1) / (uint64_t)nthreads;                    \
            T* my = sums + (size_t)c * s;                                                      \
            for (int m = 0; m < s; ++m) my[m] = 0;                                             \
            int m = (int)((lo + (uint64_t)phase) % (uint64_t)s);                               \
            for (uint64_t i = lo; i < hi; ++i) {                                               \
                my[m] += a[i];                                                                 \
                m = (m + 1 == s) ? 0 : m + 1;                                                  \
            }                                                                                  \
            _Pragma("omp barrier")                                                             \
            _Pragma("omp single")                                                              \
            {                                                                                  \
                for (int m2 = 0; m2 < s; ++m2) {                                               \
                    T run = 0;                                                                 \
                    for (int c2 = 0; c2 < nthreads; ++c2) {                                    \
                        T v = sums[(size_t)c2 * s + m2];                                       \
                        sums[(size_t)c2 * s + m2] = run;                                       \
                        run += v;                                                              \
                    }                                                                          \
                }                                                                              \
            }                                                                                  \
            m = (int)((lo + (uint64_t)phase) % (uint64_t)s);                                   \
            for (uint64_t i = lo; i < hi; ++i) {                                               \
                my[m] += a[i];                                                                 \
                a[i] = my[m];                                                                  \
                m = (m + 1 == s) ? 0 : m + 1;                                                  \
            }                                                                                  \
        }                                                                                      \
    }                                                                                          \
    free(sums);                                                                                \
    return 0;

int allcores_scan_u32(uint32_t* a, uint64_t n, int k, int s, int phase, int nthreads) { ALLCORES_SCAN(uint32_t) }
int allcores_scan_u64(uint64_t* a, uint64_t n, int k, int s, int phase, int nthreads) { ALLCORES_SCAN(uint64_t) }
