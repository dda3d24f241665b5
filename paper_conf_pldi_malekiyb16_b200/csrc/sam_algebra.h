// sam_algebra.h -- carry algebra of order-k, tuple-s scans (host + device).
//
// Per tuple lane, the order-k scan is the linear recurrence
//     y_1[r] = y_1[r-1] + x[r],   y_t[r] = y_t[r-1] + y_{t-1}[r]   (t = 2..k).
// Its state at a lane position is the k-vector (y_1..y_k).  Over a span of L lane positions
// with zero input the state maps by M(L), unit lower-triangular Toeplitz with
//     M(L)[t][j] = C(L-1+t-j, t-j)       (M(1) = one recurrence step, M(L) = M(1)^L),
// stored as its first column b_d(L) = C(L-1+d, d), d = 0..k-1.  M(a)M(b) = M(a+b) for all
// integers a, b (Vandermonde), M(-1) = I - N.  A span with input is (L, v): s -> M(L)s + v, and
//     (L_a, a) (+) (L_b, b) = (L_a + L_b, M(L_b) a + b)
// is the associative carry operator of the look-back.
//
// Integers are computed mod 2^w (reading R2): C(N, d) mod 2^64 is formed exactly from
// the product N(N-1)..(N-d+1) mod 2^128, divided by the power of two of d! and multiplied by
// the inverse of d!'s odd part mod 2^64.  Floats use double.
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define SAM_HD __host__ __device__ __forceinline__
#else
#define SAM_HD inline
#endif

namespace sam {

constexpr int MAXK = 8;
constexpr int MAXS = 8;

// inverse of an odd number mod 2^64 (Newton: each step doubles the correct low bits)
SAM_HD uint64_t inv_odd64(uint64_t o) {
    uint64_t x = o;  // o*o == 1 mod 8
    for (int i = 0; i < 6; ++i) x *= 2u - o * x;
    return x;
}

// C(N, d) mod 2^64 for any signed N and 0 <= d <= 7 (generalised binomial N(N-1)..(N-d+1)/d!)
SAM_HD uint64_t binom_mod64(int64_t N, int d) {
    if (d == 0) return 1;
    bool neg = false;
    if (N < 0) {  // C(N, d) = (-1)^d C(d-N-1, d)
        N = (int64_t)d - N - 1;
        neg = (d & 1) != 0;
    }
    if (N < d) return 0;
    // d! = 2^e * odd
    const int e2[8] = {0, 0, 1, 1, 3, 3, 4, 4};
    const uint64_t odd[8] = {1, 1, 1, 3, 3, 15, 45, 315};
    unsigned __int128 p = 1;
    for (int i = 0; i < d; ++i) p *= (unsigned __int128)(uint64_t)(N - i);
    uint64_t q = (uint64_t)(p >> e2[d]);
    uint64_t r = q * inv_odd64(odd[d]);
    return neg ? (uint64_t)(0 - r) : r;
}

SAM_HD double binom_f64(int64_t N, int d) {
    if (d == 0) return 1.0;
    double sign = 1.0;
    if (N < 0) {
        N = (int64_t)d - N - 1;
        if (d & 1) sign = -1.0;
    }
    if (N < d) return 0.0;
    double r = 1.0;
    for (int i = 0; i < d; ++i) r = r * (double)(N - i) / (double)(i + 1);
    return sign * r;
}

template <typename T> struct Arith;
template <> struct Arith<uint32_t> {
    static SAM_HD uint32_t binom(int64_t N, int d) { return (uint32_t)binom_mod64(N, d); }
};
template <> struct Arith<uint64_t> {
    static SAM_HD uint64_t binom(int64_t N, int d) { return binom_mod64(N, d); }
};
template <> struct Arith<float> {
    static SAM_HD float binom(int64_t N, int d) { return (float)binom_f64(N, d); }
};
template <> struct Arith<double> {
    static SAM_HD double binom(int64_t N, int d) { return binom_f64(N, d); }
};

// b[d] = C(L-1+d, d), d = 0..k-1 : first column of M(L)
template <typename T>
SAM_HD void mcol(int64_t L, int k, T* b) {
    for (int d = 0; d < k; ++d) b[d] = Arith<T>::binom(L - 1 + d, d);
}

// out = M(b) v  (b = first column), out may not alias v
template <typename T>
SAM_HD void mapply(const T* b, const T* v, int k, T* out) {
    for (int t = 0; t < k; ++t) {
        T acc = v[t];
        for (int j = 0; j < t; ++j) acc += b[t - j] * v[j];
        out[t] = acc;
    }
}

// number of elements of global lane m in a stream of n elements starting at global index g
SAM_HD uint64_t lane_len(uint64_t n, uint64_t g, int s, int m) {
    uint64_t gm = g % (uint64_t)s;
    uint64_t i0 = ((uint64_t)m + (uint64_t)s - gm) % (uint64_t)s;  // first i with (g+i)%s == m
    return i0 < n ? (n - 1 - i0) / (uint64_t)s + 1 : 0;
}

// Fold `count` consecutive payloads onto the state base_m of global lane m (null = zero state):
// payload j: [u64 n_j][u64 g_j][values T [s][k]]  (stride = payload_bytes), each the zero-seeded
// state of every lane at its last element in a stream of n_j elements at global offset g_j.
// out_m[t] = state of lane m after the last of them.  out_m may alias base_m.
template <typename T>
SAM_HD void fold_payloads_from(const T* base_m, const unsigned char* payloads, size_t payload_bytes,
                               int count, int k, int s, int m, T* out_m) {
    T S[MAXK], tmp[MAXK], b[MAXK];
    for (int t = 0; t < k; ++t) S[t] = base_m ? base_m[t] : T(0);
    for (int j = 0; j < count; ++j) {
        const unsigned char* p = payloads + (size_t)j * payload_bytes;
        uint64_t nj = ((const uint64_t*)p)[0];
        uint64_t gj = ((const uint64_t*)p)[1];
        const T* v = (const T*)(p + 16) + (size_t)m * k;
        uint64_t L = lane_len(nj, gj, s, m);
        if (L == 0) continue;  // lane absent from the shard: the state passes through
        mcol<T>((int64_t)L, k, b);
        mapply<T>(b, S, k, tmp);
        for (int t = 0; t < k; ++t) S[t] = tmp[t] + v[t];
    }
    for (int t = 0; t < k; ++t) out_m[t] = S[t];
}

// Fold gathered shard payloads of ranks < rank into the seed of `rank`.
// seed[m][t] = state of global lane m at its last element before shard `rank`.
template <typename T>
SAM_HD void fold_payloads(const unsigned char* payloads, size_t payload_bytes, int rank, int k,
                          int s, int m, T* seed_m) {
    fold_payloads_from<T>(nullptr, payloads, payload_bytes, rank, k, s, m, seed_m);
}

}  // namespace sam
