// sam_generic.cuh -- generic single-pass order-k, tuple-s scan for every associative operator of
// SURVEY 8(f) NEXT-4 (add, xor, max, min; "prefix scans") with a
// selectable inter-tile carry scheme (NEXT-3, the paper's Sec. 5.4 ablation):
//
//   GEN_STATIC    SAM's persistent-block schedule: a co-resident grid of P CTAs
//                 (cooperative launch), CTA b owns tiles b, b+P, ...; the carry into tile S is
//                 the CTA's own inclusive state after S-P advanced over the P-1 aggregates the
//                 other CTAs published in between.
//   GEN_LOOKBACK  decoupled look-back (the O(n) scheme P:1589-1637 describes for CUB): tiles are
//                 claimed in order from an atomic counter by any number of CTAs (no co-residency
//                 assumption -- the fallback when a cooperative grid cannot form);
//                 each tile publishes its aggregate, folds predecessors back to the nearest
//                 inclusive state, publishes its inclusive state.
//   GEN_CHAINED   chained scan: each tile waits for its predecessor's inclusive
//                 state only.
//
// One CTA processes one tile at a time, entirely in shared memory (several CTAs per SM hide the
// latencies); the production add path is the warp-specialised kernel of sam_kernel.cuh.
// Within a tile, order k is computed as k passes of the order-1 operator,
// each pass a block-wide stride-s scan (thread chunks -> shuffle scan of per-lane thread totals ->
// cross-warp combine, the paper's three phases P:638-678).
//
// Carry algebra per tuple lane (the k-vector state at a lane's last element of a span):
//   linear ops (add; xor = addition in GF(2)^w): state after a span of L lane positions entered
//     with state c is M(L) c + a, M(L)[t][j] = C(L-1+t-j, t-j) -- mod 2^w for integer add, mod 2
//     for xor (Lucas: C(n,d) is odd iff d & ~n == 0), double for floats;
//   idempotent ops (max, min): a prefix max of a prefix max is itself, so order k = order 1 and the
//     k-fold exclusive scan is the inclusive one shifted by k lane positions (reading R14); the
//     state is the lane's last k inclusive values (v_0 newest), and a span with last-k local values
//     a (span length >= k) maps c to (op(c_0, a_j))_j.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <cfloat>
#include <climits>

#include "sam_algebra.h"

namespace sam {
namespace gen {

enum { OP_ADD = 0, OP_XOR = 1, OP_MAX = 2, OP_MIN = 3 };
enum { GEN_STATIC = 0, GEN_LOOKBACK = 1, GEN_CHAINED = 2 };

constexpr int TB = 256;    // threads per CTA
constexpr int NWG = TB / 32;

// lane positions per lane per thread: a tile is TB * ips(s) * s elements (~16 KB for any s)
template <typename T> struct Ips {
    static constexpr int BASE = sizeof(T) == 4 ? 16 : 8;
    static __host__ __device__ constexpr int of(int s) { return BASE / s > 1 ? BASE / s : 1; }
};

template <typename T, int OP> struct Op;
template <typename T> struct Op<T, OP_ADD> {
    static constexpr bool LIN = true;
    static __device__ __forceinline__ T id() { return T(0); }
    static __device__ __forceinline__ T ap(T a, T b) { return a + b; }
};
template <typename T> struct Op<T, OP_XOR> {
    static constexpr bool LIN = true;
    static __device__ __forceinline__ T id() { return T(0); }
    static __device__ __forceinline__ T ap(T a, T b) { return a ^ b; }
};
template <typename T> struct Lim;
template <> struct Lim<int32_t> { static __device__ __forceinline__ int32_t lo() { return INT_MIN; } static __device__ __forceinline__ int32_t hi() { return INT_MAX; } };
template <> struct Lim<uint32_t> { static __device__ __forceinline__ uint32_t lo() { return 0u; } static __device__ __forceinline__ uint32_t hi() { return 0xffffffffu; } };
template <> struct Lim<int64_t> { static __device__ __forceinline__ int64_t lo() { return LLONG_MIN; } static __device__ __forceinline__ int64_t hi() { return LLONG_MAX; } };
template <> struct Lim<uint64_t> { static __device__ __forceinline__ uint64_t lo() { return 0ull; } static __device__ __forceinline__ uint64_t hi() { return ~0ull; } };
template <> struct Lim<float> { static __device__ __forceinline__ float lo() { return -__int_as_float(0x7f800000); } static __device__ __forceinline__ float hi() { return __int_as_float(0x7f800000); } };
template <> struct Lim<double> { static __device__ __forceinline__ double lo() { return -__longlong_as_double(0x7ff0000000000000ll); } static __device__ __forceinline__ double hi() { return __longlong_as_double(0x7ff0000000000000ll); } };
template <typename T> __device__ __forceinline__ T vmax(T a, T b) { return b > a ? b : a; }
template <typename T> __device__ __forceinline__ T vmin(T a, T b) { return b < a ? b : a; }
template <> __device__ __forceinline__ float vmax(float a, float b) { return fmaxf(a, b); }
template <> __device__ __forceinline__ float vmin(float a, float b) { return fminf(a, b); }
template <> __device__ __forceinline__ double vmax(double a, double b) { return fmax(a, b); }
template <> __device__ __forceinline__ double vmin(double a, double b) { return fmin(a, b); }
template <typename T> struct Op<T, OP_MAX> {
    static constexpr bool LIN = false;
    static __device__ __forceinline__ T id() { return Lim<T>::lo(); }
    static __device__ __forceinline__ T ap(T a, T b) { return vmax(a, b); }
};
template <typename T> struct Op<T, OP_MIN> {
    static constexpr bool LIN = false;
    static __device__ __forceinline__ T id() { return Lim<T>::hi(); }
    static __device__ __forceinline__ T ap(T a, T b) { return vmin(a, b); }
};

// coefficient arithmetic of the linear carry algebra: b_d(L) = C(L-1+d, d) and b*x
template <typename T, int OP> struct Coefs;
template <typename T> struct Coefs<T, OP_ADD> {  // integers mod 2^w, floats in double
    using C = std::conditional_t<std::is_floating_point<T>::value, double, T>;
    static __device__ __forceinline__ C binom(int64_t N, int d) {
        if constexpr (std::is_floating_point<T>::value) return binom_f64(N, d);
        else return (C)binom_mod64(N, d);
    }
    static __device__ __forceinline__ C add(C a, C b) { return a + b; }
    static __device__ __forceinline__ C mul(C b, C x) { return b * x; }
};
template <typename T> struct Coefs<T, OP_XOR> {  // GF(2): C(N, d) mod 2 by Lucas
    using C = T;
    static __device__ __forceinline__ C binom(int64_t N, int d) {
        if (d == 0) return C(1);
        if (N < 0) {  // C(N, d) = (-1)^d C(d-N-1, d): the sign is irrelevant mod 2
            N = (int64_t)d - N - 1;
        }
        return ((uint64_t)d & ~(uint64_t)N) == 0 ? C(1) : C(0);
    }
    static __device__ __forceinline__ C add(C a, C b) { return a ^ b; }
    static __device__ __forceinline__ C mul(C b, C x) { return b ? x : C(0); }
};

// 64-bit tagged words per value ([tag32 | 32 value bits])
template <typename T> struct GW { static constexpr int W = sizeof(T) == 4 ? 1 : 2; };
template <typename T> __device__ __forceinline__ uint64_t tbits(T v) {
    uint64_t b = 0;
    memcpy(&b, &v, sizeof(T));
    return b;
}
template <typename T> __device__ __forceinline__ T fbits(uint64_t b) {
    T v;
    memcpy(&v, &b, sizeof(T));
    return v;
}

template <typename T, int K>
struct GParams {
    const T* in;
    T* out;
    uint64_t n;
    uint64_t num_tiles;
    int s, k, inclusive, mode;
    unsigned long long* words;   // per tile: [s][K][agg W | incl W] tagged words
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned int* epoch_ptr;
};

__device__ __forceinline__ unsigned long long g_ld(const unsigned long long* p) {
    unsigned long long a;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(a) : "l"(p) : "memory");
    return a;
}
__device__ __forceinline__ void g_st(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ int pad(int e) { return e + (e >> 5); }  // one pad word per 32: conflict-free chunks

template <typename T, int OP, int K>
struct GSmem {
    // dynamic shared memory of a launch with tuple size s: two padded tiles + warp totals + states
    static constexpr size_t bytes(int s) {
        const int TT = TB * Ips<T>::of(s) * s;
        return (size_t)(2 * (TT + TT / 32 + 8) + NWG * 8 + 3 * 8 * K) * sizeof(T);
    }
};

// One order-1 inclusive op-scan pass over buf (tile of s*U elements, lane of element e = e % s),
// seeded per lane with seed[m]; returns through `tot` (smem [8]) the lane totals (last values).
template <typename T, int OP>
__device__ __forceinline__ void block_pass(T* buf, const T* seed, int s, int items, T* wt) {
    using O = Op<T, OP>;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    T acc[8];
#pragma unroll
    for (int m = 0; m < 8; ++m) acc[m] = O::id();
    const int e0 = tid * items;
    {
        int m = 0;
        for (int i = 0; i < items; ++i) {
            const int a = pad(e0 + i);
            // acc[m] = op(acc[m], buf[a]) with a register-indexed lane (s <= 8): select
            T v = buf[a];
            T r = O::id();
#pragma unroll
            for (int mm = 0; mm < 8; ++mm) {
                if (mm == m) { acc[mm] = O::ap(acc[mm], v); r = acc[mm]; }
            }
            buf[a] = r;
            m = (m + 1 == s) ? 0 : m + 1;
        }
    }
    // block exclusive scan of the per-lane thread totals
    T inc[8];
#pragma unroll
    for (int m = 0; m < 8; ++m) inc[m] = acc[m];
#pragma unroll
    for (int l = 0; l < 5; ++l) {
        const int off = 1 << l;
#pragma unroll
        for (int m = 0; m < 8; ++m) {
            if (m < s) {
                T o = __shfl_up_sync(0xffffffffu, inc[m], off);
                if (lane >= off) inc[m] = O::ap(o, inc[m]);
            }
        }
    }
    if (lane == 31) {
#pragma unroll
        for (int m = 0; m < 8; ++m) if (m < s) wt[warp * 8 + m] = inc[m];
    }
    __syncthreads();
    T pre[8];
#pragma unroll
    for (int m = 0; m < 8; ++m) {
        if (m < s) {
            T wp = seed[m];
            for (int w = 0; w < warp; ++w) wp = O::ap(wp, wt[w * 8 + m]);
            T ex = __shfl_up_sync(0xffffffffu, inc[m], 1);
            pre[m] = lane == 0 ? wp : O::ap(wp, ex);
        } else {
            pre[m] = O::id();
        }
    }
    {
        int m = 0;
        for (int i = 0; i < items; ++i) {
            const int a = pad(e0 + i);
            T pm = O::id();
#pragma unroll
            for (int mm = 0; mm < 8; ++mm) if (mm == m) pm = pre[mm];
            buf[a] = O::ap(pm, buf[a]);
            m = (m + 1 == s) ? 0 : m + 1;
        }
    }
    __syncthreads();  // buf complete; wt free for the next pass
}

// the generic kernel: one tile per CTA iteration
template <typename T, int OP, int K>
__global__ void __launch_bounds__(TB)
sam_generic_kernel(const __grid_constant__ GParams<T, K> p) {
    using O = Op<T, OP>;
    using S = GSmem<T, OP, K>;
    constexpr bool LIN = O::LIN;
    constexpr int W1 = GW<T>::W;
    extern __shared__ __align__(16) unsigned char smem[];
    const int s = p.s;
    const int IPS = Ips<T>::of(s);
    const int U = TB * IPS;                  // lane positions per tile
    const int TT = U * s;                    // tile elements
    const int BUF = TT + TT / 32 + 8;        // padded buffer
    T* xs = (T*)smem;
    T* ys = xs + BUF;
    T* wt = ys + BUF;                        // [NWG][8] warp totals
    T* st_agg = wt + NWG * 8;                // [8][K] tile aggregate
    T* st_c = st_agg + 8 * K;                // [8][K] carry (state before the tile)
    T* st_i = st_c + 8 * K;                  // [8][K] inclusive (own previous, static mode)
    __shared__ long long sh_tile;
    __shared__ unsigned sh_tag;
    const int tid = threadIdx.x, lane = tid & 31;
    const int items = IPS * s;
    const int kk = LIN ? K : p.k;             // state length (idempotent ops: the shift k)
    if (tid == 0) sh_tag = *(volatile unsigned*)p.epoch_ptr + 1u;
    __syncthreads();
    const uint32_t tag = sh_tag;
    using CC = typename std::conditional_t<LIN, Coefs<T, (OP == OP_XOR ? OP_XOR : OP_ADD)>, Coefs<T, OP_ADD>>::C;
    auto cbin = [&](int64_t N, int d) -> CC {
        if constexpr (OP == OP_XOR) return Coefs<T, OP_XOR>::binom(N, d);
        else return Coefs<T, OP_ADD>::binom(N, d);
    };
    auto cadd = [&](CC a, CC b) -> CC {
        if constexpr (OP == OP_XOR) return a ^ b;
        else return a + b;
    };
    auto cmul = [&](CC b, CC x) -> CC {
        if constexpr (OP == OP_XOR) return b ? x : CC(0);
        else return b * x;
    };
    // out = M(L) v  (LIN), lane-local k-vectors in CC
    auto mapply = [&](int64_t L, const CC* v, CC* out) {
        CC b[K];
#pragma unroll
        for (int d = 0; d < K; ++d) b[d] = cbin(L - 1 + d, d);
#pragma unroll
        for (int t = 0; t < K; ++t) {
            CC a = v[t];
#pragma unroll
            for (int j = 0; j < t; ++j) a = cadd(a, cmul(b[t - j], v[j]));
            out[t] = a;
        }
    };
    auto wslot = [&](int64_t tile, int m, int t) -> unsigned long long* {
        return p.words + (((size_t)tile * s + m) * K + t) * (2 * W1);
    };
    auto put = [&](unsigned long long* w, T v) {
        const uint64_t b = tbits(v), hi = (uint64_t)tag << 32;
        g_st(w, hi | (b & 0xffffffffull));
        if (W1 == 2) g_st(w + 1, hi | (b >> 32));
    };
    // read value (agg: half 0, incl: half 1) if its tag is current
    auto get = [&](const unsigned long long* w, T& v) -> bool {
        const uint64_t a = g_ld(w);
        uint64_t b = a & 0xffffffffull;
        bool ok = (uint32_t)(a >> 32) == tag;
        if (W1 == 2) {
            const uint64_t c = g_ld(w + 1);
            ok &= (uint32_t)(c >> 32) == tag;
            b |= c << 32;
        }
        v = fbits<T>(b);
        return ok;
    };

    const bool is_static = p.mode == GEN_STATIC;
    for (int64_t iter = 0;; ++iter) {
        // ---- which tile
        if (tid == 0) {
            if (is_static) sh_tile = (long long)blockIdx.x + iter * (long long)gridDim.x;
            else sh_tile = iter == 0 ? (long long)atomicAdd(p.tile_ctr, 1ull) : (long long)p.num_tiles;
        }
        __syncthreads();
        const int64_t tile = sh_tile;
        if ((uint64_t)tile >= p.num_tiles) break;
        const uint64_t e0 = (uint64_t)tile * TT;
        const uint64_t ne = (e0 + TT <= p.n) ? TT : p.n - e0;
        // ---- load (coalesced), identity beyond n
        for (int e = tid; e < TT; e += TB) {
            const T v = (uint64_t)e < ne ? p.in[e0 + e] : O::id();
            xs[pad(e)] = v;
            ys[pad(e)] = v;
        }
        __syncthreads();
        // ---- phase A: local (identity-seeded) passes, tile aggregate per lane
        __shared__ T zseed[8];
        if (tid < 8) zseed[tid] = O::id();
        __syncthreads();
        const int npass = LIN ? K : 1;
        for (int t = 0; t < npass; ++t) {
            block_pass<T, OP>(ys, zseed, s, items, wt);
            if (LIN && tid < s) st_agg[tid * K + t] = ys[pad(TT - s + tid)];
        }
        if (!LIN && tid < s) {
            for (int j = 0; j < kk; ++j) st_agg[tid * K + j] = ys[pad(TT - s + tid - j * s)];
        }
        __syncthreads();
        // ---- publish the aggregate (look-back, static)
        if (p.mode != GEN_CHAINED && tid < s * K) {
            const int m = tid / K, t = tid % K;
            if (LIN || t < kk) put(wslot(tile, m, t), st_agg[m * K + t]);
        }
        // ---- carry into this tile (warp 0, lane m < s owns tuple lane m)
        if (tid < 32) {
            const int m = lane;
            const bool lm = m < s;
            CC c[K];
            T cv[K];  // idempotent: carry's last-k values
#pragma unroll
            for (int t = 0; t < K; ++t) { c[t] = CC(0); cv[t] = O::id(); }
            if (tile > 0) {
                if (p.mode == GEN_CHAINED) {
                    // wait for the predecessor's inclusive state
                    bool ok = false;
                    while (!__all_sync(0xffffffffu, ok)) {
                        ok = true;
                        if (lm) {
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                if (!LIN && t >= kk) continue;
                                T v;
                                ok &= get(wslot(tile - 1, m, t) + W1, v);
                                if (LIN) c[t] = CC(v); else cv[t] = v;
                            }
                        }
                    }
                } else if (p.mode == GEN_LOOKBACK) {
                    // fold predecessors back to the nearest inclusive state
                    CC acc[K], pm[K], bU[K], np[K];
                    T vnear[K];
                    T red = O::id();
#pragma unroll
                    for (int t = 0; t < K; ++t) { acc[t] = CC(0); pm[t] = cbin(t - 1, t); bU[t] = cbin((int64_t)U - 1 + t, t); vnear[t] = O::id(); }
                    // pm = b(0 * U) = identity column (1, 0, ...)
                    int64_t j = tile - 1;
                    int depth = 0;
                    for (;;) {
                        T vi[K], va[K];
                        bool inc_ok = true, agg_ok = true;
                        if (lm) {
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                if (!LIN && t >= kk) { vi[t] = va[t] = O::id(); continue; }
                                inc_ok &= get(wslot(j, m, t) + W1, vi[t]);
                                agg_ok &= get(wslot(j, m, t), va[t]);
                            }
                        }
                        const bool all_inc = __all_sync(0xffffffffu, inc_ok);
                        const bool all_agg = __all_sync(0xffffffffu, agg_ok);
                        if (!all_inc && !all_agg) continue;  // predecessor still busy: re-poll
                        const bool use_inc = all_inc;
                        const T* v = use_inc ? vi : va;
                        if (LIN) {
                            // acc += M(depth U) v ; for the stop: c = acc + M(depth U) I
                            CC x[K], y[K];
#pragma unroll
                            for (int t = 0; t < K; ++t) x[t] = CC(v[t]);
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                CC a = x[t];
#pragma unroll
                                for (int q = 0; q < t; ++q) a = cadd(a, cmul(pm[t - q], x[q]));
                                y[t] = a;
                            }
#pragma unroll
                            for (int t = 0; t < K; ++t) acc[t] = cadd(acc[t], y[t]);
                            // pm <- pm * M(U)  (truncated polynomial product of first columns)
#pragma unroll
                            for (int d = 0; d < K; ++d) {
                                CC a = CC(0);
#pragma unroll
                                for (int e2 = 0; e2 <= d; ++e2) a = cadd(a, cmul(pm[e2], bU[d - e2]));
                                np[d] = a;
                            }
#pragma unroll
                            for (int d = 0; d < K; ++d) pm[d] = np[d];
                        } else {
                            if (depth == 0) {
#pragma unroll
                                for (int t = 0; t < K; ++t) vnear[t] = v[t];
                            } else {
                                red = O::ap(v[0], red);  // farther spans' newest values, oldest first
                            }
                        }
                        ++depth;
                        if (use_inc || j == 0) break;
                        --j;
                    }
                    if (LIN) {
#pragma unroll
                        for (int t = 0; t < K; ++t) c[t] = acc[t];
                    } else {
                        // c_j = op(op(I_0, farther), vnear_j); with depth 1, vnear is the inclusive itself
                        if (depth == 1) {
#pragma unroll
                            for (int t = 0; t < K; ++t) cv[t] = vnear[t];
                        } else {
#pragma unroll
                            for (int t = 0; t < K; ++t) cv[t] = O::ap(red, vnear[t]);
                        }
                    }
                    (void)np;
                } else {  // GEN_STATIC: own previous inclusive + the P-1 aggregates in between
                    // windows of 32 predecessors, one lane each (one round trip per window),
                    // tuple lane by tuple lane; lane 0 ends with the fold, then shares it
                    const int64_t P = gridDim.x;
                    const int64_t Sprev = tile - P;
                    const int64_t npred = tile - (Sprev >= 0 ? Sprev + 1 : 0);  // aggregates to fold
                    for (int mm = 0; mm < s; ++mm) {
                        CC tot[K];
                        T far = O::id(), near_v[K];
#pragma unroll
                        for (int t = 0; t < K; ++t) { tot[t] = CC(0); near_v[t] = O::id(); }
                        for (int64_t w0 = 0; w0 < npred; w0 += 32) {
                            const int64_t dd = w0 + lane;  // distance below tile-1
                            const bool valid = dd < npred;
                            T va[K];
#pragma unroll
                            for (int t = 0; t < K; ++t) va[t] = O::id();
                            bool ok = !valid;
                            while (!__all_sync(0xffffffffu, ok)) {
                                if (!ok) {
                                    ok = true;
#pragma unroll
                                    for (int t = 0; t < K; ++t) {
                                        if (!LIN && t >= kk) continue;
                                        ok &= get(wslot(tile - 1 - dd, mm, t), va[t]);
                                    }
                                }
                            }
                            if (LIN) {
                                // tree over lanes: x_l <- x_l + M(2^lev U) x_{l + 2^lev}
                                CC x[K];
#pragma unroll
                                for (int t = 0; t < K; ++t) x[t] = valid ? CC(va[t]) : CC(0);
#pragma unroll
                                for (int lev = 0; lev < 5; ++lev) {
                                    const int off = 1 << lev;
                                    CC o[K], mo[K];
#pragma unroll
                                    for (int t = 0; t < K; ++t) o[t] = __shfl_down_sync(0xffffffffu, x[t], off);
                                    mapply((int64_t)off * U, o, mo);
                                    if ((lane & (2 * off - 1)) == 0) {
#pragma unroll
                                        for (int t = 0; t < K; ++t) x[t] = cadd(x[t], mo[t]);
                                    }
                                }
                                if (lane == 0) {
                                    CC y[K];
                                    mapply(w0 * U, x, y);
#pragma unroll
                                    for (int t = 0; t < K; ++t) tot[t] = cadd(tot[t], y[t]);
                                }
                            } else {
                                // nearest span: all k values; farther ones: their newest value
                                T f = (valid && dd > 0) ? va[0] : O::id();
#pragma unroll
                                for (int lev = 0; lev < 5; ++lev) f = O::ap(f, __shfl_xor_sync(0xffffffffu, f, 1 << lev));
                                far = O::ap(far, f);
                                if (w0 == 0) {
#pragma unroll
                                    for (int t = 0; t < K; ++t) near_v[t] = __shfl_sync(0xffffffffu, va[t], 0);
                                }
                            }
                        }
                        // the CTA's own previous inclusive state, at distance npred
                        if (lane == 0) {
                            if (LIN) {
                                if (Sprev >= 0) {
                                    CC iv[K], y[K];
#pragma unroll
                                    for (int t = 0; t < K; ++t) iv[t] = CC(st_i[mm * K + t]);
                                    mapply(npred * U, iv, y);
#pragma unroll
                                    for (int t = 0; t < K; ++t) tot[t] = cadd(tot[t], y[t]);
                                }
#pragma unroll
                                for (int t = 0; t < K; ++t) st_c[mm * K + t] = T(tot[t]);
                            } else {
                                if (Sprev >= 0) {
                                    if (npred == 0) {
#pragma unroll
                                        for (int t = 0; t < K; ++t) near_v[t] = st_i[mm * K + t];
                                    } else {
                                        far = O::ap(far, st_i[mm * K]);
                                    }
                                }
#pragma unroll
                                for (int t = 0; t < K; ++t) st_c[mm * K + t] = O::ap(far, near_v[t]);
                            }
                        }
                    }
                    __syncwarp();
                    if (lm) {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            if (LIN) c[t] = CC(st_c[m * K + t]); else cv[t] = st_c[m * K + t];
                        }
                    }
                }
            }
            // inclusive state of this tile: M(U) c + a  /  (op(c_0, a_j))_j
            if (lm) {
                T inc[K];
                if (LIN) {
                    CC cu[K];
                    mapply((int64_t)U, c, cu);
#pragma unroll
                    for (int t = 0; t < K; ++t) inc[t] = T(cadd(cu[t], CC(st_agg[m * K + t])));
#pragma unroll
                    for (int t = 0; t < K; ++t) st_c[m * K + t] = T(c[t]);
                } else {
#pragma unroll
                    for (int t = 0; t < K; ++t) inc[t] = t < kk ? O::ap(cv[0], st_agg[m * K + t]) : O::id();
#pragma unroll
                    for (int t = 0; t < K; ++t) st_c[m * K + t] = cv[t];
                }
                if (p.mode != GEN_STATIC) {
#pragma unroll
                    for (int t = 0; t < K; ++t)
                        if (LIN || t < kk) put(wslot(tile, m, t) + W1, inc[t]);
                }
#pragma unroll
                for (int t = 0; t < K; ++t) st_i[m * K + t] = inc[t];
            }
        }
        __syncthreads();
        // ---- phase B: seeded passes over the input again
        for (int e = tid; e < TT; e += TB) ys[pad(e)] = xs[pad(e)];
        __syncthreads();
        for (int t = 0; t < npass; ++t) {
            if (tid < 8) zseed[tid] = tid < s ? st_c[tid * K + (LIN ? t : 0)] : O::id();
            __syncthreads();
            block_pass<T, OP>(ys, zseed, s, items, wt);
        }
        // ---- store: inclusive, or the k-fold exclusive shift (first k lane positions from the carry)
        const int ksh = LIN ? K : kk;
        for (int e = tid; (uint64_t)e < ne; e += TB) {
            T v;
            if (p.inclusive) {
                v = ys[pad(e)];
            } else if (e >= ksh * s) {
                v = ys[pad(e - ksh * s)];
            } else {
                const int m = e % s, r = e / s;  // lane position r < k: y_k at r - k (before the tile)
                const int d = ksh - 1 - r;       // = position -1-d
                if (LIN) {
                    // backward differences of the carry state: y_K[-1-d] = sum_t (-1)^t C(d,t) c_{K-t}
                    CC a = CC(0);
                    for (int t = 0; t <= d; ++t) {
                        CC term = CC(st_c[m * K + (K - 1 - t)]);
                        CC bin = cbin(d, t);  // C(d, t): the generalised binomial at N = d
                        CC w = cmul(bin, term);
                        if constexpr (OP == OP_XOR) a = a ^ w;
                        else a = (t & 1) ? a - w : a + w;
                    }
                    v = T(a);
                } else {
                    v = st_c[m * K + d];  // c_d = inclusive value d+1 positions before the tile
                }
            }
            p.out[e0 + e] = v;
        }
        __syncthreads();
        if (!is_static) break;  // look-back / chained: one tile per CTA
    }
    // ---- epilogue: the last CTA resets the counters and advances the epoch
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        const unsigned prev = atomicAdd(p.done_ctr, 1u);
        if (prev == gridDim.x - 1) {
            *(volatile unsigned long long*)p.tile_ctr = 0ull;
            *(volatile unsigned int*)p.done_ctr = 0u;
            __threadfence();
            atomicAdd(p.epoch_ptr, 1u);
        }
    }
}

}  // namespace gen
}  // namespace sam
