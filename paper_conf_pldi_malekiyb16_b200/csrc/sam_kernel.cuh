// sam_kernel.cuh -- single-pass order-k, tuple-s prefix sum for sm_100a.
//
// One kernel launch reads every input element once and writes every output element once
// (P:393-395): SAM's single-pass property, kept for any order and tuple
// size.  Per tile (T = W*32*ITEMS elements, W warps):
//   a1  the tile arrives in shared memory by a 1-D cp.async.bulk (TMA bulk engine) issued by one
//       thread one tile ahead (ring of 3 buffers, mbarrier completion), so the load of tile i+1
//       overlaps the look-back, carry application and store of tile i;
//   a2  thread <-> (tuple lane m, ITEMS consecutive lane positions), read from smem at stride s;
//       a warp holds G = (largest power of two dividing s) lanes, 32/G threads each, so the
//       strided reads are bank-conflict free (ITEMS odd) and registers do not grow with s
//       (P:467-473);
//   a3  zero-seeded order-k local scan: thread-serial recurrence (k adds per element), warp scan
//       of thread states (k plain shuffle scans, order by order), block combine of warp states;
//       the paper's three-phase intra-block scan iterated per order;
//   a4  publish the tile's per-lane k-vector aggregate, then its status word with release
//       semantics (the paper's "local sum -> fence -> ready flag"; one flag for all
//       s lanes; one value per order);
//   a5  decoupled look-back: one warp polls a window of predecessor status words with acquire
//       loads and folds aggregates with the carry operator until it meets an inclusive state
//       (the O(n) scheme the paper describes for CUB, which it advises once the
//       architectural factor grows; B200's af is ~9x Titan X's);
//   a6  fused carry application: thread incoming state = M(L)*carry + local prefix, then the
//       seeded recurrence produces the outputs (the binomial fix-up C(r+t-j, t-j));
//       exclusive = inclusive shifted by k lane positions (R1), the first k from
//       finite differences of the incoming state;
//   a7  results are written back into the smem tile and leave by a cp.async.bulk store.
// Tile IDs come from an atomic counter, so a tile's predecessors are always already running:
// no co-residency assumption.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "sam_algebra.h"

namespace sam {

template <typename T> struct Cfg;
// ITEMS odd (bank-conflict-free strided smem reads); NBUF = 3: the tile being scanned, the next
// tile being loaded, the previous tile being stored; MINB = CTAs per SM the registers must allow.
template <> struct Cfg<uint32_t> { static constexpr int ITEMS = 15, NBUF = 3, MINB = 4; };
template <> struct Cfg<float>    { static constexpr int ITEMS = 15, NBUF = 3, MINB = 4; };
template <> struct Cfg<uint64_t> { static constexpr int ITEMS = 15, NBUF = 3, MINB = 2; };
template <> struct Cfg<double>   { static constexpr int ITEMS = 15, NBUF = 3, MINB = 2; };

constexpr int MAX_WARPS = 8;
constexpr int MAX_THREADS = MAX_WARPS * 32;
constexpr uint64_t FLAG_AGG = 1, FLAG_INCL = 2;

enum StoreMode { STORE_BULK = 0, STORE_STRIPED = 1, STORE_NONE = 2 };

template <typename T, int K>
struct Params {
    const T* in;
    T* out;
    uint64_t n;          // elements in this stream
    uint64_t h;          // virtual index of in[0] (= lane phase, 0 <= h < s)
    uint64_t num_tiles;  // ceil((h + n) / T)
    uint32_t delta;      // byte offset of virtual element 0 inside its 16-B chunk
    int s, G, logG, sp, c, logc, Pw, W, Wn;
    int U, T_, Uw;
    int inclusive;
    int store_mode;
    const T* seed;        // [s][K] state before the stream per global lane, or null
    T* final_state;       // [s][K] or null
    int64_t last_e[MAXS]; // virtual index of lane m's last element, -1 if none
    uint64_t* status;
    T* aggv;
    T* inclv;
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned long long* epoch_ptr;
    T bc[K];              // b_d(ITEMS)
    T bw[K];              // b_d(Uw)
    T bu[K];              // b_d(U)
    T bwin[K];            // b_d(Wn*U)
    T bt[K][32];          // b_d(v*ITEMS), v < Pw       ([d][v])
    T bq[8][K];           // b_d(q*Uw),   q < c
    T bl[32][K];          // b_d(j*U),    j < Wn
};

// ------------------------------------------------------------------------------------------
// PTX helpers
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    uint64_t st;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 %0, [%1], %2;"
                 : "=l"(st) : "r"(smem_u32(bar)), "r"(bytes) : "memory");
    (void)st;
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    uint64_t st;
    asm volatile("mbarrier.arrive.shared::cta.b64 %0, [%1];" : "=l"(st) : "r"(smem_u32(bar)) : "memory");
    (void)st;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "SAM_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra SAM_WAIT_%=;\n}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar,
                                         uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        ::"r"(smem_u32(dst_smem)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src_smem, uint32_t bytes, uint64_t policy) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
                 ::"l"(dst), "r"(smem_u32(src_smem)), "r"(bytes), "l"(policy) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t ld_acquire_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// strong (L1-bypassing) loads/stores of the carry values
template <typename T> __device__ __forceinline__ T ld_relaxed(const T* p);
template <> __device__ __forceinline__ uint32_t ld_relaxed<uint32_t>(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint64_t ld_relaxed<uint64_t>(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ float ld_relaxed<float>(const float* p) {
    return __uint_as_float(ld_relaxed<uint32_t>((const uint32_t*)p));
}
template <> __device__ __forceinline__ double ld_relaxed<double>(const double* p) {
    return __longlong_as_double((long long)ld_relaxed<uint64_t>((const uint64_t*)p));
}
template <typename T> __device__ __forceinline__ void st_relaxed(T* p, T v);
template <> __device__ __forceinline__ void st_relaxed<uint32_t>(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
template <> __device__ __forceinline__ void st_relaxed<uint64_t>(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
template <> __device__ __forceinline__ void st_relaxed<float>(float* p, float v) {
    st_relaxed<uint32_t>((uint32_t*)p, __float_as_uint(v));
}
template <> __device__ __forceinline__ void st_relaxed<double>(double* p, double v) {
    st_relaxed<uint64_t>((uint64_t*)p, (uint64_t)__double_as_longlong(v));
}

template <typename T>
__device__ __forceinline__ T shfl_up(T v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
template <typename T>
__device__ __forceinline__ T shfl_down(T v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
template <typename T>
__device__ __forceinline__ T shfl_idx(T v, int l) { return __shfl_sync(0xffffffffu, v, l); }

template <typename T> struct IsInt { static constexpr bool value = false; };
template <> struct IsInt<uint32_t> { static constexpr bool value = true; };
template <> struct IsInt<uint64_t> { static constexpr bool value = true; };

// ------------------------------------------------------------------------------------------
// shared-memory layout
// ------------------------------------------------------------------------------------------
template <typename T, int K>
struct Smem {
    static constexpr int ITEMS = Cfg<T>::ITEMS;
    static constexpr int NBUF = Cfg<T>::NBUF;
    static constexpr int TMAX = MAX_THREADS * ITEMS;
    static constexpr int BUFB = ((TMAX * (int)sizeof(T) + 32) + 127) / 128 * 128;
    // offsets (bytes)
    static constexpr int OFF_BUF = 0;
    static constexpr int OFF_MBAR = OFF_BUF + NBUF * BUFB;
    static constexpr int OFF_TILE = OFF_MBAR + NBUF * 8;
    static constexpr int OFF_MISC = OFF_TILE + NBUF * 8;                 // epoch (u64)
    static constexpr int OFF_WAGG = ((OFF_MISC + 16) + 15) / 16 * 16;     // [64][K]
    static constexpr int OFF_WIN = OFF_WAGG + 64 * K * (int)sizeof(T);   // [64][K]
    static constexpr int OFF_LAGG = OFF_WIN + 64 * K * (int)sizeof(T);   // [8][K]
    static constexpr int OFF_LIN = OFF_LAGG + 8 * K * (int)sizeof(T);    // [8][K]
    static constexpr int OFF_BT = OFF_LIN + 8 * K * (int)sizeof(T);      // [K][32]
    static constexpr int OFF_BL = OFF_BT + K * 32 * (int)sizeof(T);      // [32][K]
    static constexpr int OFF_BQ = OFF_BL + 32 * K * (int)sizeof(T);      // [8][K]
    static constexpr int BYTES = OFF_BQ + 8 * K * (int)sizeof(T);
};

// ------------------------------------------------------------------------------------------
// the kernel
// ------------------------------------------------------------------------------------------
template <typename T, int K>
__global__ void __launch_bounds__(MAX_THREADS, Cfg<T>::MINB)
sam_scan_kernel(const __grid_constant__ Params<T, K> p) {
    using S = Smem<T, K>;
    constexpr int ITEMS = S::ITEMS;
    constexpr int NBUF = S::NBUF;
    static_assert(NBUF == 3, "ring: scanning / loading / storing");
    static_assert(ITEMS >= K, "exclusive shift needs ITEMS >= K");
    static_assert(ITEMS % 2 == 1, "ITEMS odd keeps the stride-s smem reads bank-conflict free");

    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* mbar = (uint64_t*)(smem + S::OFF_MBAR);
    int64_t* tile_of = (int64_t*)(smem + S::OFF_TILE);
    unsigned long long* sm_epoch = (unsigned long long*)(smem + S::OFF_MISC);
    T* wagg = (T*)(smem + S::OFF_WAGG);
    T* win = (T*)(smem + S::OFF_WIN);
    T* lagg = (T*)(smem + S::OFF_LAGG);
    T* lin = (T*)(smem + S::OFF_LIN);
    T* bt_s = (T*)(smem + S::OFF_BT);
    T* bl_s = (T*)(smem + S::OFF_BL);
    T* bq_s = (T*)(smem + S::OFF_BQ);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int s = p.s, G = p.G, c = p.c, Pw = p.Pw;
    const int NT = p.W * 32;
    const int Tt = p.T_;
    // thread <-> (lane m, lane positions [u*ITEMS, u*ITEMS + ITEMS))
    const int g = warp % p.sp, q = warp / p.sp;
    const int a = lane & (G - 1), v = lane >> p.logG;
    const int m = g * G + a;
    const int u = q * Pw + v;
    const int base_loc = u * ITEMS * s + m;  // element index inside the tile of item 0
    const uint64_t pol = policy_evict_first();

    // ---- prologue ----------------------------------------------------------------------
    for (int i = tid; i < K * 32; i += NT) bt_s[i] = (&p.bt[0][0])[i];
    for (int i = tid; i < 32 * K; i += NT) bl_s[i] = (&p.bl[0][0])[i];
    for (int i = tid; i < 8 * K; i += NT) bq_s[i] = (&p.bq[0][0])[i];

    auto issue_load = [&](int slot) -> bool {  // thread 0 only; returns false when exhausted
        unsigned long long t = atomicAdd(p.tile_ctr, 1ull);
        if (t >= p.num_tiles) {
            tile_of[slot] = -1;
            mbar_arrive(&mbar[slot]);
            return false;
        }
        tile_of[slot] = (int64_t)t;
        const uint64_t e0 = t * (uint64_t)Tt;
        const uint64_t lo = e0 > p.h ? e0 : p.h;
        const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
        const uintptr_t src_lo = (uintptr_t)p.in + (lo - p.h) * sizeof(T);
        const uintptr_t src_hi = (uintptr_t)p.in + (hi - p.h) * sizeof(T);
        const uintptr_t a16 = src_lo & ~(uintptr_t)15;
        const uintptr_t b16 = (src_hi + 15) & ~(uintptr_t)15;
        unsigned char* dst = smem + S::OFF_BUF + slot * S::BUFB + p.delta + (lo - e0) * sizeof(T) - (src_lo - a16);
        mbar_arrive_expect_tx(&mbar[slot], (uint32_t)(b16 - a16));
        bulk_g2s(dst, (const void*)a16, (uint32_t)(b16 - a16), &mbar[slot], pol);
        return true;
    };

    // Tile claims: one at start, then exactly one per processed tile, made right after the
    // tile's aggregate is published.  Claims are thus never bursty, so a tile's predecessor is
    // always claimed earlier by a CTA that starts it no later than one tile-time after.
    bool claiming = true;
    if (tid == 0) {
        for (int b = 0; b < NBUF; ++b) mbar_init(&mbar[b], 1);
        fence_mbar_init();
        *sm_epoch = *(volatile unsigned long long*)p.epoch_ptr;
        claiming = issue_load(0);
    }
    __syncthreads();
    const unsigned long long epoch = *sm_epoch;

    for (int it = 0;; ++it) {
        const int slot = it % NBUF;
        mbar_wait(&mbar[slot], (uint32_t)((it / NBUF) & 1));
        const int64_t tile = tile_of[slot];
        if (tile < 0) break;

        T* xs = (T*)(smem + S::OFF_BUF + slot * S::BUFB + p.delta);
        const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
        const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);

        // ---- a2/a3: load lane run, thread-serial zero-seeded recurrence ----------------
        T acc[K];
#pragma unroll
        for (int t = 0; t < K; ++t) acc[t] = T(0);
        if (!masked) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                T x = xs[base_loc + i * s];
                acc[0] += x;
#pragma unroll
                for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
            }
        } else {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                const int el = base_loc + i * s;
                const uint64_t ve = e0 + el;
                T x = (ve >= p.h && ve < p.h + p.n) ? xs[el] : T(0);
                acc[0] += x;
#pragma unroll
                for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
            }
        }

        // ---- a3: warp scan of thread states (order by order, plain shuffle scans) --------
        // e_{v+1} = M(ITEMS) e_v + a_v  =>  component t: e_{v+1}[t] = e_v[t] + z_v[t],
        // z_v[t] = a_v[t] + sum_{j<t} b_{t-j}(ITEMS) e_v[j]
        T e[K];
#pragma unroll
        for (int t = 0; t < K; ++t) {
            T z = acc[t];
#pragma unroll
            for (int j = 0; j < t; ++j) z += p.bc[t - j] * e[j];
            T y = z;
            for (int off = G; off < 32; off <<= 1) {
                T o = shfl_up(y, off);
                if (lane >= off) y += o;
            }
            if constexpr (IsInt<T>::value) {
                e[t] = y - z;
            } else {
                T o = shfl_up(y, G);
                e[t] = (lane >= G) ? o : T(0);
            }
            if (v == Pw - 1) wagg[(q * s + m) * K + t] = y;  // warp aggregate of lane m
        }
        __syncthreads();  // S1

        // ---- warp 0: block combine, publish, look-back, carries -------------------------
        if (warp == 0) {
            const int npair = s * c;
            T E0[K], E1[K];
            auto combine = [&](int pair, T* E) {
                const bool ok = pair < npair;
                const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
                T y_last[K];
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T z = ok ? wagg[(qq * s + mm) * K + t] : T(0);
#pragma unroll
                    for (int j = 0; j < t; ++j) z += p.bw[t - j] * E[j];
                    T y = z;
                    for (int off = 1; off < c; off <<= 1) {
                        T o = shfl_up(y, off);
                        if (qq >= off) y += o;
                    }
                    if constexpr (IsInt<T>::value) {
                        E[t] = y - z;
                    } else {
                        T o = shfl_up(y, 1);
                        E[t] = (qq >= 1) ? o : T(0);
                    }
                    y_last[t] = y;
                }
                if (ok && qq == c - 1) {
#pragma unroll
                    for (int t = 0; t < K; ++t) lagg[mm * K + t] = y_last[t];
                }
            };
            combine(lane, E0);
            if (npair > 32) combine(lane + 32, E1);
            __syncwarp();

            // tile aggregate A (lanes lane < s)
            T A[K], C[K];
            const bool lane_ok = lane < s;
            const int ml = lane_ok ? lane : 0;
#pragma unroll
            for (int t = 0; t < K; ++t) A[t] = lagg[ml * K + t];

            // seed of virtual tile -1 for lane ml: M(-1) applied for lanes before the phase
            auto seed_of = [&](int mm, T* out) {
                if (p.seed) {
#pragma unroll
                    for (int t = 0; t < K; ++t) out[t] = p.seed[mm * K + t];
                    if ((uint64_t)mm < p.h) {
#pragma unroll
                        for (int t = K - 1; t >= 1; --t) out[t] = out[t] - out[t - 1];
                    }
                } else {
#pragma unroll
                    for (int t = 0; t < K; ++t) out[t] = T(0);
                }
            };

            if (tile == 0) {
                seed_of(ml, C);
            } else {
                // a4: publish aggregate
                if (lane_ok) {
                    T* dst = p.aggv + ((size_t)tile * s + lane) * K;
#pragma unroll
                    for (int t = 0; t < K; ++t) st_relaxed(dst + t, A[t]);
                    __threadfence();
                }
                __syncwarp();
                if (lane == 0) st_release_u64(p.status + tile, (epoch << 2) | FLAG_AGG);
            }
            // prefetch: claim the next tile and start its load (overlaps look-back, pass 2, store)
            if (lane == 0 && claiming) {
                bulk_wait_read<1>();  // the slot being refilled was stored from 2 iterations ago
                claiming = issue_load((it + 1) % NBUF);
            }
            if (tile != 0) {

                // a5: decoupled look-back over windows of Wn tiles x s lanes
                const int Wn = p.Wn;
                const int jl = lane / s, mlb = lane - jl * s;
                const bool active = jl < Wn;
                T total[K], Pm[K];
#pragma unroll
                for (int t = 0; t < K; ++t) { total[t] = T(0); Pm[t] = (t == 0) ? T(1) : T(0); }
                int64_t basei = tile - 1;
                bool first = true;
                for (;;) {
                    const int64_t idx = basei - jl;
                    uint64_t flag = 0;
                    if (active && idx < 0) flag = FLAG_INCL;
                    // poll until the window is valid up to its nearest inclusive predecessor
                    // (tiles beyond that one are not needed, so they are not waited for)
                    int jin;
                    for (;;) {
                        if (active && flag == 0) {
                            const uint64_t st = ld_acquire_u64(p.status + idx);
                            flag = ((st >> 2) == epoch) ? (st & 3ull) : 0ull;
                        }
                        const unsigned im = __ballot_sync(0xffffffffu, active && flag == FLAG_INCL);
                        const unsigned iv = __ballot_sync(0xffffffffu, active && flag == 0);
                        jin = im ? (__ffs(im) - 1) / s : Wn;
                        const int jinv = iv ? (__ffs(iv) - 1) / s : Wn;
                        if (jinv == Wn || jin < jinv) break;
                    }
                    T Y[K];
                    if (active && jl <= jin) {
                        T X[K];
                        if (idx < 0) {
                            seed_of(mlb, X);
                        } else {
                            const T* src = ((jl == jin) ? p.inclv : p.aggv) + ((size_t)idx * s + mlb) * K;
#pragma unroll
                            for (int t = 0; t < K; ++t) X[t] = ld_relaxed(src + t);
                        }
                        // contribution M(jl*U) X
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            T acc2 = X[t];
#pragma unroll
                            for (int j = 0; j < t; ++j) acc2 += bl_s[jl * K + (t - j)] * X[j];
                            Y[t] = acc2;
                        }
                    } else {
#pragma unroll
                        for (int t = 0; t < K; ++t) Y[t] = T(0);
                    }
                    for (int off = 1; off < Wn; off <<= 1) {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            T o = shfl_down(Y[t], off * s);
                            if (jl + off < Wn) Y[t] += o;
                        }
                    }
                    // lanes jl == 0 hold the window sum; total += M(window offset) * Y
                    if (first) {
#pragma unroll
                        for (int t = 0; t < K; ++t) total[t] = Y[t];
                    } else {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            T acc2 = Y[t];
#pragma unroll
                            for (int j = 0; j < t; ++j) acc2 += Pm[t - j] * Y[j];
                            total[t] += acc2;
                        }
                    }
                    if (jin < Wn) break;
                    // next window: Pm <- Pm * M(Wn*U)  (truncated polynomial product)
                    {
                        T np[K];
#pragma unroll
                        for (int d = 0; d < K; ++d) {
                            T acc2 = T(0);
#pragma unroll
                            for (int e2 = 0; e2 <= d; ++e2) acc2 += Pm[e2] * p.bwin[d - e2];
                            np[d] = acc2;
                        }
#pragma unroll
                        for (int d = 0; d < K; ++d) Pm[d] = np[d];
                    }
                    basei -= Wn;
                    first = false;
                }
#pragma unroll
                for (int t = 0; t < K; ++t) C[t] = total[t];
            }

            // publish inclusive state of this tile: M(U) C + A
            if ((uint64_t)tile + 1 < p.num_tiles) {
                if (lane_ok) {
                    T* dst = p.inclv + ((size_t)tile * s + lane) * K;
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T acc2 = C[t] + A[t];
#pragma unroll
                        for (int j = 0; j < t; ++j) acc2 += p.bu[t - j] * C[j];
                        st_relaxed(dst + t, acc2);
                    }
                    __threadfence();
                }
                __syncwarp();
                if (lane == 0) st_release_u64(p.status + tile, (epoch << 2) | FLAG_INCL);
            }
            if (lane_ok) {
#pragma unroll
                for (int t = 0; t < K; ++t) lin[lane * K + t] = C[t];
            }
            __syncwarp();
            // per-warp incoming state C_{m,q} = M(q*Uw) C_m + E_{m,q}
            auto warp_in = [&](int pair, const T* E) {
                if (pair >= npair) return;
                const int mm = pair >> p.logc, qq = pair & (c - 1);
                T Cm[K];
#pragma unroll
                for (int t = 0; t < K; ++t) Cm[t] = lin[mm * K + t];
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T acc2 = Cm[t] + E[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) acc2 += bq_s[qq * K + (t - j)] * Cm[j];
                    win[(qq * s + mm) * K + t] = acc2;
                }
            };
            warp_in(lane, E0);
            if (npair > 32) warp_in(lane + 32, E1);
        }
        __syncthreads();  // S2

        // ---- a6: thread incoming state, seeded recurrence, outputs -------------------------
        T y[K];
        {
            T Cq[K];
#pragma unroll
            for (int t = 0; t < K; ++t) Cq[t] = win[(q * s + m) * K + t];
#pragma unroll
            for (int t = 0; t < K; ++t) {
                T acc2 = e[t] + Cq[t];
#pragma unroll
                for (int j = 0; j < t; ++j) acc2 += bt_s[(t - j) * 32 + v] * Cq[j];
                y[t] = acc2;
            }
        }
        // exclusive: first K outputs are y_K at positions before the thread's first item,
        // by backward differences of the incoming state: y_K[r0-1-d] = sum_t (-1)^t C(d,t) y[K-1-t]
        T hist[K];
        if (!p.inclusive) {
            T w[K];
#pragma unroll
            for (int t = 0; t < K; ++t) w[t] = y[t];
            // hist[d] = y_K at r0-1-d ; w holds successive backward differences
#pragma unroll
            for (int d = 0; d < K; ++d) {
                hist[d] = w[K - 1];
#pragma unroll
                for (int t = K - 1; t >= 1; --t) w[t] = w[t] - w[t - 1];
            }
        }

        const bool want_final = (p.final_state != nullptr);
        const bool store_smem = (p.store_mode != STORE_NONE);
        T ring[K];  // last K inclusive outputs (exclusive mode)
#pragma unroll
        for (int d = 0; d < K; ++d) ring[d] = hist[K - 1 - d];
        // ring[j] for j<K: y_K at r0-K+j ; consumed FIFO-style below
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const int el = base_loc + i * s;
            T x;
            if (!masked) {
                x = xs[el];
            } else {
                const uint64_t ve = e0 + el;
                x = (ve >= p.h && ve < p.h + p.n) ? xs[el] : T(0);
            }
            y[0] += x;
#pragma unroll
            for (int t = 1; t < K; ++t) y[t] += y[t - 1];
            T outv;
            if (p.inclusive) {
                outv = y[K - 1];
            } else {
                outv = ring[i % K];
                ring[i % K] = y[K - 1];
            }
            if (store_smem) xs[el] = outv;
            if (want_final && masked) {
                if ((int64_t)(e0 + el) == p.last_e[m]) {
#pragma unroll
                    for (int t = 0; t < K; ++t) p.final_state[m * K + t] = y[t];
                }
            }
        }
        if (want_final && !masked) {
            // the last element of a lane can sit in an unmasked tile only if it is the tile end
            const int64_t le = p.last_e[m];
            if (le >= (int64_t)(e0 + base_loc) && le == (int64_t)(e0 + base_loc + (ITEMS - 1) * s)) {
#pragma unroll
                for (int t = 0; t < K; ++t) p.final_state[m * K + t] = y[t];
            }
        }

        // ---- a7: store ---------------------------------------------------------------------
        if (p.store_mode == STORE_BULK) {
            fence_proxy_async_smem();
            __syncthreads();  // S3
            const uint64_t lo = e0 > p.h ? e0 : p.h;
            const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
            const uintptr_t ob = (uintptr_t)p.out + (lo - p.h) * sizeof(T);
            const uintptr_t oe = (uintptr_t)p.out + (hi - p.h) * sizeof(T);
            const uintptr_t bs = (ob + 15) & ~(uintptr_t)15;
            const uintptr_t be = oe & ~(uintptr_t)15;
            if (tid == 0) {
                if (be > bs) {
                    const unsigned char* src = (const unsigned char*)xs + (lo - e0) * sizeof(T) + (bs - ob);
                    bulk_s2g((void*)bs, src, (uint32_t)(be - bs), pol);
                }
                bulk_commit();
            }
            // partial 16-B chunks at the ends of the tile's output range: plain stores
            if (bs != ob || be != oe || be <= bs) {
                const int n_head = (int)((be > bs ? bs : oe) - ob) / (int)sizeof(T);
                const int n_tail = be > bs ? (int)(oe - be) / (int)sizeof(T) : 0;
                const int tot = n_head + n_tail;
                for (int j = tid; j < tot; j += NT) {
                    const uint64_t ve = (j < n_head) ? lo + j : (hi - n_tail) + (j - n_head);
                    p.out[ve - p.h] = xs[ve - e0];
                }
            }
        } else if (p.store_mode == STORE_STRIPED) {
            __syncthreads();  // S3
            const uint64_t lo = e0 > p.h ? e0 : p.h;
            const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
            for (uint64_t ve = lo + tid; ve < hi; ve += NT) p.out[ve - p.h] = xs[ve - e0];
        } else {
            __syncthreads();  // S3 (buffer reuse)
        }
        // make sure the final-state writes of a lane's last element land before kernel end
    }

    // ---- epilogue: drain bulk stores, reset counters for the next launch -----------------
    if (tid == 0) {
        bulk_wait<0>();
        __threadfence();
        const unsigned prev = atomicAdd(p.done_ctr, 1u);
        if (prev == gridDim.x - 1) {
            *(volatile unsigned long long*)p.tile_ctr = 0ull;
            *(volatile unsigned int*)p.done_ctr = 0u;
            __threadfence();
            atomicAdd(p.epoch_ptr, 1ull);
        }
    }
}

// Fold gathered shard payloads into the seed of `rank` (one thread per lane).
template <typename T>
__global__ void sam_fold_kernel(const unsigned char* payloads, size_t payload_bytes, int rank, int k,
                                int s, T* seed) {
    const int m = threadIdx.x;
    if (m < s) fold_payloads<T>(payloads, payload_bytes, rank, k, s, m, seed + (size_t)m * k);
}

// Payload header + lanes with no element in the stream: final state = seed (or 0).
template <typename T>
__global__ void sam_payload_init_kernel(unsigned char* payload, uint64_t n, uint64_t g, int k, int s,
                                        const T* seed, int write_header, T* final_state) {
    const int i = threadIdx.x;
    if (write_header && i == 0) {
        ((uint64_t*)payload)[0] = n;
        ((uint64_t*)payload)[1] = g;
    }
    if (i < s * k) {
        const int mm = i / k;
        if (lane_len(n, g, s, mm) == 0) final_state[i] = seed ? seed[i] : T(0);
    }
}

}  // namespace sam
