// sam_kernel.cuh -- single-pass order-k, tuple-s prefix sum for sm_100a.
//
// One kernel launch reads every input element once and writes every output element once
// (P:393-395): SAM's single-pass property, kept for any order and tuple
// size.  One CTA scans one tile of T = W*32*ITEMS elements (W warps):
//   a1  the CTA claims its tile from an atomic counter (so every predecessor tile belongs to a
//       CTA that is already running: no co-residency assumption) and one thread
//       pulls the whole tile into shared memory with a 1-D cp.async.bulk (TMA bulk engine);
//   a2  thread <-> (tuple lane m, ITEMS consecutive lane positions), read from smem at stride s;
//       a warp holds G = (largest power of two dividing s) lanes, 32/G threads each, so the
//       strided reads are bank-conflict free (ITEMS odd) and registers do not grow with s
//       (P:467-473);
//   a3  zero-seeded order-k local scan: thread-serial recurrence (k adds per element), warp scan
//       of thread states (k plain shuffle scans, order by order), block combine of warp states;
//       the paper's three-phase intra-block scan iterated per order;
//   a4  publish the tile's per-lane k-vector aggregate (one value per order; the s
//       lanes together).  Every published 64-bit word carries the launch's 32-bit
//       epoch tag beside (half) a value, so a reader validates each word by itself: the paper's
//       "local sum -> fence -> ready flag" becomes a single self-validating store
//       with no fence, and a reader needs ONE L2 round trip per look-back hop, not two;
//   a5  decoupled look-back: warp 0 reads a window of up to 128 predecessor tiles in one round
//       trip, finds the nearest one with an inclusive state and folds the aggregates between
//       with the carry operator (M(L) s + v).  This is the O(n) scheme the paper describes for
//       CUB and advises once the architectural factor grows (B200's
//       af is ~9x the paper's GPUs), made wide because B200 retires ~100+ tiles per microsecond;
//   a6  fused carry application: thread incoming state = M(L) carry + local prefix, then the
//       seeded recurrence produces the outputs (the binomial fix-up C(r+t-j, t-j));
//       exclusive = inclusive shifted by k lane positions (R1), the first k from
//       finite differences of the incoming state;
//   a7  results are written back into the smem tile and leave by a cp.async.bulk store.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "sam_algebra.h"

namespace sam {

template <typename T> struct Cfg;
// ITEMS odd (bank-conflict-free strided smem reads); MINB = CTAs per SM the registers must allow.
template <> struct Cfg<uint32_t> { static constexpr int ITEMS = 31, MINB = 4; };
template <> struct Cfg<float>    { static constexpr int ITEMS = 31, MINB = 4; };
template <> struct Cfg<uint64_t> { static constexpr int ITEMS = 31, MINB = 3; };
template <> struct Cfg<double>   { static constexpr int ITEMS = 31, MINB = 3; };

constexpr int MAX_WARPS = 8;
constexpr int MAX_THREADS = MAX_WARPS * 32;
constexpr int MAX_LB = 128;  // max predecessor tiles per look-back round trip

enum StoreMode { STORE_BULK = 0, STORE_STRIPED = 1, STORE_NONE = 2 };

// 64-bit tagged words per value: 1 for 32-bit types ([tag|value]), 2 for 64-bit ([tag|lo],[tag|hi])
template <typename T> struct TagW { static constexpr int W = sizeof(T) == 4 ? 1 : 2; };
// look-back windows per round trip (register budget: V*K*2W words per lane)
template <typename T, int K> struct LB {
    static constexpr int W = TagW<T>::W;
    static constexpr int V0 = 8 / (K * W);
    static constexpr int V = V0 < 1 ? 1 : (V0 > 4 ? 4 : V0);
};

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
    unsigned long long* carry;  // tagged carry words: [tile][m][t][agg W | incl W]
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned int* epoch_ptr;
    T bc[K];              // b_d(ITEMS)
    T bw[K];              // b_d(Uw)
    T bu[K];              // b_d(U)
    T bwin[K];            // b_d(Wn*V*U)   (one look-back round trip further)
    T bt[K][32];          // b_d(v*ITEMS),  v < Pw        ([d][v])
    T bq[8][K];           // b_d(q*Uw),     q < c
    T bl[MAX_LB][K];      // b_d(d*U),      d < Wn*V
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
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}"
                 ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
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
__device__ __forceinline__ void bulk_wait_read0() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void ld_relaxed_v2(const unsigned long long* p, unsigned long long& a,
                                              unsigned long long& b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// bit views of the element types
template <typename T> struct Bits;
template <> struct Bits<uint32_t> {
    static __device__ __forceinline__ uint64_t to(uint32_t v) { return v; }
    static __device__ __forceinline__ uint32_t from(uint64_t b) { return (uint32_t)b; }
};
template <> struct Bits<uint64_t> {
    static __device__ __forceinline__ uint64_t to(uint64_t v) { return v; }
    static __device__ __forceinline__ uint64_t from(uint64_t b) { return b; }
};
template <> struct Bits<float> {
    static __device__ __forceinline__ uint64_t to(float v) { return __float_as_uint(v); }
    static __device__ __forceinline__ float from(uint64_t b) { return __uint_as_float((uint32_t)b); }
};
template <> struct Bits<double> {
    static __device__ __forceinline__ uint64_t to(double v) { return (uint64_t)__double_as_longlong(v); }
    static __device__ __forceinline__ double from(uint64_t b) { return __longlong_as_double((long long)b); }
};

// publish value v of slot (tile, m, t), half = 0 (aggregate) or 1 (inclusive)
template <typename T>
__device__ __forceinline__ void put_tagged(unsigned long long* slot, int half, uint32_t tag, T v) {
    constexpr int W = TagW<T>::W;
    const uint64_t b = Bits<T>::to(v);
    const uint64_t hi = (uint64_t)tag << 32;
    if constexpr (W == 1) {
        st_relaxed_u64(slot + half, hi | (b & 0xffffffffull));
    } else {
        st_relaxed_u64(slot + 2 * half, hi | (b & 0xffffffffull));
        st_relaxed_u64(slot + 2 * half + 1, hi | (b >> 32));
    }
}

template <typename T>
__device__ __forceinline__ T shfl_up(T v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
template <typename T>
__device__ __forceinline__ T shfl_down(T v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }

template <typename T> struct IsInt { static constexpr bool value = false; };
template <> struct IsInt<uint32_t> { static constexpr bool value = true; };
template <> struct IsInt<uint64_t> { static constexpr bool value = true; };

// ------------------------------------------------------------------------------------------
// shared-memory layout
// ------------------------------------------------------------------------------------------
template <typename T, int K>
struct Smem {
    static constexpr int ITEMS = Cfg<T>::ITEMS;
    static constexpr int TMAX = MAX_THREADS * ITEMS;
    static constexpr int NBL = 32 * LB<T, K>::V;  // look-back binomial rows
    static constexpr int BUFB = ((TMAX * (int)sizeof(T) + 32) + 127) / 128 * 128;
    static constexpr int OFF_BUF = 0;
    static constexpr int OFF_MBAR = OFF_BUF + BUFB;                      // u64
    static constexpr int OFF_TILE = OFF_MBAR + 8;                        // i64 tile id
    static constexpr int OFF_TAG = OFF_TILE + 8;                         // u32 tag
    static constexpr int OFF_WAGG = (OFF_TAG + 8 + 15) / 16 * 16;        // [64][K] (also warp-in)
    static constexpr int OFF_LAGG = OFF_WAGG + 64 * K * (int)sizeof(T);  // [8][K]
    static constexpr int OFF_LIN = OFF_LAGG + 8 * K * (int)sizeof(T);    // [8][K]
    static constexpr int OFF_BT = OFF_LIN + 8 * K * (int)sizeof(T);      // [K][32]
    static constexpr int OFF_BL = OFF_BT + K * 32 * (int)sizeof(T);      // [NBL][K]
    static constexpr int OFF_BQ = OFF_BL + NBL * K * (int)sizeof(T);     // [8][K]
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
    constexpr int W2 = 2 * TagW<T>::W;  // tagged words per slot (aggregate + inclusive)
    constexpr int V = LB<T, K>::V;
    static_assert(ITEMS >= K, "exclusive shift needs ITEMS >= K");
    static_assert(ITEMS % 2 == 1, "ITEMS odd keeps the stride-s smem reads bank-conflict free");

    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* mbar = (uint64_t*)(smem + S::OFF_MBAR);
    int64_t* sm_tile = (int64_t*)(smem + S::OFF_TILE);
    uint32_t* sm_tag = (uint32_t*)(smem + S::OFF_TAG);
    T* wagg = (T*)(smem + S::OFF_WAGG);
    T* win = wagg;  // warp-in states overwrite the warp aggregates once those are consumed
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
    const int g = warp % p.sp, q = warp / p.sp;
    const int a = lane & (G - 1), v = lane >> p.logG;
    const int m = g * G + a;
    const int u = q * Pw + v;
    const int base_loc = u * ITEMS * s + m;  // element index inside the tile of item 0
    const uint64_t pol = policy_evict_first();

    // ---- a1: claim the tile and start its bulk load -----------------------------------------
    if (tid == 0) {
        mbar_init(mbar, 1);
        fence_mbar_init();
        const unsigned long long t = atomicAdd(p.tile_ctr, 1ull);
        *sm_tile = (int64_t)t;
        *sm_tag = *(volatile unsigned int*)p.epoch_ptr + 1u;  // tags are never 0 (zeroed workspace)
        const uint64_t e0 = t * (uint64_t)Tt;
        const uint64_t lo = e0 > p.h ? e0 : p.h;
        const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
        const uintptr_t src_lo = (uintptr_t)p.in + (lo - p.h) * sizeof(T);
        const uintptr_t src_hi = (uintptr_t)p.in + (hi - p.h) * sizeof(T);
        const uintptr_t a16 = src_lo & ~(uintptr_t)15;
        const uintptr_t b16 = (src_hi + 15) & ~(uintptr_t)15;
        unsigned char* dst = smem + S::OFF_BUF + p.delta + (lo - e0) * sizeof(T) - (src_lo - a16);
        mbar_arrive_expect_tx(mbar, (uint32_t)(b16 - a16));
        bulk_g2s(dst, (const void*)a16, (uint32_t)(b16 - a16), mbar, pol);
    }
    for (int i = tid; i < K * 32; i += NT) bt_s[i] = (&p.bt[0][0])[i];
    for (int i = tid; i < S::NBL * K; i += NT) bl_s[i] = (&p.bl[0][0])[i];
    for (int i = tid; i < 8 * K; i += NT) bq_s[i] = (&p.bq[0][0])[i];
    __syncthreads();
    const int64_t tile = *sm_tile;
    const uint32_t tag = *sm_tag;
    mbar_wait(mbar, 0);

    T* xs = (T*)(smem + S::OFF_BUF + p.delta);
    const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
    const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);

    // ---- a2/a3: lane run, thread-serial zero-seeded recurrence -------------------------------
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

    // ---- a3: warp scan of thread states (order by order, plain shuffle scans) ----------------
    // e_{v+1} = M(ITEMS) e_v + a_v  =>  e_{v+1}[t] = e_v[t] + z_v[t],
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

    // ---- warp 0: block combine, publish, look-back, carries ----------------------------------
    if (warp == 0) {
        const int npair = s * c;
        T E0[K], E1[K];
        auto combine = [&](int pair, T* E, T* yl) {
            const bool ok = pair < npair;
            const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
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
                yl[t] = y;
            }
            if (ok && qq == c - 1) {
#pragma unroll
                for (int t = 0; t < K; ++t) lagg[mm * K + t] = yl[t];
            }
        };
        {
            T yl[K];
            combine(lane, E0, yl);
            if (npair > 32) combine(lane + 32, E1, yl);
        }
        __syncwarp();

        const bool lane_ok = lane < s;
        const int ml = lane_ok ? lane : 0;
        T A[K], C[K];
#pragma unroll
        for (int t = 0; t < K; ++t) A[t] = lagg[ml * K + t];

        // seed of virtual tile -1 for lane mm: M(-1) applied for lanes before the phase
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
        unsigned long long* const carry_tile = p.carry + (size_t)tile * s * K * W2;

        if (tile == 0) {
            seed_of(ml, C);
        } else {
            // a4: publish the aggregate (self-validating tagged words, no fence needed)
            if (lane_ok) {
#pragma unroll
                for (int t = 0; t < K; ++t) put_tagged<T>(carry_tile + (lane * K + t) * W2, 0, tag, A[t]);
            }
            // a5: decoupled look-back.  lane = (jl, mlb): predecessor distance d = jl + Wn*vv (+ window base)
            const int Wn = p.Wn;
            const int jl = lane / s, mlb = lane - jl * s;
            const bool active = jl < Wn;
            const unsigned smask = (1u << s) - 1u;
            T total[K], Pm[K];
#pragma unroll
            for (int t = 0; t < K; ++t) { total[t] = T(0); Pm[t] = (t == 0) ? T(1) : T(0); }
            int64_t basei = tile - 1;
            bool first = true;
            for (;;) {
                unsigned long long w[V][K][W2];
                int st[V];  // 0 invalid, 1 aggregate valid, 2 inclusive valid, 3 beyond the seed
#pragma unroll
                for (int vv = 0; vv < V; ++vv) {
                    const int64_t idx = basei - jl - (int64_t)Wn * vv;
                    st[vv] = !active ? 3 : (idx == -1 ? 2 : (idx < -1 ? 3 : 0));
                }
                int dI;
                for (;;) {
#pragma unroll
                    for (int vv = 0; vv < V; ++vv) {
                        if (st[vv] == 0) {
                            const int64_t idx = basei - jl - (int64_t)Wn * vv;
                            const unsigned long long* src = p.carry + ((size_t)idx * s + mlb) * K * W2;
                            bool ag = true, in = true;
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                if constexpr (W2 == 2) {
                                    ld_relaxed_v2(src + t * 2, w[vv][t][0], w[vv][t][1]);
                                    ag &= (uint32_t)(w[vv][t][0] >> 32) == tag;
                                    in &= (uint32_t)(w[vv][t][1] >> 32) == tag;
                                } else {
                                    ld_relaxed_v2(src + t * 4, w[vv][t][0], w[vv][t][1]);
                                    ld_relaxed_v2(src + t * 4 + 2, w[vv][t][2], w[vv][t][3]);
                                    ag &= (uint32_t)(w[vv][t][0] >> 32) == tag && (uint32_t)(w[vv][t][1] >> 32) == tag;
                                    in &= (uint32_t)(w[vv][t][2] >> 32) == tag && (uint32_t)(w[vv][t][3] >> 32) == tag;
                                }
                            }
                            st[vv] = in ? 2 : (ag ? 1 : 0);
                        }
                    }
                    // nearest predecessor whose s lanes are all inclusive-valid, nearest invalid one
                    dI = 1 << 30;
                    int dX = 1 << 30;
#pragma unroll
                    for (int vv = 0; vv < V; ++vv) {
                        const unsigned bv = __ballot_sync(0xffffffffu, st[vv] >= 1);
                        const unsigned bi = __ballot_sync(0xffffffffu, st[vv] >= 2);
                        // lanes jl*s holding a whole valid group
                        unsigned gv = bv, gi = bi;
                        if (s > 1) {
                            gv = gi = 0;
                            for (int j = 0; j < Wn; ++j) {
                                if (((bv >> (j * s)) & smask) == smask) gv |= 1u << j;
                                if (((bi >> (j * s)) & smask) == smask) gi |= 1u << j;
                            }
                        }
                        const unsigned full = (Wn == 32) ? 0xffffffffu : ((1u << Wn) - 1u);
                        const unsigned inv = ~gv & full;
                        if (gi && dI == (1 << 30)) dI = Wn * vv + (__ffs(gi) - 1);
                        if (inv && dX == (1 << 30)) dX = Wn * vv + (__ffs(inv) - 1);
                    }
                    if (dI < dX || (dX == (1 << 30) && dI == (1 << 30))) break;
                }
                // fold: sum over d <= dI of M(d*U) X_d  (X = inclusive at dI, aggregates before)
                T Y[K];
#pragma unroll
                for (int t = 0; t < K; ++t) Y[t] = T(0);
#pragma unroll
                for (int vv = 0; vv < V; ++vv) {
                    const int d = jl + Wn * vv;
                    if (active && d <= dI && st[vv] != 3) {
                        T X[K];
                        const int64_t idx = basei - d;
                        if (idx == -1) {
                            seed_of(mlb, X);
                        } else {
                            const int half = (d == dI) ? 1 : 0;
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                if constexpr (W2 == 2) {
                                    X[t] = Bits<T>::from(w[vv][t][half] & 0xffffffffull);
                                } else {
                                    X[t] = Bits<T>::from((w[vv][t][2 * half] & 0xffffffffull) |
                                                         (w[vv][t][2 * half + 1] << 32));
                                }
                            }
                        }
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            T acc2 = X[t];
#pragma unroll
                            for (int j = 0; j < t; ++j) acc2 += bl_s[d * K + (t - j)] * X[j];
                            Y[t] += acc2;
                        }
                    }
                }
                for (int off = 1; off < Wn; off <<= 1) {
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T o = shfl_down(Y[t], off * s);
                        if (jl + off < Wn) Y[t] += o;
                    }
                }
                // lanes jl == 0 hold this round trip's sum; total += M(offset) Y
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
                if (dI < (1 << 30)) break;
                {   // Pm <- Pm * M(Wn*V*U)  (truncated polynomial product)
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
                basei -= (int64_t)Wn * V;
                first = false;
            }
#pragma unroll
            for (int t = 0; t < K; ++t) C[t] = total[t];
        }

        // publish the inclusive state of this tile: M(U) C + A
        if ((uint64_t)tile + 1 < p.num_tiles && lane_ok) {
#pragma unroll
            for (int t = 0; t < K; ++t) {
                T acc2 = C[t] + A[t];
#pragma unroll
                for (int j = 0; j < t; ++j) acc2 += p.bu[t - j] * C[j];
                put_tagged<T>(carry_tile + (lane * K + t) * W2, 1, tag, acc2);
            }
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

    // ---- a6: thread incoming state, seeded recurrence, outputs -------------------------------
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
    // exclusive: the first K outputs are y_K at positions before the thread's first item, by
    // backward differences of the incoming state: y_K[r0-1-d] = sum_t (-1)^t C(d,t) y[K-1-t]
    T ring[K];
    if (!p.inclusive) {
        T w[K];
#pragma unroll
        for (int t = 0; t < K; ++t) w[t] = y[t];
#pragma unroll
        for (int d = 0; d < K; ++d) {
            ring[K - 1 - d] = w[K - 1];  // y_K at r0-1-d
#pragma unroll
            for (int t = K - 1; t >= 1; --t) w[t] = w[t] - w[t - 1];
        }
    } else {
#pragma unroll
        for (int t = 0; t < K; ++t) ring[t] = T(0);
    }

    const bool want_final = (p.final_state != nullptr);
    const bool store_smem = (p.store_mode != STORE_NONE);
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
        } else {  // y_K of item i-K (ring slot i%K holds it), then remember y_K of item i
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
        // in an unmasked tile a lane's last element can only be the lane's last tile position
        if (p.last_e[m] == (int64_t)(e0 + base_loc + (ITEMS - 1) * s)) {
#pragma unroll
            for (int t = 0; t < K; ++t) p.final_state[m * K + t] = y[t];
        }
    }

    // ---- a7: store ----------------------------------------------------------------------------
    if (p.store_mode == STORE_BULK) {
        fence_proxy_async_smem();
        __syncthreads();  // S3
        const uint64_t lo = e0 > p.h ? e0 : p.h;
        const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
        const uintptr_t ob = (uintptr_t)p.out + (lo - p.h) * sizeof(T);
        const uintptr_t oe = (uintptr_t)p.out + (hi - p.h) * sizeof(T);
        const uintptr_t bs = (ob + 15) & ~(uintptr_t)15;
        const uintptr_t be = oe & ~(uintptr_t)15;
        if (tid == 0 && be > bs) {
            const unsigned char* src = (const unsigned char*)xs + (lo - e0) * sizeof(T) + (bs - ob);
            bulk_s2g((void*)bs, src, (uint32_t)(be - bs), pol);
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
        if (tid == 0) bulk_wait_read0();  // smem must outlive the bulk engine's read
    } else if (p.store_mode == STORE_STRIPED) {
        __syncthreads();  // S3
        const uint64_t lo = e0 > p.h ? e0 : p.h;
        const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
        for (uint64_t ve = lo + tid; ve < hi; ve += NT) p.out[ve - p.h] = xs[ve - e0];
    }

    // ---- epilogue: the last CTA resets the tile counter and advances the epoch ----------------
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

// Fold gathered shard payloads into the seed of `rank` (one thread per lane).
template <typename T>
__global__ void sam_fold_kernel(const unsigned char* payloads, size_t payload_bytes, int rank, int k,
                                int s, T* seed) {
    const int mm = threadIdx.x;
    if (mm < s) fold_payloads<T>(payloads, payload_bytes, rank, k, s, mm, seed + (size_t)mm * k);
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
