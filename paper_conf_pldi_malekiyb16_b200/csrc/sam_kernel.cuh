// sam_kernel.cuh -- single-pass order-k, tuple-s prefix sum for sm_100a.
//
// One kernel launch reads every input element once and writes every output element once
// (P:393-395): SAM's single-pass property, kept for any order and tuple
// size.  Persistent, warp-specialised CTAs (one per SM) stream tiles of
// T = W*32*ITEMS elements through a ring of NB shared-memory buffers:
//
//   producer warp  a1: claims tiles from an atomic counter, one at a time as buffers free up (so
//                  a claimed tile's predecessors all belong to running CTAs -- no co-residency
//                  assumption, cf. P:2475-2479 -- and claims stay interleaved across CTAs), pulls
//                  each tile into smem with a 1-D cp.async.bulk (TMA bulk engine, mbarrier
//                  completion) and a7: writes finished tiles back with cp.async.bulk stores.
//   compute warps  a2: thread <-> (tuple lane m, ITEMS consecutive lane positions), read from
//                  smem at stride s; a warp holds G = (largest power of two dividing s) lanes,
//                  32/G threads each, so the strided reads are bank-conflict free (ITEMS odd)
//                  and registers do not grow with s;
//                  a3: zero-seeded order-k local scan -- thread-serial recurrence (k adds per
//                  element), warp scan of thread states (k plain shuffle scans, order by order),
//                  block combine of warp states: the paper's three-phase intra-block scan
//                   iterated per order;
//                  a4: warp 0 publishes the tile's per-lane k-vector aggregate (one value per
//                  order; all s lanes together) right after the local
//                  scan -- never behind a look-back;
//                  a6: LAG tiles later, the fused carry application: thread incoming state =
//                  M(L) carry + local prefix, then the seeded recurrence produces the outputs
//                  (the binomial fix-up C(r+t-j, t-j)); exclusive = inclusive shifted by k lane
//                  positions (R1), the first k from finite differences of the state.
//   carry warp     a5: decoupled look-back per tile, overlapped with the compute warps' local
//                  scans of the next tiles.  Every published 64-bit word carries the launch's
//                  32-bit epoch tag beside (half) a value, so each word validates itself: the
//                  paper's "local sum -> fence -> ready flag" becomes one store with
//                  no fence, and a look-back hop is ONE L2 round trip over a window of up to 256
//                  predecessor tiles; it folds aggregates with the carry operator (M(L) s + v)
//                  back to the nearest inclusive state -- the O(n) scheme the paper describes for
//                  CUB and advises once the architectural factor grows
//                  (B200's af is ~9x the paper's GPUs).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

#include "sam_algebra.h"

namespace sam {

template <typename T> struct Cfg;
// ITEMS odd (bank-conflict-free strided smem reads); NB smem tile buffers; LAG = tiles between a
// tile's local scan and its carry application (the look-back's latency budget).
template <> struct Cfg<uint32_t> { static constexpr int ITEMS = 31, NB = 6, LAG = 2; };
template <> struct Cfg<float>    { static constexpr int ITEMS = 31, NB = 6, LAG = 2; };
template <> struct Cfg<uint64_t> { static constexpr int ITEMS = 15, NB = 6, LAG = 2; };
template <> struct Cfg<double>   { static constexpr int ITEMS = 15, NB = 6, LAG = 2; };

constexpr int MAX_CWARPS = 8;                      // compute warps
constexpr int NCARRY = 2;                          // carry (look-back) warps, alternating tiles
constexpr int SERVICE_WARPS = 2 + NCARRY;          // producer + aggregator + carry warps
constexpr int MAX_THREADS = (MAX_CWARPS + SERVICE_WARPS) * 32;
constexpr int MAX_LB = 256;                        // max predecessor tiles per look-back round trip
constexpr int TILE_THREADS = MAX_CWARPS * 32;

enum StoreMode { STORE_BULK = 0, STORE_STRIPED = 1, STORE_NONE = 2 };

// 64-bit tagged words per value: 1 for 32-bit types ([tag|value]), 2 for 64-bit ([tag|lo],[tag|hi])
template <typename T> struct TagW { static constexpr int W = sizeof(T) == 4 ? 1 : 2; };
// look-back windows per round trip (carry-warp register budget: V*K*2W <= 64 words per lane)
template <typename T, int K> struct LB {
    static constexpr int W2 = 2 * TagW<T>::W;
    static constexpr int V0 = 64 / (K * W2);
    static constexpr int V = V0 < 1 ? 1 : (V0 > 8 ? 8 : V0);
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
    unsigned long long* trace;  // optional per-tile event timestamps [tile][8] (diagnostics), or null
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
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n}" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}" : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
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
__device__ __forceinline__ void bulk_wait_all0() {
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// diagnostics: record event ev (0..7) of tile `tile` when tracing is on
#define SAM_TRACE(ev, tile)                                                        \
    do {                                                                           \
        if (p.trace) p.trace[(size_t)(tile) * 8 + (ev)] = globaltimer();           \
    } while (0)
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
    static constexpr int NB = Cfg<T>::NB;
    static constexpr int TMAX = TILE_THREADS * ITEMS;
    static constexpr int NBL = 32 * LB<T, K>::V;  // look-back binomial rows
    static constexpr int BUFB = ((TMAX * (int)sizeof(T) + 32) + 127) / 128 * 128;
    static constexpr int WQ = 64 * K;             // per-buffer warp states   [64][K]
    static constexpr int LA = 8 * K;              // per-buffer tile aggregate [8][K]
    static constexpr int OFF_BUF = 0;
    static constexpr int OFF_BAR = OFF_BUF + NB * BUFB;                  // 5 x NB mbarriers
    static constexpr int OFF_TILE = OFF_BAR + 5 * NB * 8;                // NB x i64
    static constexpr int OFF_TAG = OFF_TILE + NB * 8;                    // u32 tag, i32 end iteration
    static constexpr int OFF_WQ = (OFF_TAG + 8 + 15) / 16 * 16;          // NB x [64][K]
    static constexpr int OFF_LA = OFF_WQ + NB * WQ * (int)sizeof(T);     // NB x [8][K]
    static constexpr int OFF_BT = OFF_LA + NB * LA * (int)sizeof(T);     // [K][32]
    static constexpr int OFF_BL = OFF_BT + K * 32 * (int)sizeof(T);      // [NBL][K]
    static constexpr int OFF_BQ = OFF_BL + NBL * K * (int)sizeof(T);     // [8][K]
    static constexpr int BYTES = OFF_BQ + 8 * K * (int)sizeof(T);
};

// ------------------------------------------------------------------------------------------
// the kernel
// ------------------------------------------------------------------------------------------
template <typename T, int K>
__global__ void __launch_bounds__(MAX_THREADS, 1)
sam_scan_kernel(const __grid_constant__ Params<T, K> p) {
    using S = Smem<T, K>;
    constexpr int ITEMS = S::ITEMS;
    constexpr int NB = S::NB;
    constexpr int LAG = Cfg<T>::LAG;
    constexpr int W2 = 2 * TagW<T>::W;  // tagged words per slot (aggregate + inclusive)
    constexpr int V = LB<T, K>::V;
    static_assert(ITEMS >= K, "exclusive shift needs ITEMS >= K");
    static_assert(ITEMS % 2 == 1, "ITEMS odd keeps the stride-s smem reads bank-conflict free");
    static_assert(NB >= LAG + 3, "ring: LAG+1 tiles awaiting carries, one storing, one loading");

    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* bar_full = (uint64_t*)(smem + S::OFF_BAR);
    uint64_t* bar_agg = bar_full + NB;
    uint64_t* bar_carry = bar_agg + NB;
    uint64_t* bar_stored = bar_carry + NB;
    uint64_t* bar_p1 = bar_stored + NB;
    int64_t* tile_of = (int64_t*)(smem + S::OFF_TILE);
    uint32_t* sm_tag = (uint32_t*)(smem + S::OFF_TAG);
    volatile int* sm_end = (volatile int*)(smem + S::OFF_TAG + 4);
    T* wq_all = (T*)(smem + S::OFF_WQ);
    T* la_all = (T*)(smem + S::OFF_LA);
    T* bt_s = (T*)(smem + S::OFF_BT);
    T* bl_s = (T*)(smem + S::OFF_BL);
    T* bq_s = (T*)(smem + S::OFF_BQ);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int s = p.s, c = p.c;
    const int NW = p.W;          // compute warps
    const int NCT = NW * 32;     // compute threads
    const int Tt = p.T_;
    const uint64_t pol = policy_evict_first();

    // ---- prologue: barriers, tables, epoch tag -------------------------------------------------
    if (tid == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(&bar_full[b], 1);
            mbar_init(&bar_agg[b], 32);
            mbar_init(&bar_carry[b], 32);
            mbar_init(&bar_stored[b], NCT);
            mbar_init(&bar_p1[b], NCT);
        }
        fence_mbar_init();
        *sm_tag = *(volatile unsigned int*)p.epoch_ptr + 1u;  // tags are never 0 (zeroed workspace)
        *sm_end = -1;
    }
    for (int i = tid; i < K * 32; i += blockDim.x) bt_s[i] = (&p.bt[0][0])[i];
    for (int i = tid; i < S::NBL * K; i += blockDim.x) bl_s[i] = (&p.bl[0][0])[i];
    for (int i = tid; i < 8 * K; i += blockDim.x) bq_s[i] = (&p.bq[0][0])[i];
    __syncthreads();
    const uint32_t tag = *sm_tag;

    if (warp == NW) {
        // =========================== producer warp: claims, loads, stores ======================
        if (lane == 0) {
            auto store_tile = [&](int b) {
                const int64_t tile = tile_of[b];
                if (p.store_mode != STORE_BULK || tile < 0) return;
                const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
                const uint64_t lo = e0 > p.h ? e0 : p.h;
                const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
                const uintptr_t ob = (uintptr_t)p.out + (lo - p.h) * sizeof(T);
                const uintptr_t oe = (uintptr_t)p.out + (hi - p.h) * sizeof(T);
                const uintptr_t bs = (ob + 15) & ~(uintptr_t)15;
                const uintptr_t be = oe & ~(uintptr_t)15;
                if (be > bs) {
                    const unsigned char* src =
                        smem + S::OFF_BUF + b * S::BUFB + p.delta + (lo - e0) * sizeof(T) + (bs - ob);
                    bulk_s2g((void*)bs, src, (uint32_t)(be - bs), pol);
                    bulk_commit();
                }
            };
            int j = 0;
            for (;; ++j) {
                const int b = j % NB;
                if (j >= NB) {  // buffer b last held iteration j-NB: store it, wait for the read
                    const int jo = j - NB;
                    mbar_wait(&bar_stored[b], (uint32_t)((jo / NB) & 1));
                    if (tile_of[b] >= 0) SAM_TRACE(7, tile_of[b]);
                    store_tile(b);
                    bulk_wait_read0();
                }
                const unsigned long long t = atomicAdd(p.tile_ctr, 1ull);
                if (t >= p.num_tiles) {
                    tile_of[b] = -1;
                    mbar_arrive(&bar_full[b]);
                    break;
                }
                tile_of[b] = (int64_t)t;
                SAM_TRACE(0, t);
                const uint64_t e0 = t * (uint64_t)Tt;
                const uint64_t lo = e0 > p.h ? e0 : p.h;
                const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
                const uintptr_t src_lo = (uintptr_t)p.in + (lo - p.h) * sizeof(T);
                const uintptr_t src_hi = (uintptr_t)p.in + (hi - p.h) * sizeof(T);
                const uintptr_t a16 = src_lo & ~(uintptr_t)15;
                const uintptr_t b16 = (src_hi + 15) & ~(uintptr_t)15;
                unsigned char* dst =
                    smem + S::OFF_BUF + b * S::BUFB + p.delta + (lo - e0) * sizeof(T) - (src_lo - a16);
                mbar_arrive_expect_tx(&bar_full[b], (uint32_t)(b16 - a16));
                bulk_g2s(dst, (const void*)a16, (uint32_t)(b16 - a16), &bar_full[b], pol);
            }
            // drain: iterations loaded but not yet stored
            for (int jo = (j - NB + 1 > 0 ? j - NB + 1 : 0); jo < j; ++jo) {
                const int b = jo % NB;
                mbar_wait(&bar_stored[b], (uint32_t)((jo / NB) & 1));
                store_tile(b);
            }
            bulk_wait_all0();
        }
    } else if (warp == NW + 1) {
        // =========================== aggregator warp: block combine, aggregate publish ===========
        const int npair = s * c;
        for (int i = 0;; ++i) {
            const int b = i % NB;
            mbar_wait(&bar_full[b], (uint32_t)((i / NB) & 1));
            const int64_t tile = tile_of[b];
            if (tile < 0) {  // end of stream: the carry warps poll this marker while they wait
                if (lane == 0) *sm_end = i;
                break;
            }
            mbar_wait(&bar_p1[b], (uint32_t)((i / NB) & 1));
            if (lane == 0) SAM_TRACE(2, tile);
            T* wq = wq_all + b * S::WQ;
            T* la = la_all + b * S::LA;
            for (int pair = lane; pair < 64; pair += 32) {
                const bool ok = pair < npair;
                const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
                T E[K], yl[K];
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T z = ok ? wq[(qq * s + mm) * K + t] : T(0);
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
                __syncwarp();
                if (ok) {
#pragma unroll
                    for (int t = 0; t < K; ++t) wq[(qq * s + mm) * K + t] = E[t];  // warp-exclusive prefix
                    if (qq == c - 1) {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            la[mm * K + t] = yl[t];
                            if (tile > 0) {  // a4: publish the tile aggregate
                                put_tagged<T>(p.carry + (((size_t)tile * s + mm) * K + t) * W2, 0, tag, yl[t]);
                            }
                        }
                    }
                }
            }
            __syncwarp();
            if (lane == 0) SAM_TRACE(3, tile);
            mbar_arrive(&bar_agg[b]);
        }
    } else if (warp >= NW + 2) {
        // =========================== carry warps: look-back, inclusive states ===================
        const int npair = s * c;
        for (int i = warp - (NW + 2);; i += NCARRY) {
            const int b = i % NB;
            bool ended = false;
            while (!mbar_try_wait(&bar_agg[b], (uint32_t)((i / NB) & 1))) {
                const int end = *sm_end;
                if (end >= 0 && i >= end) { ended = true; break; }
            }
            if (__any_sync(0xffffffffu, ended)) break;
            const int64_t tile = tile_of[b];
            if (lane == 0) SAM_TRACE(4, tile);
            T* wq = wq_all + b * S::WQ;
            const T* la = la_all + b * S::LA;
            const bool lane_ok = lane < s;
            const int ml = lane_ok ? lane : 0;
            T A[K], C[K];
#pragma unroll
            for (int t = 0; t < K; ++t) A[t] = la[ml * K + t];

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
                // a5: decoupled look-back.  lane = (jl, mlb): predecessor distance d = jl + Wn*vv
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
                                        ag &= (uint32_t)(w[vv][t][0] >> 32) == tag &&
                                              (uint32_t)(w[vv][t][1] >> 32) == tag;
                                        in &= (uint32_t)(w[vv][t][2] >> 32) == tag &&
                                              (uint32_t)(w[vv][t][3] >> 32) == tag;
                                    }
                                }
                                st[vv] = in ? 2 : (ag ? 1 : 0);
                            }
                        }
                        // nearest predecessor whose s lanes are all inclusive-valid / nearest invalid
                        dI = 1 << 30;
                        int dX = 1 << 30;
#pragma unroll
                        for (int vv = 0; vv < V; ++vv) {
                            const unsigned bv = __ballot_sync(0xffffffffu, st[vv] >= 1);
                            const unsigned bi = __ballot_sync(0xffffffffu, st[vv] >= 2);
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
            // per-warp incoming states C_{m,q} = M(q*Uw) C_m + E_{m,q}  (E in wq, from the combine)
            for (int pair = lane; pair < 64; pair += 32) {
                const bool ok = pair < npair;
                const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
                T Cm[K];
#pragma unroll
                for (int t = 0; t < K; ++t) Cm[t] = shfl_idx(C[t], mm);
                if (ok) {
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T acc2 = Cm[t] + wq[(qq * s + mm) * K + t];
#pragma unroll
                        for (int j = 0; j < t; ++j) acc2 += bq_s[qq * K + (t - j)] * Cm[j];
                        wq[(qq * s + mm) * K + t] = acc2;
                    }
                }
            }
            __syncwarp();
            if (lane == 0) SAM_TRACE(5, tile);
            mbar_arrive(&bar_carry[b]);
        }
    } else {
        // =========================== compute warps ===============================================
        const int G = p.G, Pw = p.Pw;
        const int g = warp % p.sp, q = warp / p.sp;
        const int a = lane & (G - 1), v = lane >> p.logG;
        const int m = g * G + a;
        const int u = q * Pw + v;
        const int base_loc = u * ITEMS * s + m;  // element index inside the tile of item 0

        // a6 for iteration `it` (tile `tile`, local exclusive state e)
        auto carry_apply = [&](int it, int64_t tile, const T* e) {
            const int b = it % NB;
            mbar_wait(&bar_carry[b], (uint32_t)((it / NB) & 1));
            if (tid == 0) SAM_TRACE(6, tile);
            T* xs = (T*)(smem + S::OFF_BUF + b * S::BUFB + p.delta);
            const T* wq = wq_all + b * S::WQ;
            const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
            const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);
            T y[K];
            {
                T Cq[K];
#pragma unroll
                for (int t = 0; t < K; ++t) Cq[t] = wq[(q * s + m) * K + t];
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T acc2 = e[t] + Cq[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) acc2 += bt_s[(t - j) * 32 + v] * Cq[j];
                    y[t] = acc2;
                }
            }
            // exclusive: the first K outputs are y_K at positions before the thread's first item,
            // by backward differences of the incoming state: y_K[r0-1-d] = sum_t (-1)^t C(d,t) y[K-1-t]
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
            // output bytes outside the bulk-store range [bs, be) are stored by the owning thread
            const uint64_t lo = e0 > p.h ? e0 : p.h;
            const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
            const uintptr_t ob = (uintptr_t)p.out + (lo - p.h) * sizeof(T);
            const uintptr_t oe = (uintptr_t)p.out + (hi - p.h) * sizeof(T);
            const uintptr_t bs = (ob + 15) & ~(uintptr_t)15;
            const uintptr_t be = oe & ~(uintptr_t)15;
            const bool direct_edges = (p.store_mode == STORE_BULK) && (bs != ob || be != oe || be <= bs);
            // does this tile hold the last element of some lane (final-state write)?
            bool has_final = false;
            if (p.final_state != nullptr) {
                for (int mm = 0; mm < s; ++mm)
                    has_final |= (p.last_e[mm] >= (int64_t)e0 && p.last_e[mm] < (int64_t)(e0 + Tt));
            }
            const bool slow = masked || direct_edges || has_final;
            if (slow || p.store_mode != STORE_NONE) {
                // per-item loop, specialised so the common case carries no per-element checks
                auto items = [&](auto excl_tag, auto slow_tag) {
                    constexpr bool EXCL = decltype(excl_tag)::value;
                    constexpr bool SLOW = decltype(slow_tag)::value;
#pragma unroll
                    for (int i = 0; i < ITEMS; ++i) {
                        const int el = base_loc + i * s;
                        T x;
                        bool valid = true;
                        uint64_t ve = 0;
                        if constexpr (SLOW) {
                            ve = e0 + el;
                            valid = !masked || (ve >= p.h && ve < p.h + p.n);
                            x = valid ? xs[el] : T(0);
                        } else {
                            x = xs[el];
                        }
                        y[0] += x;
#pragma unroll
                        for (int t = 1; t < K; ++t) y[t] += y[t - 1];
                        T outv;
                        if constexpr (EXCL) {  // y_K of item i-K (ring slot i%K), then remember item i
                            outv = ring[i % K];
                            ring[i % K] = y[K - 1];
                        } else {
                            outv = y[K - 1];
                        }
                        if constexpr (SLOW) {
                            if (p.store_mode != STORE_NONE) xs[el] = outv;
                            if (direct_edges && valid) {
                                const uintptr_t ad = (uintptr_t)(p.out + (ve - p.h));
                                if (ad < bs || ad >= be || be <= bs) p.out[ve - p.h] = outv;
                            }
                            if (has_final && valid && (int64_t)ve == p.last_e[m]) {
#pragma unroll
                                for (int t = 0; t < K; ++t) p.final_state[m * K + t] = y[t];
                            }
                        } else {
                            xs[el] = outv;
                        }
                    }
                };
                using TT = std::true_type;
                using FF = std::false_type;
                if (p.inclusive) {
                    if (slow) items(FF{}, TT{}); else items(FF{}, FF{});
                } else {
                    if (slow) items(TT{}, TT{}); else items(TT{}, FF{});
                }
            }
            if (p.store_mode == STORE_BULK) {
                fence_proxy_async_smem();
            } else if (p.store_mode == STORE_STRIPED) {
                named_bar_sync(2, NCT);
                for (uint64_t ve = lo + tid; ve < hi; ve += NCT) p.out[ve - p.h] = xs[ve - e0];
            }
            mbar_arrive(&bar_stored[b]);
        };

        T eq[LAG][K];
        int64_t tq[LAG];
        int i = 0;
        for (;; ++i) {
            const int b = i % NB;
            mbar_wait(&bar_full[b], (uint32_t)((i / NB) & 1));
            const int64_t tile = tile_of[b];
            if (tile < 0) break;
            if (tid == 0) SAM_TRACE(1, tile);
            T* xs = (T*)(smem + S::OFF_BUF + b * S::BUFB + p.delta);
            T* wq = wq_all + b * S::WQ;
            const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
            const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);

            // ---- a2/a3: lane run, thread-serial zero-seeded recurrence ----------------------
            T acc[K];
#pragma unroll
            for (int t = 0; t < K; ++t) acc[t] = T(0);
            if (!masked) {
#pragma unroll
                for (int it = 0; it < ITEMS; ++it) {
                    const T x = xs[base_loc + it * s];
                    acc[0] += x;
#pragma unroll
                    for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
                }
            } else {
#pragma unroll
                for (int it = 0; it < ITEMS; ++it) {
                    const int el = base_loc + it * s;
                    const uint64_t ve = e0 + el;
                    const T x = (ve >= p.h && ve < p.h + p.n) ? xs[el] : T(0);
                    acc[0] += x;
#pragma unroll
                    for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
                }
            }
            // ---- a3: warp scan of thread states (order by order, plain shuffle scans) -------
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
                if (v == Pw - 1) wq[(q * s + m) * K + t] = y;  // warp aggregate of lane m
            }
            mbar_arrive(&bar_p1[b]);  // warp states ready for the aggregator warp

            // ---- a6 for the tile LAG iterations back ------------------------------------------
            if (i >= LAG) carry_apply(i - LAG, tq[0], eq[0]);
#pragma unroll
            for (int j = 0; j + 1 < LAG; ++j) {
                tq[j] = tq[j + 1];
#pragma unroll
                for (int t = 0; t < K; ++t) eq[j][t] = eq[j + 1][t];
            }
            tq[LAG - 1] = tile;
#pragma unroll
            for (int t = 0; t < K; ++t) eq[LAG - 1][t] = e[t];
        }
        // drain the tiles still waiting for their carries
#pragma unroll
        for (int j = 0; j < LAG; ++j) {
            const int it = i - LAG + j;
            if (it >= 0) carry_apply(it, tq[j], eq[j]);
        }
    }

    // ---- epilogue: the last CTA resets the tile counter and advances the epoch ----------------
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
