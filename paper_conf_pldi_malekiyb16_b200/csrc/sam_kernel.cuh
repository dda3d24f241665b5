// sam_kernel.cuh -- single-pass order-k, tuple-s prefix sum for sm_100a.
//
// One kernel launch reads every input element once from HBM and writes every output element
// once: SAM's single-pass property, kept for any order and
// tuple size.  Persistent, warp-specialised CTAs (one per SM) stream tiles of
// T = W*32*ITEMS elements:
//
//   producer warp   a1: walks this CTA's static schedule (super-tiles b, b+P, b+2P, ..., P = the
//                   co-resident grid of a cooperative launch) at most PF tiles ahead of the local
//                   scans, and pulls each tile from HBM into a ring of NB1 smem buffers with a 1-D
//                   cp.async.bulk (TMA bulk engine) marked L2::evict_last.  When the tile's carry
//                   is known it pulls the same bytes again -- now from the 126 MB L2 (~18 TB/s vs
//                   ~7 TB/s HBM) -- into a second ring of NB2 buffers, and a7: writes the finished
//                   tile back with a cp.async.bulk store.  The carry's latency is spent with the
//                   tile parked in L2, not in shared memory, so it does not throttle the stream.
//   compute warps   a2: thread <-> (tuple lane m, ITEMS consecutive lane positions), read from
//                   smem at stride s; a warp holds G = (largest power of two dividing s) lanes,
//                   32/G threads each, so the strided reads are bank-conflict free (ITEMS odd)
//                   and registers do not grow with s;
//                   a3: zero-seeded order-k local scan -- thread-serial recurrence (k adds per
//                   element) and a warp scan of thread states (k plain shuffle scans, order by
//                   order): the paper's three-phase intra-block scan iterated per
//                   order;
//                   a6: once the carry is known, the fused carry application: thread incoming
//                   state = M(L) carry + local prefix, then the seeded recurrence produces the
//                   outputs (the binomial fix-up C(r+t-j, t-j)); exclusive = inclusive shifted by
//                   k lane positions (R1), the first k from finite differences.
//                   A loaded tile's local scan always goes first (its aggregate gates other
//                   CTAs' carry folds); up to LAG tiles may await their carries.
//   aggregator warp a3/a4: combines the warp states of a tile and publishes its per-lane k-vector
//                   aggregate (one value per order; all s lanes).
//   carry warps     a5: SAM's carry scheme on a static schedule: the carry into
//                   super-tile S is this CTA's own inclusive state after S-P (handed over in
//                   shared memory) advanced over the P-1 aggregates the other CTAs published in
//                   between, read in windows (one L2 round trip each) and folded with the carry
//                   operator (M(L) s + v).  Every published 64-bit word carries the launch's
//                   32-bit epoch tag beside (half) a value, so each word validates itself: the
//                   paper's "local sum -> fence -> ready flag" becomes one store
//                   with no fence.  All P CTAs must be co-resident (cooperative launch); there
//                   is no inclusive chain between CTAs, only between a CTA's own super-tiles.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string.h>

#include <type_traits>

#include "sam_algebra.h"

namespace sam {

template <typename T> struct Cfg;
// ITEMS odd (bank-conflict-free strided smem reads); NB1 / NB2 smem buffers for local scans / carry
// application + store; LAG = max tiles between local scan and carry application (the carry fold's
// latency budget, states in registers); PF = max claimed-but-unscanned tiles per CTA.
template <> struct Cfg<uint32_t> { static constexpr int ITEMS = 27; };
template <> struct Cfg<float>    { static constexpr int ITEMS = 27; };
template <> struct Cfg<uint64_t> { static constexpr int ITEMS = 13; };
template <> struct Cfg<double>   { static constexpr int ITEMS = 13; };
// VEC (tuple 1, 16-B aligned input): a thread's items are contiguous and 16-B aligned, read and
// written with 128-bit shared-memory accesses (ITEMS*sizeof(T) = 112 B: the 8 addresses of a
// quarter-warp phase fall in distinct 16-B bank groups, conflict free)
template <typename T, bool VEC> struct Items {
    static constexpr int V = VEC ? 112 / (int)sizeof(T) : Cfg<T>::ITEMS;
};
// 128-bit shared-memory load / store of N consecutive elements (16-B aligned)
template <typename T, int N>
__device__ __forceinline__ void lds_vec(const T* p, T (&d)[N]) {
    constexpr int E = 16 / (int)sizeof(T);
    if constexpr (N % E != 0) {  // not vectorisable (never taken at run time: VEC kernels only)
#pragma unroll
        for (int i = 0; i < N; ++i) d[i] = p[i];
        return;
    }
#pragma unroll
    for (int q = 0; q < N / E; ++q) {
        const uint4 v = reinterpret_cast<const uint4*>(p)[q];
        T t[E];
        memcpy(t, &v, 16);
#pragma unroll
        for (int j = 0; j < E; ++j) d[q * E + j] = t[j];
    }
}
template <typename T, int N>
__device__ __forceinline__ void sts_vec(T* p, const T (&d)[N]) {
    constexpr int E = 16 / (int)sizeof(T);
    if constexpr (N % E != 0) {
#pragma unroll
        for (int i = 0; i < N; ++i) p[i] = d[i];
        return;
    }
#pragma unroll
    for (int q = 0; q < N / E; ++q) {
        T t[E];
#pragma unroll
        for (int j = 0; j < E; ++j) t[j] = d[q * E + j];
        uint4 v;
        memcpy(&v, t, 16);
        reinterpret_cast<uint4*>(p)[q] = v;
    }
}
// Pipeline shape by per-thread state size K * sizeof(T) (struct Lag below):
//   <= 8 B : 3 local-scan buffers, 4 carry buffers, pending states in smem (LAG = 12)
//   <= 16 B: 3 + 2 buffers, pending states in smem (LAG = 8)
//   larger : 3 + 2 buffers, pending states in an L2-resident global scratch (LAG = 8)
// super-tile sizes (tiles per carry unit) come from the launch (MMAX, the autotune table); warp roles
// (carry warps, split compute groups) from struct Threads.  The SAM_* macros are compile-time overrides
// for experiments (tools/build_variant.py).  (Pending states <= 16 B in smem since round 1, larger ones in
// global scratch since round 2.)
#ifndef SAM_LAG_SMALL
#define SAM_LAG_SMALL 12
#endif
// SAM_EARLY_RELOAD: 1 = re-fetch a tile into a carry buffer as soon as its local scan is done, 2 = as
// soon as its super-tile's carry fold starts (one L2 round trip before the carry is expected) (the
// carry application then also waits for the carry) instead of once its carry is known
#ifndef SAM_EARLY_RELOAD
#define SAM_EARLY_RELOAD 0
#endif
// back-off (ns) of the carry-fold re-polls, of idle compute warps and of the idle producer
#ifndef SAM_POLL_NS
#define SAM_POLL_NS 0
#endif
#ifndef SAM_IDLE_NS
#define SAM_IDLE_NS 32
#endif
#ifndef SAM_PROD_NS
#define SAM_PROD_NS 16
#endif
// orders >= SAM_KS_MIN_K scan thread/warp k-vector states Kogge-Stone style, lower orders order by order
#ifndef SAM_TRANSFORM
#define SAM_TRANSFORM 1
#endif
// carry folds read their aggregates through one bulk copy into a smem landing buffer
#ifndef SAM_LAND
#define SAM_LAND 1
#endif
#ifndef SAM_TR32_MIN_K
#define SAM_TR32_MIN_K 2
#endif
#ifndef SAM_KS_MIN_K
#define SAM_KS_MIN_K 3
#endif
#ifndef SAM_LAG8
#define SAM_LAG8 12
#endif
#ifndef SAM_LAG16
#define SAM_LAG16 8
#endif
// max tiles per super-tile for states > 8 B (the carry team's work is per super-tile)
#ifndef SAM_MMAX_BIG
#define SAM_MMAX_BIG 2
#endif
// 8-byte states of up to SAM_SPLIT_MAXB bytes (int64 order 3) also get the two warp groups, their
// pending states in L2: 22 warps cap registers at 80, which order 3 fits without spills (measured
// +17% int64 k=3, +38% int64 k=3 s=3; orders >= 4 spill and lose, profiles/r2b_ab_splitbig.txt)
#ifndef SAM_SPLIT_BIG
#define SAM_SPLIT_BIG 1
#endif
#ifndef SAM_SPLIT_MAXB
#define SAM_SPLIT_MAXB 24
#endif
#ifndef SAM_SPLIT_MIN_K
#define SAM_SPLIT_MIN_K 2
#endif
// states of 17..32 B (int32 orders 5-8, int64 orders 3-4): pending in shared memory, LAG 6
#ifndef SAM_SMEM32
#define SAM_SMEM32 1
#endif
#ifndef SAM_LAG32
#define SAM_LAG32 6
#endif
#ifndef SAM_GPEND
#define SAM_GPEND 1
#endif
#ifndef SAM_LAGG
#define SAM_LAGG 8
#endif
// states of 33..64 B (int64 orders 5-8) without SAM_GPEND: pending in shared memory, LAG 4
#ifndef SAM_SMEM64
#define SAM_SMEM64 1
#endif
#ifndef SAM_LAG64
#define SAM_LAG64 4
#endif
template <typename T, int K> struct Lag {
    static constexpr int SB = K * (int)sizeof(T);
    static constexpr bool BIG32 = SAM_SMEM32 && SB > 16 && SB <= 32;
    static constexpr bool BIG64 = SAM_SMEM64 && SB > 32;
    // states > 16 B: pending in global memory (L2-resident scratch), so the pipeline depth is not
    // bounded by shared memory
    static constexpr bool GPEND = SAM_GPEND && SB > 16;
    static constexpr bool SMEM = !GPEND && (SB <= 16 || BIG32 || BIG64);  // pending local states in shared memory
    static constexpr int LAG = GPEND ? SAM_LAGG : (SB <= 4 ? SAM_LAG_SMALL : (SB <= 8 ? SAM_LAG8 : (SB <= 16 ? SAM_LAG16 : (BIG32 ? SAM_LAG32 : SAM_LAG64))));
    // max tiles per super-tile (carry unit); measured: 3 for 4-byte, 2 for 8-byte elements
    static constexpr int MMAX = (SB <= 8 && sizeof(T) == 4) ? 3 : (SB <= 8 ? 2 : SAM_MMAX_BIG);
    static constexpr int NB1 = 3;                    // local-scan (HBM) buffers
    static constexpr int NB2 = SB <= 8 ? 4 : 2;      // carry-application (L2 reload) buffers
    static constexpr int PF = NB1;                   // max claimed-but-unscanned tiles
    // orders 2..4 with smem-resident pending states: separate warp groups for local scans (P1) and
    // carry applications (P2) (measured faster there; order 1 keeps one group)
};

constexpr int MAX_CWARPS = 8;                      // compute warps
#ifndef SAM_NCARRY
#define SAM_NCARRY 4
#endif
constexpr int NCARRY = SAM_NCARRY;                 // carry warps (the fold of each super-tile's carry)
constexpr int NCARRY_P1 = NCARRY + 1;
constexpr int SERVICE_WARPS = 2 + NCARRY;          // producer + aggregator + carry warps
constexpr int MAX_THREADS = (MAX_CWARPS + SERVICE_WARPS) * 32;
// Warp roles of one instantiation.  NC carry warps: 2 for the 128-bit tuple-1 kernels of orders >= 2
// (their folds are small -- s*k <= 8 values -- and the two warps' registers go to the compute warps;
// measured +5..+19% for int32 k=4,8 and int64 k=2,4,5,8; int32 k=2 and int64 k=3 keep four:
// profiles/r2b_ab_ncarry.txt), else 4.  SPLIT: separate warp
// groups for local scans and carry applications -- states <= 16 B, and 8-byte states up to 24 B (32 B
// with two carry warps), the register cap of the larger CTA still holding them without spills.
// 4-byte states of 20..32 B (int32 orders 5-8) with two carry warps: split too (96 registers, no spills;
// sustained +1/+7/+20/+14% at orders 5/6/7/8, profiles/r2b_ab_split4b.txt)
#ifndef SAM_SPLIT_NV
#define SAM_SPLIT_NV 1
#endif
#ifndef SAM_SPLIT_4B
#define SAM_SPLIT_4B 1
#endif
// 8-byte order-1 tuple kernels: their fold is a plain sum of s values, two carry warps suffice
// (measured int64 k=1 s=2..7 +1..+8%, s=8 -5%, fp64 s=2/5/8 +2/+10/+2%; 4-byte tuples lose 3-7%:
// profiles/r2b_ab_nc2_tuples.txt, r2b_ab_nc2_t8k1.txt); the 128-bit tuple-1 kernels too (int64 +3%, fp64 +5%,
// profiles/r2b_ab_nc2_t8k1v.txt)
#ifndef SAM_NC_T8K1
#define SAM_NC_T8K1 1
#endif
#ifndef SAM_NC_T8K1V
#define SAM_NC_T8K1V 1
#endif
#ifndef SAM_NC_VEC2
#define SAM_NC_VEC2 1
#endif
template <typename T, int K, bool VEC> struct Threads {
    static constexpr int SB = K * (int)sizeof(T);
    static constexpr int NC =
        ((SAM_NC_VEC2 && VEC && K >= 2 && !(sizeof(T) == 4 && K == 2) && !(sizeof(T) == 8 && K == 3)) ||
         (SAM_NC_T8K1 && (!VEC || SAM_NC_T8K1V) && sizeof(T) == 8 && K == 1)) ? 2 : NCARRY;
    static constexpr bool SPLIT =
        (SB <= 16 || (SAM_SPLIT_BIG && (sizeof(T) == 8 || (SAM_SPLIT_4B && NC == 2)) && SB <= (NC == 2 ? 32 : SAM_SPLIT_MAXB))) &&
        K >= SAM_SPLIT_MIN_K && (VEC || SAM_SPLIT_NV);
    static constexpr int GROUPS = SPLIT ? 2 : 1;
    static constexpr int VALUE = (GROUPS * MAX_CWARPS + 2 + NC) * 32;
};
constexpr int TILE_THREADS = MAX_CWARPS * 32;

enum StoreMode { STORE_BULK = 0, STORE_STRIPED = 1, STORE_NONE = 2 };

// 64-bit tagged words per value: 1 for 32-bit types ([tag|value]), 2 for 64-bit ([tag|lo],[tag|hi])
template <typename T> struct TagW { static constexpr int W = sizeof(T) == 4 ? 1 : 2; };
// carry-fold window rows per round trip (carry-warp register budget: V*K*2W <= 16 words per lane)
template <typename T, int K> struct LB {
    static constexpr int W1 = TagW<T>::W;
    static constexpr int V0 = 16 / (K * W1);
    static constexpr int V = V0 < 1 ? 1 : (V0 > 16 ? 16 : V0);
};

// Coefficient / carry-fold type: fp32 scans fold their carries in double -- the binomial weights
// of spans of many super-tiles (C(L-1+d, d), L up to n) exceed the fp32 range at high orders, and
// double keeps the fold's rounding below the tile-local one.  Integers: the element type (mod 2^w).
template <typename T> struct Coef { using type = T; };
template <> struct Coef<float> { using type = double; };

template <typename T, int K>
struct Params {
    using CT = typename Coef<T>::type;
    const T* in;
    T* out;
    uint64_t n;          // elements in this stream
    uint64_t h;          // virtual index of in[0] (= lane phase, 0 <= h < s)
    uint64_t num_tiles;  // ceil((h + n) / T)
    uint64_t num_super;  // ceil(num_tiles / M)
    int M;               // tiles per super-tile (carry unit), 1..MMAX
    uint32_t delta;      // byte offset of virtual element 0 inside its 16-B chunk
    int s, G, logG, sp, c, logc, Pw, W, Wn;
    int U, T_, Uw;
    int inclusive;
    int store_mode;
    int claim_slack;      // experiments: extra claimed-but-blocked tiles (0 = never block a local scan)
    const T* seed;        // [s][K] state before the stream per global lane, or null
    T* final_state;       // [s][K] or null
    int64_t last_e[MAXS]; // virtual index of lane m's last element, -1 if none
    T* pend;              // GPEND: pending local states [grid][LAG][K][TILE_THREADS] (workspace)
    int lag;              // pipeline depth used (1..LAG): max tiles between a local scan and its carry application
    int land;             // carry folds read through the smem landing buffer (when it fits)
    int teams;            // carry teams: the 4 carry warps form `teams` teams working on successive super-tiles
    int vfold;            // integers + landing: value-parallel fold (else the windowed fold from the buffer)
    int dyn;              // dynamic claims: super-tiles taken from an atomic counter in claim order (else the
                          // static schedule b, b+P, ...); the fold spans (own previous, S) whatever its length
    unsigned long long* carry;  // tagged carry words: [tile][m][t][agg W | incl W]
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned int* epoch_ptr;
    unsigned long long carry_words;  // words of the carry ring actually used (R * rec_words)
    unsigned long long ring;         // R: super-tile slots of the O(1) carry ring (a power of two >= 32 grids)
    int ring_log2;
    unsigned int rec_words;          // words per super-tile record (16-B multiple)
    unsigned int* reset_ctr;         // grid barrier of the epoch wrap-around reset
    unsigned long long* trace;  // optional per-tile event timestamps [tile][8] (diagnostics), or null
    uint32_t stress;            // testing: nonzero = seed of pseudo-random delays at every pipeline hand-over
    T bc[K];              // b_d(ITEMS)
    T bw[K];              // b_d(Uw)
    T bu[K];              // b_d(U)        (one tile)
    CT bus[K];            // b_d(M*U)      (one super-tile)
    CT bwinj[NCARRY_P1][K]; // b_d(j*Wn*V*M*U), j <= NCARRY (carry-fold windows further)
    int coop;             // all carry warps fold each super-tile's windows together
    int Vr;               // window rows used per round trip (<= V)
    CT bprev[K];          // b_d((P-1)*M*U): from this CTA's previous super-tile to the one before S
    CT bwn[K];            // b_d(Wn*M*U)   (one window row further)
    T bt[K][32];          // b_d(v*ITEMS),  v < Pw        ([d][v])
    T bn[K][32];          // b_d(-(v+1)*ITEMS), v < Pw    ([d][v]; integer similarity transform)
    T bq[8][K];           // b_d(q*Uw),     q < c
    T bqn[8][K];          // b_d(-q*Uw),    q < c         (integer similarity transform)
    T bposP[K];           // b_d(P*M*U)     (global-frame carries: one round further)
    T bnegP[K];           // b_d(-P*M*U)
    CT bl[32][K];         // b_d(j*M*U),    j < Wn
    CT bsub[8][K];        // b_d(j*U),      j < M         (sub-tile offsets in a super-tile)
    T bks[5][K];          // b_d(2^l*ITEMS) (Kogge-Stone warp scan of thread states, K >= 3)
    T bkw[3][K];          // b_d(2^l*Uw)    (Kogge-Stone combine of warp states, K >= 3)
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
// non-blocking probe (mbarrier.test_wait never suspends the thread; for event loops)
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}" : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
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
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
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
        if (p.trace) p.trace[(size_t)(tile) * 16 + (ev)] = globaltimer();          \
    } while (0)
// testing (sam_debug_set_stress): a pseudo-random delay of up to ~16 us at 1 in 8 of the
// pipeline events, so the hand-overs between warps and CTAs happen in shuffled orders
static __device__ __noinline__ void stress_delay(uint32_t seed, uint64_t tile, uint32_t ev) {
    uint64_t h = tile * 0x9E3779B97F4A7C15ull ^ (uint64_t)(ev + 1) * 0xC2B2AE3D27D4EB4Full ^ seed;
    h ^= h >> 29;
    h *= 0xBF58476D1CE4E5B9ull;
    h ^= h >> 32;
    const uint32_t r = (uint32_t)h;
    if ((r & 7) == 0) __nanosleep((r >> 8) & 16383);
}
#define SAM_STRESS(ev, tile)                                                       \
    do {                                                                           \
        if (p.stress) stress_delay(p.stress, (uint64_t)(tile), (ev));              \
    } while (0)
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// CTA-scope flags in shared memory (end-of-stream, progress counters, hand-off stamps): atomic
// accesses (racecheck treats them as synchronisation; they sit only on wait paths), the data they
// guard ordered by CTA fences (writer: fence, then the flag; reader: the flag, then a fence)
__device__ __forceinline__ int flag_ld(const volatile int* p) { return atomicOr((int*)p, 0); }
__device__ __forceinline__ int flag_ld_acq(const volatile int* p) {
    const int v = atomicOr((int*)p, 0);
    __threadfence_block();
    return v;
}
__device__ __forceinline__ void flag_st(volatile int* p, int v) { atomicExch((int*)p, v); }
__device__ __forceinline__ void flag_st_rel(volatile int* p, int v) {
    __threadfence_block();
    atomicExch((int*)p, v);
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
    unsigned long long a;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(a) : "l"(p) : "memory");
    return a;
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
__device__ __forceinline__ void put_tagged(unsigned long long* slot, uint32_t tag, T v) {
    constexpr int W = TagW<T>::W;
    const uint64_t b = Bits<T>::to(v);
    const uint64_t hi = (uint64_t)tag << 32;
    if constexpr (W == 1) {
        st_relaxed_u64(slot, hi | (b & 0xffffffffull));
    } else {
        st_relaxed_u64(slot, hi | (b & 0xffffffffull));
        st_relaxed_u64(slot + 1, hi | (b >> 32));
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

// b_d(L) = C(L-1+d, d), d < K (first column of M(L)), lane d computing one binomial, broadcast to
// the warp (all 32 lanes must call it)
template <typename T, int K>
__device__ __forceinline__ void mcol_warp(int64_t L, T (&b)[K]) {
    const int lane = threadIdx.x & 31;
    const int d = lane < K ? lane : 0;
    const T mine = Arith<T>::binom(L - 1 + d, d);
#pragma unroll
    for (int t = 0; t < K; ++t) b[t] = __shfl_sync(0xffffffffu, mine, t);
}

// ------------------------------------------------------------------------------------------
// shared-memory layout
// ------------------------------------------------------------------------------------------
template <typename T, int K, bool VEC, int NB1_, int NB2_>
struct SmemL {
    using CT = typename Coef<T>::type;
    static constexpr int ITEMS = Items<T, VEC>::V;
    static constexpr int NB1 = NB1_;
    static constexpr int NB2 = NB2_;
    static constexpr int LAG = Lag<T, K>::LAG;
    static constexpr int NQ = (LAG + 1 > NB1 ? LAG + 1 : NB1) + 1;  // per-iteration state ring
    static constexpr int ELAG = Lag<T, K>::SMEM ? LAG : 0;          // smem-resident pending states
    static constexpr int TMAX = TILE_THREADS * ITEMS;
    static constexpr int NBL = 32;                // carry-fold binomial rows
    static constexpr int BUFB = ((TMAX * (int)sizeof(T) + 32) + 127) / 128 * 128;
    static constexpr int WQ = (VEC ? 8 : 64) * K; // per-iteration warp states [pairs][K] (VEC: s = 1, 8 warps)
    static constexpr int LA = 8 * K;              // per-iteration tile aggregate [8][K]
    static constexpr int OFF_BUF1 = 0;
    static constexpr int OFF_BUF2 = OFF_BUF1 + NB1 * BUFB;
    static constexpr int OFF_BAR = OFF_BUF2 + NB2 * BUFB;  // full1[NB1] full2[NB2] stored2[NB2] p1/agg/carry[NQ]
    static constexpr int NBAR = NB1 + 2 * NB2 + 3 * NQ + 2 * NCARRY;  // ... bar_cw[NCARRY], bar_land[NCARRY]
    static constexpr int OFF_TILE = OFF_BAR + NBAR * 8;                  // NQ x i64 tile id
    static constexpr int OFF_SUP = OFF_TILE + NQ * 8;                    // NQ x i64 super-tile id
    static constexpr int OFF_SUB = OFF_SUP + NQ * 8;                     // NQ x (i32 sub index, i32 count)
    static constexpr int OFF_TAG = OFF_SUB + NQ * 8;                     // u32 tag, i32 end, i32 agg progress, i32 p2, i32 claims
    static constexpr int OFF_CW = OFF_TAG + 32;                          // NCARRY x i32 super-tile taken
    static constexpr int OFF_WQ = (OFF_CW + 4 * NCARRY + 15) / 16 * 16;  // NQ x [64][K]
    static constexpr int OFF_LA = OFF_WQ + NQ * WQ * (int)sizeof(T);     // NQ x [8][K]
    static constexpr int OFF_LP = OFF_LA + NQ * LA * (int)sizeof(T);     // NQ x [8][K] in-super prefix
    static constexpr int OFF_BT = OFF_LP + NQ * LA * (int)sizeof(T);     // [K][32]
    static constexpr int OFF_BN = OFF_BT + K * 32 * (int)sizeof(T);      // [K][32]
    static constexpr int OFF_BL = OFF_BN + K * 32 * (int)sizeof(T);      // [NBL][K]
    static constexpr int OFF_BQ = OFF_BL + NBL * K * (int)sizeof(CT);    // [8][K]
    static constexpr int HOB = 16 + MAXS * K * (int)sizeof(CT);          // hand-off entry: i32 r, pad, [MAXS][K]
    static constexpr int OFF_HO = OFF_BQ + 8 * K * (int)sizeof(T);       // [NCARRY] inclusive-state hand-off
    static constexpr int OFF_PART = (OFF_HO + NCARRY * HOB + 15) / 16 * 16;   // [2][NCARRY][MAXS][K]
    static constexpr int OFF_PV = OFF_PART + 2 * NCARRY * MAXS * K * (int)sizeof(CT);  // [NCARRY][64] value-parallel fold partials
    static constexpr int OFF_GN = OFF_PV + NCARRY * 64 * (int)sizeof(CT);                // [2][K] next b(S US) (global frame)
    static constexpr int OFF_EQ = OFF_GN + 2 * K * (int)sizeof(CT);                     // [ELAG][TILE_THREADS][K]
    static constexpr int BYTES0 = OFF_EQ + ELAG * TILE_THREADS * K * (int)sizeof(T);
    // carry-fold landing buffer: the P-1 aggregates a fold reads, pulled from L2 in ONE bulk copy
    // (whatever shared memory is left, up to 40 KB; the fold falls back to windowed loads if short)
    static constexpr int OFF_LAND = (BYTES0 + 127) / 128 * 128;
    static constexpr int LAND_ROOM = 227 * 1024 - OFF_LAND;
    static constexpr int LANDB = LAND_ROOM < 0 ? 0 : (LAND_ROOM > 40960 ? 40960 : LAND_ROOM / 128 * 128);
    static constexpr int BYTES = OFF_LAND + LANDB;
};
// one carry-application buffer fewer when the larger VEC tiles would not fit, then one local-scan
// buffer fewer (large smem-resident pending states)
template <typename T, int K, bool VEC>
struct SmemPick {
    static constexpr int B1 = Lag<T, K>::NB1, B2 = Lag<T, K>::NB2;
    static constexpr int B2m = B2 - 1 < 2 ? 2 : B2 - 1;
    using C1 = SmemL<T, K, VEC, B1, B2>;
    using C2 = SmemL<T, K, VEC, B1, B2m>;
    using C3 = SmemL<T, K, VEC, B1 - 1, B2m>;
    static constexpr int LIM = 227 * 1024;
    using type = std::conditional_t<(C1::BYTES0 <= LIM), C1, std::conditional_t<(C2::BYTES0 <= LIM), C2, C3>>;
};
template <typename T, int K, bool VEC>
struct Smem : SmemPick<T, K, VEC>::type {};

// ------------------------------------------------------------------------------------------
// the kernel
// ------------------------------------------------------------------------------------------
template <typename T, int K, bool VEC>
__global__ void __launch_bounds__(Threads<T, K, VEC>::VALUE, 1)
sam_scan_kernel(const __grid_constant__ Params<T, K> p) {
    using S = Smem<T, K, VEC>;
    using CT = typename Coef<T>::type;
    constexpr int ITEMS = S::ITEMS;
    constexpr int NB1 = S::NB1;
    constexpr int NB2 = S::NB2;
    constexpr int NQ = S::NQ;
    constexpr int LAG = S::LAG;
    constexpr bool ESMEM = Lag<T, K>::SMEM;
    constexpr bool EGMEM = Lag<T, K>::GPEND;
    const int lag = p.lag;
    constexpr int PF = S::NB1;  // max claimed-but-unscanned tiles
    constexpr int W1 = TagW<T>::W;      // tagged words per published value
    constexpr int V = LB<T, K>::V;
    // integer similarity-transform scans / global-frame carries (int32: from order SAM_TR32_MIN_K)
    constexpr bool TRANSFORM = IsInt<T>::value && K >= 2 && SAM_TRANSFORM && (sizeof(T) == 8 || K >= SAM_TR32_MIN_K);
    static_assert(ITEMS >= K, "exclusive shift needs ITEMS >= K");
    static_assert(VEC || ITEMS % 2 == 1, "ITEMS odd keeps the stride-s smem reads bank-conflict free");
    static_assert(PF <= NB1 && NQ > LAG && NQ > NB1 && NB2 <= 4, "ring sizes");
    static_assert(S::BYTES <= 227 * 1024, "shared memory budget");

    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* bar_full1 = (uint64_t*)(smem + S::OFF_BAR);
    uint64_t* bar_full2 = bar_full1 + NB1;
    uint64_t* bar_stored2 = bar_full2 + NB2;
    uint64_t* bar_p1 = bar_stored2 + NB2;
    uint64_t* bar_agg = bar_p1 + NQ;
    uint64_t* bar_carry = bar_agg + NQ;
    uint64_t* bar_cw = bar_carry + NQ;  // [NCARRY]: a super-tile is ready for carry warp w
    uint64_t* bar_land = bar_cw + NCARRY;  // [team] the team's landing buffer is full
    volatile int* cw_taken = (volatile int*)(smem + S::OFF_CW);  // last super-tile each carry warp took
    int64_t* tile_of = (int64_t*)(smem + S::OFF_TILE);
    int64_t* sup_of = (int64_t*)(smem + S::OFF_SUP);
    int* sub_of = (int*)(smem + S::OFF_SUB);  // [q][0] sub index, [q][1] sub-tiles in the super-tile
    T* lp_all = (T*)(smem + S::OFF_LP);
    uint32_t* sm_tag = (uint32_t*)(smem + S::OFF_TAG);
    volatile int* sm_end = (volatile int*)(smem + S::OFF_TAG + 4);
    volatile int* agg_done = (volatile int*)(smem + S::OFF_TAG + 8);  // iterations aggregated
    volatile int* lb_started = (volatile int*)(smem + S::OFF_TAG + 20);  // last super-tile whose fold began
    volatile int* claimed = (volatile int*)(smem + S::OFF_TAG + 24);     // iterations claimed (dynamic claims)
    T* wq_all = (T*)(smem + S::OFF_WQ);
    T* la_all = (T*)(smem + S::OFF_LA);
    T* bt_s = (T*)(smem + S::OFF_BT);
    T* bn_s = (T*)(smem + S::OFF_BN);
    CT* bl_s = (CT*)(smem + S::OFF_BL);
    T* bq_s = (T*)(smem + S::OFF_BQ);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int s = p.s, c = p.c;
    constexpr bool SPLIT = Threads<T, K, VEC>::SPLIT;
    constexpr int NC = Threads<T, K, VEC>::NC;  // carry warps (ring depths stay NCARRY)
    const int NW = p.W;          // compute warps per group
    const int NCT = NW * 32;     // compute threads per group
    const int NCW = SPLIT ? 2 * NW : NW;  // compute warps (both groups); service warps follow
    const int Tt = p.T_;

    // ---- prologue: barriers, tables, epoch tag -------------------------------------------------
    if (tid == 0) {
        for (int b = 0; b < NB1; ++b) mbar_init(&bar_full1[b], 1);
        for (int b = 0; b < NB2; ++b) {
            mbar_init(&bar_full2[b], 1);
            mbar_init(&bar_stored2[b], NCT);
        }
        for (int q = 0; q < NQ; ++q) {
            mbar_init(&bar_p1[q], NCT);
            mbar_init(&bar_agg[q], 32);
            mbar_init(&bar_carry[q], 32);
        }
        for (int w = 0; w < NCARRY; ++w) {
            mbar_init(&bar_cw[w], 32);
            mbar_init(&bar_land[w], 1);
            cw_taken[w] = -1;
            *(volatile int*)(smem + S::OFF_HO + w * S::HOB) = -1;
        }
        fence_mbar_init();
        // tag of a word = [20-bit launch epoch | 12-bit ring lap of its super-tile]; the epoch part
        // cycles 1..2^20-1 (never 0: zero-filled memory never validates); when it restarts at 1 this
        // launch first zeroes the ring (below) so no word of a launch 2^20-1 launches ago validates
        const unsigned ep = *(volatile unsigned int*)p.epoch_ptr;
        const unsigned ep20 = ep % 1048575u + 1u;
        *sm_tag = ep20 == 1u ? 0u : (ep20 << 12);
        *sm_end = -1;
        *agg_done = 0;
        *(volatile int*)(smem + S::OFF_TAG + 12) = 0;
        *lb_started = -1;
        *claimed = 0;
    }
    for (int i = tid; i < K * 32; i += blockDim.x) bt_s[i] = (&p.bt[0][0])[i];
    for (int i = tid; i < K * 32; i += blockDim.x) bn_s[i] = (&p.bn[0][0])[i];
    for (int i = tid; i < S::NBL * K; i += blockDim.x) bl_s[i] = (&p.bl[0][0])[i];
    for (int i = tid; i < 8 * K; i += blockDim.x) bq_s[i] = (&p.bq[0][0])[i];
    __syncthreads();
    if (*sm_tag == 0u) {  // epoch wrap-around (once per 2^20-1 launches of a workspace; the ring is small)
        for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + tid; i < p.carry_words;
             i += (unsigned long long)gridDim.x * blockDim.x)
            p.carry[i] = 0ull;
        __syncthreads();
        if (tid == 0) {  // grid barrier (all CTAs co-resident: cooperative launch)
            __threadfence();
            atomicAdd(p.reset_ctr, 1u);
            while (*(volatile unsigned int*)p.reset_ctr < gridDim.x) __nanosleep(100);
            __threadfence();
            *sm_tag = 1u << 12;
        }
        __syncthreads();
    }
    const uint32_t tag = *sm_tag;  // base tag: | ring lap of the super-tile
    // O(1) carry ring: super-tile S lives in slot S mod R, tagged with its lap S / R, so a
    // word of the previous lap (or launch) never validates
    auto ctag = [&](int64_t S) -> uint32_t { return tag | (uint32_t)(((uint64_t)S >> p.ring_log2) & 0xfffu); };
    auto cslot = [&](int64_t S) -> unsigned long long* {
        return p.carry + ((uint64_t)S & (p.ring - 1)) * p.rec_words;
    };

    // wait for barrier phase `par`, or return false once the stream has ended before iteration it
    auto wait_or_end = [&](uint64_t* bar, uint32_t par, int it) -> bool {
        bool ended = false;
        while (!mbar_try_wait(bar, par)) {
            const int end = flag_ld(sm_end);
            if (end >= 0 && it >= end) { ended = true; break; }
        }
        return !__any_sync(0xffffffffu, ended);
    };

    if (warp == NCW) {
        // =========================== producer warp: claims, loads, reloads, stores =============
        if (lane == 0) {
            const uint64_t pol_keep = policy_evict_last();
            const uint64_t pol_stream = policy_evict_first();
            auto tile_range = [&](int64_t tile, uint64_t& lo, uint64_t& hi) {
                const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
                lo = e0 > p.h ? e0 : p.h;
                hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
            };
            auto load_tile = [&](int64_t tile, unsigned char* buf, uint64_t* bar, uint64_t pol) {
                uint64_t lo, hi;
                tile_range(tile, lo, hi);
                const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
                const uintptr_t src_lo = (uintptr_t)p.in + (lo - p.h) * sizeof(T);
                const uintptr_t src_hi = (uintptr_t)p.in + (hi - p.h) * sizeof(T);
                const uintptr_t a16 = src_lo & ~(uintptr_t)15;
                const uintptr_t b16 = (src_hi + 15) & ~(uintptr_t)15;
                unsigned char* dst = buf + p.delta + (lo - e0) * sizeof(T) - (src_lo - a16);
                mbar_arrive_expect_tx(bar, (uint32_t)(b16 - a16));
                bulk_g2s(dst, (const void*)a16, (uint32_t)(b16 - a16), bar, pol);
            };
            auto store_tile = [&](int64_t tile, const unsigned char* buf) {
                if (p.store_mode != STORE_BULK) return;
                uint64_t lo, hi;
                tile_range(tile, lo, hi);
                const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
                const uintptr_t ob = (uintptr_t)p.out + (lo - p.h) * sizeof(T);
                const uintptr_t oe = (uintptr_t)p.out + (hi - p.h) * sizeof(T);
                const uintptr_t bs = (ob + 15) & ~(uintptr_t)15;
                const uintptr_t be = oe & ~(uintptr_t)15;
                if (be > bs) {
                    const unsigned char* src = buf + p.delta + (lo - e0) * sizeof(T) + (bs - ob);
                    bulk_s2g((void*)bs, src, (uint32_t)(be - bs), pol_stream);
                }
                bulk_commit();  // one group per stored iteration (possibly empty)
            };
            int j1 = 0, j2 = 0, j3 = 0, jend = -1;
            int64_t cur_sup = -1;
            int cur_j = 0, cur_cnt = 0, nsup = 0;
            for (;;) {
                // (1) store the oldest iteration whose carry application is done
                if (j3 < j2 && mbar_test(&bar_stored2[j3 % NB2], (uint32_t)((j3 / NB2) & 1))) {
                    if (p.trace) SAM_TRACE(7, tile_of[j3 % NQ]);
                    store_tile(tile_of[j3 % NQ], smem + S::OFF_BUF2 + (j3 % NB2) * S::BUFB);
                    ++j3;
                    continue;
                }
                // (2) reload (from L2) the next tile whose carry is known, into a free carry buffer
                if (j2 < j1 && j2 - j3 < NB2 &&
                    (SAM_EARLY_RELOAD == 2 ? (j2 / p.M <= flag_ld(lb_started))
                                           : mbar_test(SAM_EARLY_RELOAD ? &bar_p1[j2 % NQ] : &bar_carry[j2 % NQ],
                                                       (uint32_t)((j2 / NQ) & 1)))) {
                    // groups committed after the store that last used this buffer (iteration j2-NB2)
                    const int later = j3 - 1 - (j2 - NB2);
                    if (later <= 0) bulk_wait_read<0>();
                    else if (later == 1) bulk_wait_read<1>();
                    else if (later == 2) bulk_wait_read<2>();
                    else bulk_wait_read<3>();
                    // state-only pass (sam_shard_state): a tile holding no lane's last element needs
                    // no carry application, so it is not re-fetched -- the barrier is just released
                    bool need = true;
                    if (p.store_mode == STORE_NONE) {
                        const int64_t t0 = tile_of[j2 % NQ] * (int64_t)Tt;
                        need = false;
                        for (int mm = 0; mm < s; ++mm)
                            need |= (p.last_e[mm] >= t0 && p.last_e[mm] < t0 + Tt);
                    }
                    if (need) {
                        load_tile(tile_of[j2 % NQ], smem + S::OFF_BUF2 + (j2 % NB2) * S::BUFB, &bar_full2[j2 % NB2],
                                  pol_stream);
                    } else {
                        mbar_arrive(&bar_full2[j2 % NB2]);
                    }
                    ++j2;
                    continue;
                }
                // (3) load the next tile of this CTA's static schedule (super-tiles b, b+P, ...) once
                // a buffer is free, at most PF tiles are unscanned and a pending-state slot is free
                // (tile j1's local scan needs the carry application of j1 - LAG done, and a loaded
                // tile must never wait for that -- its aggregate gates the other CTAs' carries)
                if (jend < 0 && j1 < j3 + lag + p.claim_slack &&
                    (j1 < NB1 || mbar_test(&bar_p1[(j1 - NB1) % NQ], (uint32_t)(((j1 - NB1) / NQ) & 1))) &&
                    (j1 < PF || mbar_test(&bar_p1[(j1 - PF) % NQ], (uint32_t)(((j1 - PF) / NQ) & 1)))) {
                    if (cur_j == cur_cnt) {  // start the next super-tile
                        // static schedule: b, b+P, ...; dynamic: the next one in claim order
                        cur_sup = p.dyn ? (int64_t)atomicAdd(p.tile_ctr, 1ull)
                                        : (int64_t)blockIdx.x + (int64_t)nsup * gridDim.x;
                        ++nsup;
                        cur_j = 0;
                        cur_cnt = 0;
                        if ((uint64_t)cur_sup < p.num_super) {
                            const uint64_t rest = p.num_tiles - (uint64_t)cur_sup * p.M;
                            cur_cnt = rest < (uint64_t)p.M ? (int)rest : p.M;
                        }
                    }
                    if (cur_cnt == 0) {
                        jend = j1;
                        flag_st(sm_end, j1);
                    } else {
                        const int64_t t = cur_sup * p.M + cur_j;
                        const int qs = j1 % NQ;
                        tile_of[qs] = t;
                        sup_of[qs] = cur_sup;
                        sub_of[2 * qs] = cur_j;
                        sub_of[2 * qs + 1] = cur_cnt;
                        ++cur_j;
                        SAM_TRACE(0, t);
                        SAM_STRESS(0, t);
                        load_tile(t, smem + S::OFF_BUF1 + (j1 % NB1) * S::BUFB, &bar_full1[j1 % NB1], pol_keep);
                        ++j1;
                        if (p.dyn) flag_st_rel(claimed, j1);  // tile_of / sup_of / sub_of of iteration j1-1 are set
                    }
                    continue;
                }
                if (jend >= 0 && j3 == jend) break;
                __nanosleep(SAM_PROD_NS);
            }
            bulk_wait_all0();
        }
    } else if (warp == NCW + 1) {
        // =========================== aggregator warp: block combine, aggregate publish ===========
        // Per tile: combine the warp states (E = warp-exclusive prefixes, tile aggregate A_j); per
        // super-tile: the running prefix P_j = A_0 (+) ... (+) A_{j-1} (kept in registers by the
        // lane that owns lane m's aggregate), and after the last sub-tile the super-tile aggregate,
        // published for the other CTAs' carry folds (a4).
        const int npair = s * c;
        T Pref[2][K];
        T gneg[K];  // global frame (integers): b(-(S+1) US) of this CTA's current super-tile
        if constexpr (TRANSFORM) mcol<T>(-((int64_t)blockIdx.x + 1) * p.M * p.U, K, gneg);
        for (int i = 0;; ++i) {
            const int qs = i % NQ;
            if (!wait_or_end(&bar_p1[qs], (uint32_t)((i / NQ) & 1), i)) break;
            const int64_t tile = tile_of[qs];
            const int64_t sup = sup_of[qs];
            const int jsub = sub_of[2 * qs], cnt = sub_of[2 * qs + 1];
            if constexpr (TRANSFORM) {  // dynamic claims: b(-(S+1) US) of this super-tile, from its id
                if (p.dyn && jsub == 0) mcol_warp<T, K>(-(sup + 1) * (int64_t)p.M * p.U, gneg);
            }
            if (lane == 0) SAM_TRACE(2, tile);
            SAM_STRESS(1, tile);
            T* wq = wq_all + qs * S::WQ;
            T* la = la_all + qs * S::LA;
            T* lp = lp_all + qs * S::LA;
#pragma unroll
            for (int ch = 0; ch < 2; ++ch) {
                if (32 * ch >= npair) break;  // warp-uniform: second pass only for s = 8
                const int pair = lane + 32 * ch;
                const bool ok = pair < npair;
                const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
                T E[K], yl[K];
                if constexpr (TRANSFORM) {
                    // Integers: the compute warps left each warp's total Z_q in its transformed frame
                    // (warp aggregate A_q = M(Uw) Z_q).  With z'_q = M(-q Uw) Z_q,
                    //   E_q = sum_{p<q} M((q-1-p) Uw) A_p = M(q Uw) sum_{p<q} z'_p,
                    // so the combine is K plain scans over the c warps; E'_q = sum_{p<q} z'_p is
                    // stored (the carry team applies M(q Uw) with its own), and the tile aggregate
                    // is M(U) (sum of all z'), folded into the running prefix as M(U)(Pref + sum).
                    T zq[K];
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T acc2 = ok ? wq[(qq * s + mm) * K + t] : T(0);
                        yl[t] = acc2;
                    }
#pragma unroll
                    for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                        for (int j = 0; j < t; ++j) yl[t] += p.bqn[qq][t - j] * yl[j];
                    }
#pragma unroll
                    for (int t = 0; t < K; ++t) zq[t] = yl[t];
#pragma unroll
                    for (int l = 0; l < 3; ++l) {  // offsets 1, 2, 4 < c
                        const int off = 1 << l;
                        if (off < c) {
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                T o = shfl_up(yl[t], off);
                                if (qq >= off) yl[t] += o;
                            }
                        }
                    }
#pragma unroll
                    for (int t = 0; t < K; ++t) E[t] = yl[t] - zq[t];  // E'_q; yl = inclusive sum
                } else                 if constexpr (K < SAM_KS_MIN_K) {
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T z = ok ? wq[(qq * s + mm) * K + t] : T(0);
#pragma unroll
                        for (int j = 0; j < t; ++j) z += p.bw[t - j] * E[j];
                        T y = z;
#pragma unroll
                        for (int l = 0; l < 3; ++l) {  // offsets 1, 2, 4 < c (unrolled)
                            const int off = 1 << l;
                            if (off < c) {
                                T o = shfl_up(y, off);
                                if (qq >= off) y += o;
                            }
                        }
                        if constexpr (IsInt<T>::value) {
                            E[t] = y - z;
                        } else {
                            T o = shfl_up(y, 1);
                            E[t] = (qq >= 1) ? o : T(0);
                        }
                        yl[t] = y;
                    }
                } else {  // Kogge-Stone on k-vectors: yl <- M(2^l Uw) yl_partner + yl
#pragma unroll
                    for (int t = 0; t < K; ++t) yl[t] = ok ? wq[(qq * s + mm) * K + t] : T(0);
#pragma unroll
                    for (int l = 0; l < 3; ++l) {
                        const int off = 1 << l;
                        if (off < c) {
                            T o[K];
#pragma unroll
                            for (int t = 0; t < K; ++t) o[t] = shfl_up(yl[t], off);
                            if (qq >= off) {
#pragma unroll
                                for (int t = K - 1; t >= 0; --t) {
                                    T acc2 = yl[t] + o[t];
#pragma unroll
                                    for (int j = 0; j < t; ++j) acc2 += p.bkw[l][t - j] * o[j];
                                    yl[t] = acc2;
                                }
                            }
                        }
                    }
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T o = shfl_up(yl[t], 1);
                        E[t] = (qq >= 1) ? o : T(0);
                    }
                }
                __syncwarp();
                if (ok) {
#pragma unroll
                    for (int t = 0; t < K; ++t) wq[(qq * s + mm) * K + t] = E[t];  // warp-exclusive prefix
                    if (qq == c - 1) {  // this lane owns lane mm's tile aggregate yl
                        if (jsub == 0) {
#pragma unroll
                            for (int t = 0; t < K; ++t) Pref[ch][t] = T(0);
                        }
#pragma unroll
                        for (int t = 0; t < K; ++t) lp[mm * K + t] = Pref[ch][t];  // state before sub-tile
                        if constexpr (TRANSFORM) {  // Pref <- M(U) (Pref + sum z')
#pragma unroll
                            for (int t = 0; t < K; ++t) Pref[ch][t] += yl[t];
#pragma unroll
                            for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                                for (int j = 0; j < t; ++j) Pref[ch][t] += p.bu[t - j] * Pref[ch][j];
                            }
                        } else {
#pragma unroll
                        for (int t = K - 1; t >= 0; --t) {  // Pref <- M(U) Pref + A_j
                            T acc2 = Pref[ch][t] + yl[t];
#pragma unroll
                            for (int j = 0; j < t; ++j) acc2 += p.bu[t - j] * Pref[ch][j];
                            Pref[ch][t] = acc2;
                        }
                        }
                        if (jsub == cnt - 1) {
                            T av[K];
#pragma unroll
                            for (int t = 0; t < K; ++t) av[t] = Pref[ch][t];
                            if constexpr (TRANSFORM) {  // global frame: A~_S = M(-(S+1) US) A_S
#pragma unroll
                                for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                                    for (int j = 0; j < t; ++j) av[t] += gneg[t - j] * av[j];
                                }
                            }
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                la[mm * K + t] = av[t];  // super-tile aggregate (transformed for integers)
                                {  // a4: publish it
                                    put_tagged<T>(cslot(sup) + (mm * K + t) * W1, ctag(sup), av[t]);
                                }
                            }
                        }
                    }
                }
            }
            __syncwarp();
            if (lane == 0) SAM_TRACE(3, tile);
            mbar_arrive(&bar_agg[qs]);
            if (TRANSFORM && !p.dyn && jsub == cnt - 1) {  // next super-tile of this CTA: one round further
                T ng[K];
#pragma unroll
                for (int d = 0; d < K; ++d) {
                    T acc2 = T(0);
#pragma unroll
                    for (int e2 = 0; e2 <= d; ++e2) acc2 += gneg[e2] * p.bnegP[d - e2];
                    ng[d] = acc2;
                }
#pragma unroll
                for (int d = 0; d < K; ++d) gneg[d] = ng[d];
            }
            if (jsub == cnt - 1) {  // super-tile complete: wake its carry warp (super-tiles round-robin)
                const int r = i / p.M;
                // at most one unconsumed phase per barrier: the warp must have taken super-tile r-NCARRY
                while (flag_ld(&cw_taken[r % NCARRY]) < r - NCARRY) __nanosleep(32);
                mbar_arrive(&bar_cw[r % NCARRY]);
            }
            __syncwarp();
            if (lane == 0) flag_st(agg_done, i + 1);
        }
    } else if (warp >= NCW + 2) {
        // =========================== carry warps: carry-in of each super-tile ===================
        // a5, SAM's carry scheme on a static schedule: CTA b owns super-tiles
        // b, b+P, b+2P, ... (P = gridDim.x, all CTAs co-resident: cooperative launch).  The carry
        // into super-tile S is this CTA's own inclusive state after S-P (kept in shared memory)
        // advanced over the P-1 aggregates published by the other CTAs in between:
        //   C_S = M((P-1) US) I_{S-P} + sum_{j=S-P+1}^{S-1} M((S-1-j) US) A_j
        // read in windows of Wn*V super-tiles, one L2 round trip each (no inclusive chain
        // between CTAs, hence no serial latency).
        const int npair = s * c;
        const int cw = warp - (NCW + 2);
        // p.coop: the fold needs several windows (large states, tuples): all carry warps work on
        // every super-tile, warp w folding windows w, w+NCARRY, ... (round trips in parallel);
        // otherwise the carry warps take super-tiles round-robin, one warp folding all windows
        const bool coop = p.coop != 0;
        // Teams: the carry warps form NT teams of TW warps; team t takes this CTA's super-tiles t, t+NT,
        // ... (folds of successive super-tiles overlap; only the short chain step is ordered, through
        // the hand-off entries).  coop = 0 is NT = 4 teams of one warp.
        const int NT = coop ? (p.teams == 2 && NC >= 2 ? 2 : 1) : NC;  // 1, 2 or NC teams
        const int lgNT = NT == 1 ? 0 : (NT == 2 ? 1 : 2);
        const int TW = NC >> lgNT;
        const int team = cw / TW, tw = cw - team * TW;
        const bool lead = tw == 0;  // finishes the super-tile (hand-off, sub-tile states)
        const int WV = p.Wn * p.Vr;          // super-tiles per window
        CT* const part_s = (CT*)(smem + S::OFF_PART);  // [2][NCARRY][MAXS][K] coop partial folds
        // landing: the whole range of aggregates a fold reads (at most P-1 super-tiles of s*K values)
        // arrives in shared memory with one bulk copy; words whose tag is not yet this launch's are
        // re-polled from L2 (the nearest predecessors, published last)
        constexpr uint64_t SUPB = (uint64_t)K * W1 * 8;  // bytes per (super-tile, lane)
        const int land_part = (S::LANDB / NT) / 128 * 128;  // each team's landing buffer
        // (static schedule: every fold spans P-1 super-tiles; dynamic claims: checked per fold)
        const bool use_land = SAM_LAND && p.land && coop && land_part > 0 &&
                              (p.dyn || (uint64_t)(gridDim.x - 1) * p.rec_words * 8 <= (uint64_t)land_part);
        unsigned char* const land_s = smem + S::OFF_LAND + team * land_part;
        uint64_t* const bar_lt = &bar_land[team];
        int nland = 0;  // landing copies consumed so far (mbarrier parity)
        CT gpos[K];     // global frame: b(S US) of the current super-tile (lead, coop: advanced per round)
        CT tsum[K];     // global frame: I~_prev + sum of the folded A~_j (the next hand-off adds A~_S)
#pragma unroll
        for (int t = 0; t < K; ++t) { gpos[t] = CT(0); tsum[t] = CT(0); }
        int64_t sprev_dyn = -1;  // dynamic claims: this CTA's previous super-tile
        for (int r = team;; r += NT) {  // this CTA's r-th super-tile
            const int i0 = r * p.M;       // its first iteration
            int64_t tile, Sprev;          // global super-tile id; this CTA's previous one (-1: none)
            if (p.dyn) {
                // the producer claims super-tiles in order: wait until it has taken this CTA's r-th
                // (its id is then in sup_of), or the stream has ended before it
                int st2 = 0;
                if (lane == 0) {
                    for (;;) {
                        if (flag_ld_acq(claimed) > i0) { st2 = 1; break; }
                        const int e = flag_ld(sm_end);
                        if (e >= 0 && i0 >= e) break;
                        __nanosleep(32);
                    }
                }
                if (!__shfl_sync(0xffffffffu, st2, 0)) break;
                tile = sup_of[i0 % NQ];
                Sprev = sprev_dyn;
                sprev_dyn = tile;
                if constexpr (TRANSFORM) {
                    // b(S US) for the lead's chain step, by the team's second warp while the fold runs
                    if (coop && TW > 1 && tw == 1) {
                        CT gp[K];
                        mcol_warp<CT, K>(tile * (int64_t)p.M * p.U, gp);
                        CT* gn = (CT*)(smem + S::OFF_GN) + (r & 1) * K;
                        if (lane < K) gn[lane] = gp[lane];
                    }
                }
            } else {
                tile = (int64_t)blockIdx.x + (int64_t)r * gridDim.x;
                if ((uint64_t)tile >= p.num_super) break;
                Sprev = r == 0 ? (int64_t)-1 : tile - gridDim.x;
            }
            const bool lane_ok = lane < s;
            const int ml = lane_ok ? lane : 0;
            const int bw = (int)(r % NCARRY);  // the aggregator's barrier for super-tile r
            // landing range [lo_sup, tile) in bytes, 16-B aligned.  The copy is issued before the wait
            // for this super-tile's own aggregate: the previous round's aggregates are long published,
            // the current round's (the nearest) are re-polled from L2 if not yet there.
            const int64_t lo_sup = Sprev + 1;
            const bool land_r = use_land && tile > lo_sup &&
                                (uint64_t)(tile - lo_sup) * p.rec_words * 8 <= (uint64_t)land_part;
            // landing offset of super-tile j: (j - lo_sup) * REC; the ring range may wrap: two copies
            if (land_r && lead && lane == 0) {
                const uint64_t REC = (uint64_t)p.rec_words * 8;
                const uint64_t cnt = (uint64_t)(tile - lo_sup);
                const uint64_t slot0 = (uint64_t)lo_sup & (p.ring - 1);
                const uint64_t c1 = slot0 + cnt <= p.ring ? cnt : p.ring - slot0;
                fence_proxy_async_smem();  // the previous fold's generic reads of the buffer come first
                mbar_arrive_expect_tx(bar_lt, (uint32_t)(cnt * REC));
                bulk_g2s(land_s, (const void*)(p.carry + slot0 * p.rec_words), (uint32_t)(c1 * REC), bar_lt,
                         policy_evict_last());
                if (c1 < cnt)
                    bulk_g2s(land_s + c1 * REC, (const void*)p.carry, (uint32_t)((cnt - c1) * REC), bar_lt,
                             policy_evict_last());
            }
            if (lead) {
                // Wait for the aggregator: it arrives on bar_cw[r % NCARRY] when super-tile r is
                // fully aggregated, and only after super-tile r - NCARRY was taken (cw_taken), so the
                // barrier is never more than one phase ahead and the parity below is unambiguous.
                mbar_wait(&bar_cw[bw], (uint32_t)((r / NCARRY) & 1));
                __syncwarp();
                if (lane == 0) flag_st(&cw_taken[bw], r);
            }
            if (lane == 0 && lead) {
                SAM_TRACE(4, tile * p.M);
                if (SAM_EARLY_RELOAD == 2) flag_st(lb_started, r);  // its tiles may be re-fetched from L2 now
            }

            SAM_STRESS(2 + cw, tile);
            if (land_r) {
                mbar_wait(bar_lt, (uint32_t)(nland & 1));
                ++nland;
            }
            // seed of virtual super-tile -1 for lane mm: M(-1) applied for lanes before the phase
            auto seed_of = [&](int mm, CT* out) {
                if (p.seed) {
#pragma unroll
                    for (int t = 0; t < K; ++t) out[t] = CT(p.seed[mm * K + t]);
                    if ((uint64_t)mm < p.h) {
#pragma unroll
                        for (int t = K - 1; t >= 1; --t) out[t] = out[t] - out[t - 1];
                    }
                } else {
#pragma unroll
                    for (int t = 0; t < K; ++t) out[t] = CT(0);
                }
            };

            CT C[K];
            {
                // lane = (jl, mlb); row vv of window j holds the super-tile at distance
                // d = j*WV + jl + Wn*vv before S-1; rows beyond Sprev hold nothing, the row AT Sprev
                // holds this CTA's previous inclusive state (or, for r = 0, the seed of super-tile -1)
                const int Wn = p.Wn;
                const int jl = lane / s, mlb = lane - jl * s;
                const bool active = jl < Wn;
                CT total[K], Pm[K];
                const int j0 = tw, jstep = TW;
#pragma unroll
                for (int t = 0; t < K; ++t) { total[t] = CT(0); Pm[t] = p.bwinj[j0][t]; }  // Pm = M(j0 WV US)
                int npoll = 0;
                // Integers with the landing buffer: the global-frame fold is a plain sum of the
                // transformed aggregates, done value-parallel -- lane <-> (super-tile stripe, value
                // (m, t)), consecutive lanes on consecutive words (conflict-free smem reads), the 4
                // carry warps on interleaved super-tiles; stale words are re-polled from L2 one by one.
                // (order 1: M = 1, the fold is a plain sum in any frame)
                const bool vfold = (TRANSFORM || K == 1) && land_r && p.vfold;
                if (vfold) {
                    // lane <-> (stripe st, value vi) for s*K <= 32 (stripes of super-tiles side by side),
                    // lane <-> (vi, vi + 32) otherwise; warp cw takes stripes cw*ST + st, + NCARRY*ST, ...
                    const int VPT = s * K;
                    const int VL = VPT > 32 ? 32 : VPT;
                    const int ST = 32 / VL;             // stripes per warp
                    const int st = lane / VL, vi0 = lane - st * VL;
                    const bool lact = st < ST;
                    const int64_t nsup = tile - lo_sup;
                    CT acc[2][2] = {{CT(0), CT(0)}, {CT(0), CT(0)}};  // [h][parity]: two chains for ILP
                    if (p.trace && lead && lane == 0) SAM_TRACE(8, tile * p.M);
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        const int vi = vi0 + 32 * h;
                        if (!lact || vi >= VPT) continue;
                        int par = 0;
                        for (int64_t jj = (int64_t)tw * ST + st; jj < nsup; jj += (int64_t)TW * ST, par ^= 1) {
                            const unsigned long long* ls = (const unsigned long long*)(
                                land_s + ((uint32_t)jj * p.rec_words + vi * W1) * 8);
                            const uint32_t tj = ctag(lo_sup + jj);
                            unsigned long long w0 = ls[0], w1 = W1 == 2 ? ls[1] : 0ull;
                            while ((uint32_t)(w0 >> 32) != tj || (W1 == 2 && (uint32_t)(w1 >> 32) != tj)) {
                                const unsigned long long* src = cslot(lo_sup + jj) + vi * W1;  // stale: re-poll L2
                                if constexpr (W1 == 1) {
                                    w0 = ld_relaxed_u64(src);
                                } else {
                                    ld_relaxed_v2(src, w0, w1);
                                }
                                ++npoll;
                            }
                            const uint64_t b = W1 == 1 ? (w0 & 0xffffffffull) : ((w0 & 0xffffffffull) | (w1 << 32));
                            acc[h][par] += CT(Bits<T>::from(b));
                        }
                    }
                    CT v0 = acc[0][0] + acc[0][1], v1 = acc[1][0] + acc[1][1];
                    // stripes -> stripe 0 (tree over st; ST need not be a power of two)
                    for (int step = 1; step < ST; step <<= 1) {
                        const CT o = shfl_down(v0, step * VL);
                        if (lact && (st % (2 * step)) == 0 && st + step < ST) v0 += o;
                    }
                    CT* pv_s = (CT*)(smem + S::OFF_PV);  // [NCARRY][64]
                    if (st == 0) {
                        pv_s[cw * 64 + vi0] = v0;
                        pv_s[cw * 64 + 32 + vi0] = v1;
                    }
                    if (TW > 1) named_bar_sync(4 + team, TW * 32);
                    if (lead) {
                        // value vi summed over the warps by lane vi, then lane m collects its K values
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int vi = lane + 32 * h;
                            if (vi < VPT) {
                                const int slot = vi < 32 ? vi : 32 + (vi - 32);
                                CT a2 = pv_s[slot];
#pragma unroll
                                for (int w2 = 1; w2 < TW; ++w2) a2 += pv_s[(cw + w2) * 64 + slot];
                                pv_s[cw * 64 + slot] = a2;
                            }
                        }
                        __syncwarp();
                        if (lane_ok) {
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                const int vi = lane * K + t;
                                total[t] = pv_s[cw * 64 + vi];
                            }
                        }
                        if (lane == 0) {
                            SAM_TRACE(10, tile * p.M);
                            SAM_TRACE(13, tile * p.M);
                            if (p.trace) p.trace[(size_t)(tile * p.M) * 16 + 11] = npoll;
                        }
                    }
                }
                for (int j = j0; !vfold; j += jstep) {
                    const int64_t basei = tile - 1 - (int64_t)j * WV;
                    if (basei < Sprev) break;  // window j starts beyond Sprev: nothing left for this warp
                    unsigned long long w[V][K][W1];
                    int st[V];  // 0 pending, 1 aggregate valid, 2 previous inclusive / seed, 3 nothing
#pragma unroll
                    for (int vv = 0; vv < V; ++vv) {
                        const int64_t idx = basei - jl - (int64_t)Wn * vv;
                        st[vv] = (!active || vv >= p.Vr || idx <= Sprev) ? 3 : 0;
                    }
                    bool from_land = land_r;  // first pass from the landing buffer, re-polls from L2
                    // 32-bit row bookkeeping (rows step back by Wn super-tiles): ring slot, lap and
                    // landing index of row 0; row vv wraps to the previous lap when its slot goes negative
                    const int64_t idx0 = basei - jl;
                    const int slot0 = (int)((uint64_t)idx0 & (p.ring - 1));
                    const uint32_t lap0 = (uint32_t)((uint64_t)idx0 >> p.ring_log2);
                    const int dl0 = (int)(idx0 - lo_sup);
                    const uint32_t recw = p.rec_words;
                    for (;;) {
                        if (p.trace && lane == 0 && j == 0 && npoll == 0) SAM_TRACE(8, tile * p.M);
                        // all loads first, then the tag checks: the loads of a window are then in
                        // flight together (one round trip), not one after the other
#pragma unroll
                        for (int vv = 0; vv < V; ++vv) {
                            if (st[vv] == 0) {
                                int sl = slot0 - Wn * vv;
                                if (sl < 0) sl += (int)p.ring;
                                const unsigned long long* src = p.carry + (size_t)sl * recw + mlb * K * W1;
                                if (from_land) {
                                    const unsigned long long* ls = (const unsigned long long*)(
                                        land_s + ((uint32_t)(dl0 - Wn * vv) * recw + mlb * K * W1) * 8);
#pragma unroll
                                    for (int t = 0; t < K; ++t) {
#pragma unroll
                                        for (int h = 0; h < W1; ++h) w[vv][t][h] = ls[t * W1 + h];
                                    }
                                } else {
#pragma unroll
                                for (int t = 0; t < K; ++t) {
                                    if constexpr (W1 == 1) {
                                        w[vv][t][0] = ld_relaxed_u64(src + t);
                                    } else {
                                        ld_relaxed_v2(src + 2 * t, w[vv][t][0], w[vv][t][1]);
                                    }
                                }
                                }
                            }
                        }
                        from_land = false;
                        bool pend = false;
#pragma unroll
                        for (int vv = 0; vv < V; ++vv) {
                            if (st[vv] == 0) {
                                bool ok = true;
                                const uint32_t tv = tag | ((lap0 - (slot0 - Wn * vv < 0 ? 1u : 0u)) & 0xfffu);
#pragma unroll
                                for (int t = 0; t < K; ++t) {
                                    ok &= (uint32_t)(w[vv][t][0] >> 32) == tv;
                                    if constexpr (W1 == 2) ok &= (uint32_t)(w[vv][t][1] >> 32) == tv;
                                }
                                st[vv] = ok ? 1 : 0;
                                pend |= !ok;
                            }
                        }
                        if (p.trace && lane == 0 && j == 0 && npoll == 0) SAM_TRACE(9, tile * p.M);
                        ++npoll;
                        if (!__any_sync(0xffffffffu, pend)) break;
                        if (SAM_POLL_NS > 0) __nanosleep(SAM_POLL_NS);  // back off before re-polling L2
                    }
                    const bool last = basei - (int64_t)WV < Sprev;  // this window holds Sprev
                    if (p.trace && lane == 0 && last) {
                        SAM_TRACE(10, tile * p.M);
                        p.trace[(size_t)(tile * p.M) * 16 + 11] = npoll;
                    }
                    // fold.  This lane's rows sit at d = jl + Wn*vv (+ j*WV), so by Horner in vv:
                    //   sum_vv M((jl + Wn vv) US) X_vv = M(jl US) (X_0 + M(Wn US)(X_1 + M(Wn US)(X_2 + ...)))
                    CT Y[K];
#pragma unroll
                    for (int t = 0; t < K; ++t) Y[t] = CT(0);
#pragma unroll
                    for (int vv = V - 1; vv >= 0; --vv) {
                        CT X[K];
#pragma unroll
                        for (int t = 0; t < K; ++t) X[t] = CT(0);
                        if (st[vv] == 1) {
#pragma unroll
                            for (int t = 0; t < K; ++t) {
                                if constexpr (W1 == 1) {
                                    X[t] = CT(Bits<T>::from(w[vv][t][0] & 0xffffffffull));
                                } else {
                                    X[t] = CT(Bits<T>::from((w[vv][t][0] & 0xffffffffull) | (w[vv][t][1] << 32)));
                                }
                            }
                        }
                        if (vv == V - 1) {
#pragma unroll
                            for (int t = 0; t < K; ++t) Y[t] = X[t];
                        } else if constexpr (TRANSFORM) {  // global frame: aggregates just add
#pragma unroll
                            for (int t = 0; t < K; ++t) Y[t] += X[t];
                        } else {
#pragma unroll
                            for (int t = K - 1; t >= 0; --t) {  // Y <- M(Wn US) Y + X
                                CT acc2 = Y[t] + X[t];
#pragma unroll
                                for (int jj = 0; jj < t; ++jj) acc2 += p.bwn[t - jj] * Y[jj];
                                Y[t] = acc2;
                            }
                        }
                    }
                    if (active && !TRANSFORM) {  // Y <- M(jl US) Y
#pragma unroll
                        for (int t = K - 1; t >= 1; --t) {
                            CT acc2 = Y[t];
#pragma unroll
                            for (int jj = 0; jj < t; ++jj) acc2 += bl_s[jl * K + (t - jj)] * Y[jj];
                            Y[t] = acc2;
                        }
                    }
                    for (int off = 1; off < Wn; off <<= 1) {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            CT o = shfl_down(Y[t], off * s);
                            if (jl + off < Wn) Y[t] += o;
                        }
                    }
                    // lanes jl == 0 hold this window's sum; total += M(j WV US) Y
                    if constexpr (TRANSFORM) {
#pragma unroll
                        for (int t = 0; t < K; ++t) total[t] += Y[t];
                    } else {
#pragma unroll
                    for (int t = K - 1; t >= 0; --t) {
                        CT acc2 = Y[t];
#pragma unroll
                        for (int jj = 0; jj < t; ++jj) acc2 += Pm[t - jj] * Y[jj];
                        total[t] += acc2;
                    }
                    }
                    if (last) break;
                    if (!TRANSFORM) {   // Pm <- Pm * M(jstep*WV*US)  (truncated polynomial product)
                        CT np[K];
#pragma unroll
                        for (int d = 0; d < K; ++d) {
                            CT acc2 = CT(0);
#pragma unroll
                            for (int e2 = 0; e2 <= d; ++e2) acc2 += Pm[e2] * p.bwinj[jstep][d - e2];
                            np[d] = acc2;
                        }
#pragma unroll
                        for (int d = 0; d < K; ++d) Pm[d] = np[d];
                    }
                }
                if (coop && !vfold) {  // sum the warps' partial folds (all already at their absolute offsets)
                    CT* slot = part_s + (((r >> lgNT) & 1) * NCARRY + cw) * MAXS * K;
                    if (lane_ok) {
#pragma unroll
                        for (int t = 0; t < K; ++t) slot[lane * K + t] = total[t];
                    }
                    if (TW > 1) named_bar_sync(4 + team, TW * 32);
                    if (lead && lane == 0) SAM_TRACE(13, tile * p.M);
                    if (lead && lane_ok) {
                        for (int w2 = 1; w2 < TW; ++w2) {
                            const CT* o = part_s + (((r >> lgNT) & 1) * NCARRY + cw + w2) * MAXS * K;
#pragma unroll
                            for (int t = 0; t < K; ++t) total[t] += o[lane * K + t];
                        }
                    }
                }
                if (TRANSFORM && !p.dyn && coop && TW > 1 && tw == 1) {
                    // the next super-tile's b(S' US), S' = S + NT*P, for the lead (after the team barrier of
                    // this super-tile, so the slot it fills is read only after the next one)
                    if (r < NT) mcol<CT>(tile * (int64_t)p.M * p.U, K, gpos);
                    CT np2[K];
#pragma unroll
                    for (int d = 0; d < K; ++d) {
                        CT acc2 = CT(0);
#pragma unroll
                        for (int e2 = 0; e2 <= d; ++e2) acc2 += gpos[e2] * p.bposP[d - e2];
                        np2[d] = acc2;
                    }
#pragma unroll
                    for (int d = 0; d < K; ++d) gpos[d] = np2[d];
                    CT* gn = (CT*)(smem + S::OFF_GN) + (((r + NT) >> lgNT) & 1) * K;
                    if (lane == 0) {
#pragma unroll
                        for (int t = 0; t < K; ++t) gn[t] = np2[t];
                    }
                }
                if (lead) {
                    // the CTA's own chain, kept to a few operations: C = F + M((S-1-Sprev) US) I_prev,
                    // I_prev = this CTA's inclusive state after Sprev (hand-off) or, for r = 0, the seed
                    // of virtual super-tile -1 (M(S US) computed here, once per CTA)
                    CT pv[K], bcol[K];
                    bool have = false;
                    if (Sprev >= 0) {
                        const volatile int* rt = (const volatile int*)(smem + S::OFF_HO + ((r - 1) % NCARRY) * S::HOB);
                        while (flag_ld_acq(rt) != r - 1) __nanosleep(20);
                        __syncwarp();
                        const CT* hv = (const CT*)(smem + S::OFF_HO + ((r - 1) % NCARRY) * S::HOB + 16);
#pragma unroll
                        for (int t = 0; t < K; ++t) { pv[t] = hv[ml * K + t]; bcol[t] = p.bprev[t]; }
                        if (!TRANSFORM && K > 1 && p.dyn)  // floats: span from the previous super-tile to S-1
                            mcol<CT>((tile - 1 - Sprev) * (int64_t)p.M * p.U, K, bcol);
                        have = true;
                    } else if (p.seed) {
                        seed_of(ml, pv);
                        mcol<CT>(tile * (int64_t)p.M * p.U, K, bcol);
                        have = true;
                    }
                    if constexpr (TRANSFORM) {
                        // global frame (integers): A~_j = M(-(j+1) US) A_j were published, so the fold
                        // is a plain sum and the chain is a sum too: T~ = I~_prev + sum A~_j, and
                        // C_S = M(S US) T~ (gpos = b(S US), advanced by one round per super-tile)
                        if (have) {
#pragma unroll
                            for (int t = 0; t < K; ++t) total[t] += pv[t];
                        }
#pragma unroll
                        for (int t = 0; t < K; ++t) tsum[t] = total[t];
                        if (p.dyn) {
                            if (coop && TW > 1) {  // b(S US) from the team's second warp (above)
                                const CT* gn = (const CT*)(smem + S::OFF_GN) + (r & 1) * K;
#pragma unroll
                                for (int t = 0; t < K; ++t) gpos[t] = gn[t];
                            } else {
                                mcol<CT>(tile * (int64_t)p.M * p.U, K, gpos);
                            }
                        } else if (coop && TW > 1) {
                            // b(S US): computed here for the team's first super-tile, afterwards ahead of
                            // time by the team's second warp (off this serial path, see below)
                            if (r < NT) {
                                mcol<CT>(tile * (int64_t)p.M * p.U, K, gpos);
                            } else {
                                const CT* gn = (const CT*)(smem + S::OFF_GN) + ((r >> lgNT) & 1) * K;
#pragma unroll
                                for (int t = 0; t < K; ++t) gpos[t] = gn[t];
                            }
                        } else if (coop) {
                            if (r < NT) {  // the team's first super-tile; then NT rounds at a time
                                mcol<CT>(tile * (int64_t)p.M * p.U, K, gpos);
                            } else {
                                CT np2[K];
#pragma unroll
                                for (int d = 0; d < K; ++d) {
                                    CT acc2 = CT(0);
#pragma unroll
                                    for (int e2 = 0; e2 <= d; ++e2) acc2 += gpos[e2] * p.bposP[d - e2];
                                    np2[d] = acc2;
                                }
#pragma unroll
                                for (int d = 0; d < K; ++d) gpos[d] = np2[d];
                            }
                        } else {
                            mcol<CT>(tile * (int64_t)p.M * p.U, K, gpos);
                        }
#pragma unroll
                        for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                            for (int jj = 0; jj < t; ++jj) total[t] += gpos[t - jj] * total[jj];
                        }
                    } else if (have) {
#pragma unroll
                        for (int t = K - 1; t >= 0; --t) {
                            CT acc2 = total[t] + pv[t];
#pragma unroll
                            for (int jj = 0; jj < t; ++jj) acc2 += bcol[t - jj] * pv[jj];
                            total[t] = acc2;
                        }
                    }
                }
#pragma unroll
                for (int t = 0; t < K; ++t) C[t] = total[t];
            }
            if (!lead) continue;

            const int cnt = sub_of[2 * (i0 % NQ) + 1];
            const int il = i0 + cnt - 1;                 // its last iteration
            const T* la = la_all + (il % NQ) * S::LA;    // super-tile aggregate
            // hand the inclusive state M(M US) C + A to this CTA's next super-tile (in order
            // r-1 -> r: slot r % NCARRY is free once r-1's entry exists, r-1 having waited for r-2 ...)
            if (p.dyn || (uint64_t)tile + gridDim.x < p.num_super) {  // (dynamic: a next one may follow)
                if (r > 0) {
                    const volatile int* rt = (const volatile int*)(smem + S::OFF_HO + ((r - 1) % NCARRY) * S::HOB);
                    while (flag_ld_acq(rt) != r - 1) __nanosleep(20);
                }
                __syncwarp();
                unsigned char* ho = smem + S::OFF_HO + (r % NCARRY) * S::HOB;
                if (lane_ok) {
                    if constexpr (TRANSFORM) {  // I~_S = T~ + A~_S (la holds the transformed aggregate)
#pragma unroll
                        for (int t = 0; t < K; ++t) ((CT*)(ho + 16))[lane * K + t] = tsum[t] + la[ml * K + t];
                    } else {
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        CT acc2 = C[t] + la[ml * K + t];
#pragma unroll
                        for (int j = 0; j < t; ++j) acc2 += p.bus[t - j] * C[j];
                        ((CT*)(ho + 16))[lane * K + t] = acc2;
                    }
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    flag_st_rel((volatile int*)ho, r);
                }
            }
            if (lane == 0) SAM_TRACE(14, tile * p.M);
            SAM_STRESS(6, tile);
            // each sub-tile j: C_j = M(j U) C + P_j, then per-warp incoming states
            // C_{m,q} = M(q*Uw) C_{j,m} + E_{m,q}  (E in wq, from the combine)
            for (int j = 0; j < cnt; ++j) {
                const int qj = (i0 + j) % NQ;
                T* wq = wq_all + qj * S::WQ;
                T* lp = lp_all + qj * S::LA;
                CT Cj[K];
#pragma unroll
                for (int t = K - 1; t >= 0; --t) {
                    CT acc2 = C[t] + lp[ml * K + t];
#pragma unroll
                    for (int d = 0; d < t; ++d) acc2 += p.bsub[j][t - d] * C[d];
                    Cj[t] = acc2;
                }
                if constexpr (TRANSFORM) {
                    // integers: the sub-tile's carry C_j per lane goes to the compute threads, which
                    // form M(q Uw) (C_j + E'_q) themselves (no per-warp pass on this serial path)
                    __syncwarp();
                    if (lane_ok) {
#pragma unroll
                        for (int t = 0; t < K; ++t) lp[ml * K + t] = T(Cj[t]);
                    }
                }
#pragma unroll
                for (int ch = 0; ch < 2; ++ch) {
                    if constexpr (TRANSFORM) break;
                    if (32 * ch >= npair) break;  // warp-uniform: second pass only for s = 8
                    const int pair = lane + 32 * ch;
                    const bool ok = pair < npair;
                    const int mm = ok ? (pair >> p.logc) : 0, qq = pair & (c - 1);
                    CT Cm[K];
#pragma unroll
                    for (int t = 0; t < K; ++t) Cm[t] = shfl_idx(Cj[t], mm);
                    if (ok) {
                        if constexpr (TRANSFORM) {  // M(q Uw) (C_m + E'_q)
#pragma unroll
                            for (int t = 0; t < K; ++t) Cm[t] += wq[(qq * s + mm) * K + t];
#pragma unroll
                            for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                                for (int d = 0; d < t; ++d) Cm[t] += bq_s[qq * K + (t - d)] * Cm[d];
                            }
#pragma unroll
                            for (int t = 0; t < K; ++t) wq[(qq * s + mm) * K + t] = T(Cm[t]);
                        } else {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            CT acc2 = Cm[t] + wq[(qq * s + mm) * K + t];
#pragma unroll
                            for (int d = 0; d < t; ++d) acc2 += bq_s[qq * K + (t - d)] * Cm[d];
                            wq[(qq * s + mm) * K + t] = T(acc2);
                        }
                        }
                    }
                }
                __syncwarp();
                if (lane == 0) SAM_TRACE(5, tile_of[qj]);
                mbar_arrive(&bar_carry[qj]);
            }
        }
    } else {
        // =========================== compute warps ===============================================
        const bool is_p2_group = SPLIT && warp >= NW;  // SPLIT: warps [NW, 2NW) apply carries
        const int cwarp = warp % NW;                   // warp within its group
        const int gtid = tid % NCT;                    // thread within its group
        const int G = p.G, Pw = p.Pw;
        const int g = cwarp % p.sp, q = cwarp / p.sp;
        const int a = lane & (G - 1), v = lane >> p.logG;
        const int m = g * G + a;
        const int u = q * Pw + v;
        const int base_loc = u * ITEMS * s + m;  // element index inside the tile of item 0

        // a6 for iteration `it` (tile `tile`, local exclusive state e)
        auto carry_apply = [&](int it, int64_t tile, const T* e) {
            const int b2 = it % NB2;
            const int qs = it % NQ;
            if (gtid == 0) SAM_TRACE(6, tile);
            SAM_STRESS(8 + warp, tile);
            T* xs = (T*)(smem + S::OFF_BUF2 + b2 * S::BUFB + p.delta);
            const T* wq = wq_all + qs * S::WQ;
            const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
            const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);
            T y[K];
            {
                T Cq[K];
#pragma unroll
                for (int t = 0; t < K; ++t) Cq[t] = wq[(q * s + m) * K + t];
                if constexpr (TRANSFORM) {  // y = M(v ITEMS) (M(q Uw) (C_j + E'_q) + e')
                    const T* cj = lp_all + qs * S::LA;  // the sub-tile's carry, lane m
#pragma unroll
                    for (int t = 0; t < K; ++t) Cq[t] += cj[m * K + t];
#pragma unroll
                    for (int t = K - 1; t >= 1; --t) {
#pragma unroll
                        for (int d = 0; d < t; ++d) Cq[t] += bq_s[q * K + (t - d)] * Cq[d];
                    }
#pragma unroll
                    for (int t = 0; t < K; ++t) Cq[t] += e[t];
#pragma unroll
                    for (int t = 0; t < K; ++t) {
                        T acc2 = Cq[t];
#pragma unroll
                        for (int j = 0; j < t; ++j) acc2 += bt_s[(t - j) * 32 + v] * Cq[j];
                        y[t] = acc2;
                    }
                } else {
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T acc2 = e[t] + Cq[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) acc2 += bt_s[(t - j) * 32 + v] * Cq[j];
                    y[t] = acc2;
                }
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
                    // all ITEMS loads first: interleaving them with the (possibly aliasing, as far
                    // as the compiler knows) stores would serialise every item on an smem round trip
                    // (the slow edge-tile path loads each item where it is used instead: it is cold,
                    // and holding ITEMS values there only costs registers)
                    T xv[SLOW ? 1 : ITEMS];
                    if constexpr (VEC && !SLOW) {
                        lds_vec<T, ITEMS>(xs + base_loc, xv);
                    } else if constexpr (!SLOW) {
#pragma unroll
                        for (int i = 0; i < ITEMS; ++i) xv[i] = xs[base_loc + i * s];
                    }
                    T ov[VEC && !SLOW ? ITEMS : 1];
                    if constexpr (VEC && !SLOW && K == 1) {
                        // order 1: chunked prefix (ITEMS/7 independent chains of 7, then chunk offsets):
                        // dependent-add depth 7 + ITEMS/7 instead of ITEMS
                        constexpr int L = 7, CH = ITEMS / L;
                        T pre[ITEMS];
#pragma unroll
                        for (int c2 = 0; c2 < CH; ++c2) {
                            pre[c2 * L] = xv[c2 * L];
#pragma unroll
                            for (int j = 1; j < L; ++j) pre[c2 * L + j] = pre[c2 * L + j - 1] + xv[c2 * L + j];
                        }
                        T off = y[0];
#pragma unroll
                        for (int c2 = 0; c2 < CH; ++c2) {
                            const T base = off;
                            off += pre[c2 * L + L - 1];
#pragma unroll
                            for (int j = 0; j < L; ++j) pre[c2 * L + j] += base;
                        }
                        if constexpr (EXCL) {
                            ov[0] = ring[0];  // y at the position before the thread's first item
#pragma unroll
                            for (int i = 1; i < ITEMS; ++i) ov[i] = pre[i - 1];
                        } else {
#pragma unroll
                            for (int i = 0; i < ITEMS; ++i) ov[i] = pre[i];
                        }
                        sts_vec<T, ITEMS>(xs + base_loc, ov);
                        return;
                    }
#pragma unroll(SLOW ? 1 : ITEMS)
                    for (int i = 0; i < ITEMS; ++i) {
                        const int el = base_loc + i * s;
                        bool valid = true;
                        uint64_t ve = 0;
                        T x;
                        if constexpr (SLOW) {
                            ve = e0 + el;
                            valid = !masked || (ve >= p.h && ve < p.h + p.n);
                            x = valid ? xs[el] : T(0);
                        } else {
                            x = xv[i];
                        }
                        y[0] += x;
#pragma unroll
                        for (int t = 1; t < K; ++t) y[t] += y[t - 1];
                        T outv;
                        if constexpr (EXCL && SLOW) {  // not unrolled: rotate the ring (static indices)
                            outv = ring[0];
#pragma unroll
                            for (int d = 0; d + 1 < K; ++d) ring[d] = ring[d + 1];
                            ring[K - 1] = y[K - 1];
                        } else if constexpr (EXCL) {  // y_K of item i-K (ring slot i%K), then remember item i
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
                        } else if constexpr (VEC) {
                            ov[i] = outv;
                        } else {
                            xs[el] = outv;
                        }
                    }
                    if constexpr (VEC && !SLOW) sts_vec<T, ITEMS>(xs + base_loc, ov);
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
                named_bar_sync(2 + (is_p2_group ? 1 : 0), NCT);
                for (uint64_t ve = lo + gtid; ve < hi; ve += NCT) p.out[ve - p.h] = xs[ve - e0];
            }
            mbar_arrive(&bar_stored2[b2]);
        };

        // a3 for iteration i (tile loaded in local-scan buffer b1): zero-seeded local scan, warp
        // states to wq, returns the thread's local exclusive state e
        auto local_scan = [&](int i, int b1, T* e) {
            const int qs = i % NQ;
            const int64_t tile = tile_of[qs];
            if (gtid == 0) SAM_TRACE(1, tile);
            SAM_STRESS(32 + warp, tile);
            const T* xs = (const T*)(smem + S::OFF_BUF1 + b1 * S::BUFB + p.delta);
            T* wq = wq_all + qs * S::WQ;
            const uint64_t e0 = (uint64_t)tile * (uint64_t)Tt;
            const bool masked = (e0 < p.h) || (e0 + Tt > p.h + p.n);
            // a2/a3: lane run, thread-serial zero-seeded recurrence
            T acc[K];
#pragma unroll
            for (int t = 0; t < K; ++t) acc[t] = T(0);
            if (VEC && !masked) {
                T xv[ITEMS];
                lds_vec<T, ITEMS>(xs + base_loc, xv);
                if constexpr (K == 1) {  // order 1 needs only the sum: 4 independent chains
                    T a4[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll
                    for (int it = 0; it < ITEMS; ++it) a4[it & 3] += xv[it];
                    acc[0] = (a4[0] + a4[1]) + (a4[2] + a4[3]);
                } else {
#pragma unroll
                for (int it = 0; it < ITEMS; ++it) {
                    acc[0] += xv[it];
#pragma unroll
                    for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
                }
                }
            } else if (!masked) {
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
            // a3: warp scan of thread states.  Orders 1, 2: order by order, plain shuffle scans
            //   e_{v+1} = M(ITEMS) e_v + a_v  =>  e_{v+1}[t] = e_v[t] + z_v[t],
            //   z_v[t] = a_v[t] + sum_{j<t} b_{t-j}(ITEMS) e_v[j]      (5k dependent shuffle stages)
            // Orders >= 3: Kogge-Stone on k-vectors with the carry operator, level l combining
            //   st <- M(2^l ITEMS) st_partner + st                       (5 dependent stages)
            if constexpr (TRANSFORM) {
                // Integers, orders >= 2: similarity transform.  With z_u = M(-(u+1) ITEMS) a_u,
                //   e_v = sum_{u<v} M((v-1-u) ITEMS) a_u = M(v ITEMS) sum_{u<v} z_u,
                // so the k-vector scan becomes K independent plain shuffle scans (depth 5, no
                // matrix per level); e' = sum_{u<v} z_u is kept and M(v ITEMS) is applied in the
                // carry application, where it merges with the carry's own M(v ITEMS) (exact mod 2^w).
                T z[K], Z[K];
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T acc2 = acc[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) acc2 += bn_s[(t - j) * 32 + v] * acc[j];
                    z[t] = acc2;
                    Z[t] = acc2;
                }
#pragma unroll
                for (int l = 0; l < 5; ++l) {
                    const int off = G << l;
                    if (off < 32) {
#pragma unroll
                        for (int t = 0; t < K; ++t) {
                            T o = shfl_up(Z[t], off);
                            if (lane >= off) Z[t] += o;
                        }
                    }
                }
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    e[t] = Z[t] - z[t];
                    if (v == Pw - 1) wq[(q * s + m) * K + t] = Z[t];  // transformed warp total of lane m
                }
            } else if constexpr (K < SAM_KS_MIN_K) {
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T z = acc[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) z += p.bc[t - j] * e[j];
                    T y = z;
#pragma unroll
                    for (int l = 0; l < 5; ++l) {  // shuffle offsets G, 2G, ... < 32 (unrolled)
                        const int off = G << l;
                        if (off < 32) {
                            T o = shfl_up(y, off);
                            if (lane >= off) y += o;
                        }
                    }
                    if constexpr (IsInt<T>::value) {
                        e[t] = y - z;
                    } else {
                        T o = shfl_up(y, G);
                        e[t] = (lane >= G) ? o : T(0);
                    }
                    if (v == Pw - 1) wq[(q * s + m) * K + t] = y;  // warp aggregate of lane m
                }
            } else {
                T st[K];
#pragma unroll
                for (int t = 0; t < K; ++t) st[t] = acc[t];
#pragma unroll
                for (int l = 0; l < 5; ++l) {
                    const int off = G << l;
                    if (off < 32) {
                        T o[K];
#pragma unroll
                        for (int t = 0; t < K; ++t) o[t] = shfl_up(st[t], off);
                        if (lane >= off) {
#pragma unroll
                            for (int t = K - 1; t >= 0; --t) {
                                T acc2 = st[t] + o[t];
#pragma unroll
                                for (int j = 0; j < t; ++j) acc2 += p.bks[l][t - j] * o[j];
                                st[t] = acc2;
                            }
                        }
                    }
                }
#pragma unroll
                for (int t = 0; t < K; ++t) {
                    T o = shfl_up(st[t], G);
                    e[t] = (lane >= G) ? o : T(0);
                    if (v == Pw - 1) wq[(q * s + m) * K + t] = st[t];  // warp aggregate of lane m
                }
            }
            mbar_arrive(&bar_p1[qs]);  // warp states ready; P1 buffer free for the producer
        };

        T* const eq_s = (T*)(smem + S::OFF_EQ);  // [LAG][TILE_THREADS][K] pending states (ESMEM)
        volatile int* p2_cnt = (volatile int*)(smem + S::OFF_TAG + 12);  // SPLIT: P2 warp-tiles done
        if constexpr (SPLIT) {
            // Two groups: local scans never wait behind carry applications and vice versa.
            if (!is_p2_group) {
                for (int i = 0;; ++i) {
                    const int b1 = i % NB1;
                    if (!wait_or_end(&bar_full1[b1], (uint32_t)((i / NB1) & 1), i)) break;
                    // the pending-state slot i % lag must have been consumed by P2 of i - lag
                    while (flag_ld_acq(p2_cnt) < (i - lag + 1) * NW) __nanosleep(32);
                    T e[K];
                    local_scan(i, b1, e);
                    if constexpr (EGMEM) {
                        T* pe = p.pend + ((size_t)blockIdx.x * LAG + (i % LAG)) * K * TILE_THREADS + gtid;
#pragma unroll
                        for (int t = 0; t < K; ++t) pe[t * TILE_THREADS] = e[t];
                    } else {
#pragma unroll
                        for (int t = 0; t < K; ++t) eq_s[((i % LAG) * TILE_THREADS + gtid) * K + t] = e[t];
                    }
                }
            } else {
                for (int i = 0;; ++i) {
                    const int b2 = i % NB2;
                    if (!wait_or_end(&bar_full2[b2], (uint32_t)((i / NB2) & 1), i)) break;
                    if (SAM_EARLY_RELOAD) mbar_wait(&bar_carry[i % NQ], (uint32_t)((i / NQ) & 1));
                    T e[K];
                    if constexpr (EGMEM) {
                        const T* pe = p.pend + ((size_t)blockIdx.x * LAG + (i % LAG)) * K * TILE_THREADS + gtid;
#pragma unroll
                        for (int t = 0; t < K; ++t) e[t] = pe[t * TILE_THREADS];
                    } else {
#pragma unroll
                        for (int t = 0; t < K; ++t) e[t] = eq_s[((i % LAG) * TILE_THREADS + gtid) * K + t];
                    }
                    carry_apply(i, tile_of[i % NQ], e);
                    __syncwarp();
                    if (lane == 0) {
                        __threadfence_block();  // this warp's reads of its pending states come first
                        atomicAdd((int*)p2_cnt, 1);
                    }
                }
            }
        } else {
            // One group.  A loaded tile's local scan (P1) always goes first, so its aggregate is
            // published as early as possible (predecessor aggregates gate every carry fold); a
            // tile's carry application (P2) runs once the producer has re-fetched it.  Up to LAG
            // tiles sit between P1 and P2, their local states in registers (static ring eq).
            T eq[(ESMEM || EGMEM) ? 1 : LAG][K];  // register ring only when the states are in neither smem nor L2
            int p1_next = 0, p2_next = 0;
            int end = -1;  // end-of-stream iteration, refreshed only when idle
            for (;;) {
                if ((end < 0 || p1_next < end) && p1_next < p2_next + lag) {
                    const int i = p1_next;
                    const int b1 = i % NB1;
                    const uint32_t par = (uint32_t)((i / NB1) & 1);
                    const bool ready = __shfl_sync(0xffffffffu, lane == 0 ? (int)mbar_test(&bar_full1[b1], par) : 0, 0);
                    if (ready) {
                        mbar_wait(&bar_full1[b1], par);
                        T e[K];
                        local_scan(i, b1, e);
                        if constexpr (EGMEM) {
                            T* pe = p.pend + ((size_t)blockIdx.x * LAG + (i % LAG)) * K * TILE_THREADS + gtid;
#pragma unroll
                            for (int t = 0; t < K; ++t) pe[t * TILE_THREADS] = e[t];
                        } else if constexpr (ESMEM) {
#pragma unroll
                            for (int t = 0; t < K; ++t) eq_s[((i % LAG) * TILE_THREADS + gtid) * K + t] = e[t];
                        } else {
#pragma unroll
                            for (int j = 0; j < LAG; ++j) {
                                if (j == i % LAG) {
#pragma unroll
                                    for (int t = 0; t < K; ++t) eq[j][t] = e[t];
                                }
                            }
                        }
                        ++p1_next;
                        continue;
                    }
                }
                if (p2_next < p1_next) {
                    const int i = p2_next;
                    const int b2 = i % NB2;
                    const uint32_t par = (uint32_t)((i / NB2) & 1);
                    const bool ready = __shfl_sync(0xffffffffu, lane == 0 ? (int)(mbar_test(&bar_full2[b2], par) &&
                        (!SAM_EARLY_RELOAD || mbar_test(&bar_carry[i % NQ], (uint32_t)((i / NQ) & 1)))) : 0, 0);
                    if (ready) {
                        mbar_wait(&bar_full2[b2], par);
                        if (SAM_EARLY_RELOAD) mbar_wait(&bar_carry[i % NQ], (uint32_t)((i / NQ) & 1));
                        T e[K];
                        if constexpr (EGMEM) {
                            const T* pe = p.pend + ((size_t)blockIdx.x * LAG + (i % LAG)) * K * TILE_THREADS + gtid;
#pragma unroll
                            for (int t = 0; t < K; ++t) e[t] = pe[t * TILE_THREADS];
                        } else if constexpr (ESMEM) {
#pragma unroll
                            for (int t = 0; t < K; ++t) e[t] = eq_s[((i % LAG) * TILE_THREADS + gtid) * K + t];
                        } else {
#pragma unroll
                            for (int j = 0; j < LAG; ++j) {
                                if (j == i % LAG) {
#pragma unroll
                                    for (int t = 0; t < K; ++t) e[t] = eq[j][t];
                                }
                            }
                        }
                        carry_apply(i, tile_of[i % NQ], e);
                        ++p2_next;
                        continue;
                    }
                } else if (end >= 0 && p1_next >= end) {
                    break;
                }
                // warp-uniform refresh: one atomic read, broadcast (per-lane atomics could see
                // different values and split the warp's control flow)
                end = __shfl_sync(0xffffffffu, lane == 0 ? flag_ld(sm_end) : 0, 0);
                __nanosleep(SAM_IDLE_NS);  // nothing ready: yield issue slots to the other warps
            }
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
            *(volatile unsigned int*)p.reset_ctr = 0u;
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

// Block-cyclic multi-GPU: SAM's carry scheme with the GPUs as the persistent
// blocks.  `payloads` = the nranks chunk payloads of one round (rank order), base_in =
// the state before the round (null: zero).  seed_out = base (+) payloads of ranks < rank (the carry
// into this rank's chunk); base_out (optional) = base (+) all of them (the next round's base).
// One thread per tuple lane; every rank folds the same bytes in the same order, so all ranks hold
// bit-identical bases.
template <typename T>
__global__ void sam_cyclic_fold_kernel(const unsigned char* payloads, size_t payload_bytes, int rank, int nranks,
                                       int k, int s, const T* base_in, T* seed_out, T* base_out) {
    const int mm = threadIdx.x;
    if (mm >= s) return;
    T st[MAXK];
    for (int t = 0; t < k; ++t) st[t] = base_in ? base_in[(size_t)mm * k + t] : T(0);
    fold_payloads_from<T>(st, payloads, payload_bytes, rank, k, s, mm, st);
    for (int t = 0; t < k; ++t) seed_out[(size_t)mm * k + t] = st[t];
    if (base_out) {
        fold_payloads_from<T>(st, payloads + (size_t)rank * payload_bytes, payload_bytes, nranks - rank, k, s, mm, st);
        for (int t = 0; t < k; ++t) base_out[(size_t)mm * k + t] = st[t];
    }
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
