// sam_launch.cuh -- host-side launch of the scan kernel for one (element type, order).
// Instantiated per element type in sam_inst_*.cu; called by the C ABI in sam_api.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "sam_algebra.h"
#include "sam_kernel.cuh"

namespace sam {

// Tile geometry for tuple size s: a warp holds G lanes (G = largest power of two
// dividing s) with Pw = 32/G threads per lane; sp = s/G lane groups; c warps per lane group.
struct Geom {
    int s, G, logG, sp, c, logc, Pw, W, Wn, Uw, U, T;
};

inline int ilog2(int x) {
    int r = 0;
    while ((1 << r) < x) ++r;
    return r;
}

inline Geom make_geom(int s, int items) {
    Geom g;
    g.s = s;
    g.G = s & -s;
    g.logG = ilog2(g.G);
    g.sp = s / g.G;
    int c = 8 / g.sp;
    if (c < 1) c = 1;
    while (c & (c - 1)) c &= c - 1;  // power of two
    g.c = c;
    g.logc = ilog2(c);
    g.W = g.sp * g.c;
    g.Pw = 32 / g.G;
    g.Uw = g.Pw * items;
    g.U = g.c * g.Uw;
    g.T = g.s * g.U;
    g.Wn = 32 / s;
    return g;
}

struct LaunchArgs {
    const void* in;
    void* out;
    uint64_t n;
    uint64_t g;            // global index of in[0]
    const void* seed;      // [s][k] or null
    void* final_state;     // [s][k] or null
    int s;
    int inclusive;
    int store_mode;
    cudaStream_t stream;
    // workspace
    unsigned long long* carry;
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned int* epoch_ptr;
    unsigned long long* trace;
    int num_sms;
};

template <typename T>
inline int items_of() { return Cfg<T>::ITEMS; }

template <typename T, int K, bool VEC>
struct KernelInfo {
    int max_blocks_per_sm = 0;
    bool ready = false;
    std::mutex mu;
};

// persistent grid: all co-resident CTAs, at most one per super-tile
inline uint64_t grid_of(int blocks_per_sm, int num_sms, uint64_t num_super) {
    uint64_t grid = (uint64_t)blocks_per_sm * (uint64_t)num_sms;
    if (grid > num_super) grid = num_super;
    return grid < 1 ? 1 : grid;
}

template <typename T, int K, bool VEC>
cudaError_t launch_scan_impl(const LaunchArgs& a, uint64_t* launches) {
    using S = Smem<T, K, VEC>;
    constexpr int ITEMS = Items<T, VEC>::V;
    static KernelInfo<T, K, VEC> info;
    {
        std::lock_guard<std::mutex> lk(info.mu);
        if (!info.ready) {
            cudaError_t e = cudaFuncSetAttribute(sam_scan_kernel<T, K, VEC>,
                                                 cudaFuncAttributeMaxDynamicSharedMemorySize, S::BYTES);
            if (e != cudaSuccess) return e;
            int nb = 0;
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sam_scan_kernel<T, K, VEC>, Threads<T, K>::VALUE, S::BYTES);
            if (e != cudaSuccess) return e;
            info.max_blocks_per_sm = nb > 0 ? nb : 1;
            info.ready = true;
        }
    }
    const Geom geo = make_geom(a.s, ITEMS);
    Params<T, K> p;
    memset(&p, 0, sizeof(p));
    p.in = (const T*)a.in;
    p.out = (T*)a.out;
    p.n = a.n;
    p.h = a.g % (uint64_t)a.s;
    p.num_tiles = (p.h + a.n + geo.T - 1) / geo.T;
    p.delta = (uint32_t)(((uintptr_t)a.in - p.h * sizeof(T)) & 15);
    p.s = geo.s; p.G = geo.G; p.logG = geo.logG; p.sp = geo.sp; p.c = geo.c; p.logc = geo.logc;
    p.Pw = geo.Pw; p.W = geo.W; p.Wn = geo.Wn; p.U = geo.U; p.T_ = geo.T; p.Uw = geo.Uw;
    p.inclusive = a.inclusive;
    p.store_mode = a.store_mode;
    if (const char* env = getenv("SAM_CLAIM_SLACK")) {  // experiments (ring slots allow at most 2)
        const int v = atoi(env);
        p.claim_slack = v < 0 ? 0 : (v > 2 ? 2 : v);
    }
    p.seed = (const T*)a.seed;
    p.final_state = (T*)a.final_state;
    for (int m = 0; m < MAXS; ++m) {
        p.last_e[m] = -1;
        if (m < a.s && a.n > 0) {
            const int64_t eend = (int64_t)(p.h + a.n - 1);
            const int64_t le = eend - ((eend - m) % a.s + a.s) % a.s;
            if (le >= (int64_t)p.h && le >= 0) p.last_e[m] = le;
        }
    }
    p.carry = a.carry;
    p.tile_ctr = a.tile_ctr;
    p.done_ctr = a.done_ctr;
    p.epoch_ptr = a.epoch_ptr;
    p.trace = a.trace;
    // super-tile size: up to MMAX tiles per look-back unit, but keep >= 2 super-tiles per SM
    {
        uint64_t m = p.num_tiles / (2ull * (uint64_t)(a.num_sms > 0 ? a.num_sms : 148));
        if (m < 1) m = 1;
        // measured: tuple 1: 3 (4-byte) / 2 (8-byte) tiles; tuples (more carry-team work per unit):
        // 3, or 4 for odd tuples of 4-byte elements (~1.5% better there)
        const uint64_t mmax = a.s == 1 ? (uint64_t)Lag<T, K>::MMAX : ((sizeof(T) == 4 && (a.s & 1)) ? 4u : 3u);
        if (m > mmax) m = mmax;
        if (const char* env = getenv("SAM_SUPER_TILE")) {  // experiments: force a smaller super-tile
            const int f = atoi(env);
            if (f >= 1 && f <= 8) m = (uint64_t)f;
        }
        // a super-tile is aggregated before its carry is known: at most LAG/2 tiles per unit
        // keep two units in flight per CTA (LAG bounds the tiles between load and carry application)
        const uint64_t mlag = Lag<T, K>::LAG / 2 > 1 ? Lag<T, K>::LAG / 2 : 1;
        if (m > mlag) m = mlag;
        p.M = (int)m;
        p.num_super = (p.num_tiles + m - 1) / m;
    }
    const int64_t US = (int64_t)p.M * geo.U;  // lane length of a super-tile
    mcol<T>(ITEMS, K, p.bc);
    mcol<T>(geo.Uw, K, p.bw);
    mcol<T>(geo.U, K, p.bu);
    mcol<T>(US, K, p.bus);
    constexpr int V = LB<T, K>::V;
    {   // window rows: enough for the carry warps together to cover the P-1 aggregates in one round trip
        const uint64_t P = grid_of(info.max_blocks_per_sm, a.num_sms, p.num_super);
        const uint64_t rows = (P + geo.Wn - 1) / geo.Wn;
        uint64_t vr = (rows + NCARRY - 1) / NCARRY;
        if (vr < 1) vr = 1;
        if (vr > (uint64_t)V) vr = V;
        vr = V;  // measured: the full register budget per round trip beats spreading rows over warps
        if (const char* env = getenv("SAM_VR")) { const int f = atoi(env); if (f >= 1 && f <= V) vr = f; }
        p.Vr = (int)vr;
    }
    for (int j = 0; j <= NCARRY; ++j) mcol<T>((int64_t)j * geo.Wn * p.Vr * US, K, p.bwinj[j]);
    mcol<T>((int64_t)(grid_of(info.max_blocks_per_sm, a.num_sms, p.num_super) - 1) * US, K, p.bprev);
    mcol<T>((int64_t)geo.Wn * US, K, p.bwn);
    for (int v = 0; v < 32; ++v) {
        T b[K];
        mcol<T>((int64_t)v * ITEMS, K, b);
        for (int d = 0; d < K; ++d) p.bt[d][v] = b[d];
    }
    for (int q = 0; q < 8; ++q) mcol<T>((int64_t)q * geo.Uw, K, p.bq[q]);
    for (int j = 0; j < 32; ++j) mcol<T>((int64_t)j * US, K, p.bl[j]);
    for (int j = 0; j < 8; ++j) mcol<T>((int64_t)j * geo.U, K, p.bsub[j]);
    for (int l = 0; l < 5; ++l) mcol<T>((int64_t)(1 << l) * ITEMS, K, p.bks[l]);
    for (int l = 0; l < 3; ++l) mcol<T>((int64_t)(1 << l) * geo.Uw, K, p.bkw[l]);

    // persistent: one CTA per SM (warp-specialised: geo.W compute warps + producer, aggregator, carry warps)
    // carry warps cooperate on each super-tile when its fold spans 3 or more windows
    {
        const uint64_t wv = (uint64_t)geo.Wn * V;
        const uint64_t P = grid_of(info.max_blocks_per_sm, a.num_sms, p.num_super);
        p.coop = 1;  // measured faster for every config tried, also single-window folds
        (void)P; (void)wv;
        if (const char* env = getenv("SAM_COOP")) p.coop = atoi(env) != 0;  // experiments
    }
    // Static schedule (CTA b owns super-tiles b, b+P, ...): every CTA waits on aggregates of the
    // others, so all P CTAs must be co-resident -- a cooperative launch guarantees it (or fails).
    const uint64_t grid = grid_of(info.max_blocks_per_sm, a.num_sms, p.num_super);
    cudaLaunchConfig_t cfg;
    memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3((Threads<T, K>::GROUPS * geo.W + SERVICE_WARPS) * 32);
    cfg.dynamicSmemBytes = S::BYTES;
    cfg.stream = a.stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, sam_scan_kernel<T, K, VEC>, p);
    if (launches && e == cudaSuccess) ++*launches;
    return e != cudaSuccess ? e : cudaGetLastError();
}

// tuple 1 with a 16-B aligned input: the 128-bit shared-memory variant
template <typename T, int K>
cudaError_t launch_scan_tk(const LaunchArgs& a, uint64_t* launches) {
    const bool vec = a.s == 1 && ((uintptr_t)a.in & 15) == 0 && getenv("SAM_NO_VEC") == nullptr;
    return vec ? launch_scan_impl<T, K, true>(a, launches) : launch_scan_impl<T, K, false>(a, launches);
}

template <typename T>
cudaError_t launch_fold(const void* payloads, size_t payload_bytes, int rank, int k, int s, void* seed,
                        cudaStream_t st, uint64_t* launches) {
    sam_fold_kernel<T><<<1, 32, 0, st>>>((const unsigned char*)payloads, payload_bytes, rank, k, s, (T*)seed);
    if (launches) ++*launches;
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_payload_init(void* payload, uint64_t n, uint64_t g, int k, int s, const void* seed,
                                int write_header, void* final_state, cudaStream_t st, uint64_t* launches) {
    sam_payload_init_kernel<T><<<1, 64, 0, st>>>((unsigned char*)payload, n, g, k, s, (const T*)seed,
                                                 write_header, (T*)final_state);
    if (launches) ++*launches;
    return cudaGetLastError();
}

}  // namespace sam

#define SAM_INSTANTIATE(T)                                                                             \
    namespace sam {                                                                                    \
    template cudaError_t launch_scan_tk<T, 1>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 2>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 3>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 4>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 5>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 6>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 7>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_scan_tk<T, 8>(const LaunchArgs&, uint64_t*);                           \
    template cudaError_t launch_fold<T>(const void*, size_t, int, int, int, void*, cudaStream_t,       \
                                        uint64_t*);                                                    \
    template cudaError_t launch_payload_init<T>(void*, uint64_t, uint64_t, int, int, const void*, int, \
                                                void*, cudaStream_t, uint64_t*);                       \
    }
