// sam_launch.cuh -- host-side launch of the scan kernel for one (element type, order).
// Instantiated per element type in sam_inst_*.cu; called by the C ABI in sam_api.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <dlfcn.h>
#include <stdio.h>

#include <map>
#include <mutex>
#include <string>
#include <vector>

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
    unsigned long long carry_words;  // capacity of `carry` in 64-bit words (wrap-around reset)
    unsigned int* reset_ctr;         // grid barrier of the epoch wrap-around reset
    void* pend;                      // pending-state scratch (states > 16 B), pend_bytes() of the workspace
    int num_sms;
    int dev;
};

template <typename T>
inline int items_of() { return Cfg<T>::ITEMS; }

// Experiment knobs (developer tools only), read from the environment ONCE per process -- never on
// the per-launch path.  0 / -1 = unset.
struct Knobs {
    int claim_slack = 0;   // SAM_CLAIM_SLACK: extra claimed-but-blocked tiles (ring slots allow <= 2)
    int super_tile = 0;    // SAM_SUPER_TILE: force the tiles per super-tile (1..8)
    int vr = 0;            // SAM_VR: window rows per round trip
    int coop = -1;         // SAM_COOP: carry warps fold each super-tile together (1) or round-robin (0)
    bool no_vec = false;   // SAM_NO_VEC: never take the 128-bit tuple-1 path
    int lag = 0;           // SAM_LAG: pipeline depth (tiles between local scan and carry application), <= LAG
    int land = -1;         // SAM_LAND: landing-buffer folds on (1) / off (0)
    int vfold = -1;        // SAM_VFOLD: value-parallel integer folds on (1) / off (0)
    int teams = 0;         // SAM_TEAMS: carry teams (1, 2 or 4)
    int dyn = -1;          // SAM_DYN: dynamic (claim-order) super-tile schedule (1) or static b, b+P, ... (0)
};
inline Knobs& knobs_mut() {
    static Knobs k = [] {
        Knobs r;
        if (const char* e = getenv("SAM_CLAIM_SLACK")) { const int v = atoi(e); r.claim_slack = v < 0 ? 0 : (v > 2 ? 2 : v); }
        if (const char* e = getenv("SAM_SUPER_TILE")) { const int v = atoi(e); if (v >= 1 && v <= 8) r.super_tile = v; }
        if (const char* e = getenv("SAM_VR")) r.vr = atoi(e);
        if (const char* e = getenv("SAM_COOP")) r.coop = atoi(e) != 0;
        r.no_vec = getenv("SAM_NO_VEC") != nullptr;
        if (const char* e = getenv("SAM_LAG")) r.lag = atoi(e);
        if (const char* e = getenv("SAM_LAND")) r.land = atoi(e) != 0;
        if (const char* e = getenv("SAM_VFOLD")) r.vfold = atoi(e) != 0;
        if (const char* e = getenv("SAM_DYN")) r.dyn = atoi(e) != 0;
        if (const char* e = getenv("SAM_TEAMS")) { const int v = atoi(e); r.teams = (v == 1 || v == 2 || v == 4) ? v : 0; }
        return r;
    }();
    return k;
}
inline const Knobs& knobs() { return knobs_mut(); }

constexpr int MAX_DEVICES = 64;
#ifndef SAM_DEFAULT_DYN
#define SAM_DEFAULT_DYN 0
#endif
#ifndef SAM_DEFAULT_TEAMS
#define SAM_DEFAULT_TEAMS 1
#endif

// Install-time autotune table (SAM's auto-tuner "runs when SAM is installed and determines the
// optimal number of input elements to allocate to each thread for different ranges of problem
// sizes").  Here the per-size-range choice is the carry unit -- tiles per super-tile M,
// i.e. elements per CTA carry step -- and the pipeline depth, per (element type, order, tuple).
// tools/autotune.py measures them on the installed GPU and writes lib/sam_tune.txt, one entry per line:
//     <u32|u64|f32|f64> <k> <s> <log2 n lo> <log2 n hi> <M> <lag> <vfold> <land>
// (M, lag: 0 = built-in default; vfold, land: 0 = default, 1 = off, 2 = on).  Loaded once; the
// environment knobs still win.
struct TuneEntry {
    int w, isf, k, s, lo, hi, M, lag, vfold, land;
};
inline const std::vector<TuneEntry>& tune_table() {
    static const std::vector<TuneEntry> t = [] {
        std::vector<TuneEntry> r;
        std::string path;
        if (const char* e = getenv("SAM_TUNE_FILE")) {
            path = e;
        } else {
            Dl_info di;
            if (dladdr((void*)&tune_table, &di) && di.dli_fname) {
                path = di.dli_fname;
                const size_t slash = path.rfind('/');
                path = (slash == std::string::npos ? std::string(".") : path.substr(0, slash)) + "/sam_tune.txt";
            }
        }
        FILE* f = path.empty() ? nullptr : fopen(path.c_str(), "r");
        if (!f) return r;
        char line[256], ty[8];
        while (fgets(line, sizeof(line), f)) {
            TuneEntry e;
            if (line[0] == '#') continue;
            if (sscanf(line, "%7s %d %d %d %d %d %d %d %d", ty, &e.k, &e.s, &e.lo, &e.hi, &e.M, &e.lag, &e.vfold,
                       &e.land) != 9)
                continue;
            e.w = (ty[1] == '6') ? 8 : 4;
            e.isf = ty[0] == 'f';
            r.push_back(e);
        }
        fclose(f);
        return r;
    }();
    return t;
}
template <typename T>
inline const TuneEntry* tune_lookup(int k, int s, uint64_t n) {
    int lg = 0;
    while (lg < 63 && (1ull << (lg + 1)) <= n) ++lg;
    for (const TuneEntry& e : tune_table())
        if (e.w == (int)sizeof(T) && e.isf == (int)std::is_floating_point<T>::value && e.k == k && e.s == s &&
            lg >= e.lo && lg <= e.hi)
            return &e;
    return nullptr;
}

// Per-device launch facts of one kernel instantiation: the dynamic-shared-memory opt-in
// (cudaFuncSetAttribute is per device context) and the occupancy, set on first use on each device.
template <typename T, int K, bool VEC>
struct KernelInfo {
    int max_blocks_per_sm[MAX_DEVICES] = {};
    bool ready[MAX_DEVICES] = {};
    std::mutex mu;
};

// Host-side tables of a launch shape (the binomial columns b_d(L) of every span the kernel combines
// over: ~300 exact 128-bit evaluations), cached per (device, s, M, P, Vr) so a launch only fills in
// its per-call fields.
struct ShapeKey {
    int dev, s, M, Vr, teams;
    uint64_t P;
    bool operator<(const ShapeKey& o) const {
        if (dev != o.dev) return dev < o.dev;
        if (s != o.s) return s < o.s;
        if (M != o.M) return M < o.M;
        if (Vr != o.Vr) return Vr < o.Vr;
        if (teams != o.teams) return teams < o.teams;
        return P < o.P;
    }
};

// persistent grid: all co-resident CTAs, at most one per super-tile
inline uint64_t grid_of(int blocks_per_sm, int num_sms, uint64_t num_super) {
    uint64_t grid = (uint64_t)blocks_per_sm * (uint64_t)num_sms;
    if (grid > num_super) grid = num_super;
    return grid < 1 ? 1 : grid;
}

// cooperative-grid cap per device (debug: sam_debug_limit_grid; the fallback lowers it when the
// driver refuses a cooperative grid, e.g. under MPS SM limits or in a green context)
inline uint64_t& grid_cap(int dev) {
    static uint64_t cap[MAX_DEVICES] = {};
    return cap[dev];
}
// testing (sam_debug_limit_grid): grids above the limit are treated as refused by the driver, so
// the shrink-and-retry path runs; what it learns is kept apart from grid_cap and reset with the limit
inline uint64_t& debug_grid_limit() {
    static uint64_t lim = 0;
    return lim;
}
inline uint64_t& debug_grid_cap(int dev) {
    static uint64_t cap[MAX_DEVICES] = {};
    return cap[dev];
}
// diagnostics: the shape of the last scan launch on this thread {M, lag, vfold, land, grid, ITEMS}
inline int* last_shape() {
    static thread_local int v[6] = {0, 0, 0, 0, 0, 0};
    return v;
}
inline uint32_t& debug_stress() {
    static uint32_t seed = 0;
    return seed;
}

// O(1) carry ring: R = the power of two >= RING_ROUNDS * grid super-tile records (slot and
// lap by mask and shift).  A slot is rewritten one lap (>= RING_ROUNDS rounds) later; every reader of
// the old record is a fold of one of the
// next P-1 super-tiles, and a CTA cannot run more than 2*LAG/M + 1 <= 25 rounds ahead of another's
// carries (its local scans wait on its own carries, which wait on everyone's aggregates), so 32 rounds
// leave margin; the lap in every word's tag turns a violation into a wait, never a wrong value.
#ifndef SAM_RING_ROUNDS
#define SAM_RING_ROUNDS 32
#endif
constexpr int RING_ROUNDS = SAM_RING_ROUNDS;
// 64-bit words per super-tile record: s*k values of 1 or 2 words, padded to 16 B (bulk copies)
inline unsigned rec_words_of(int w, int k, int s) {
    const unsigned words = (unsigned)(s * k * (w / 4));
    return (words + 1u) & ~1u;
}
inline int ring_log2_of(int ctas) {
    int l = 0;
    while ((1ull << l) < (unsigned long long)ctas * RING_ROUNDS) ++l;
    return l;
}
// bytes of the ring for a grid of `ctas`
inline size_t ring_bytes(int w, int k, int s, int ctas) {
    return ((size_t)1 << ring_log2_of(ctas)) * rec_words_of(w, k, s) * 8;
}

// global-memory pending-state scratch of one launch: [grid][LAG][K][TILE_THREADS] elements
template <typename T, int K>
constexpr size_t pend_bytes_tk(int num_ctas) {
    return Lag<T, K>::GPEND ? (size_t)num_ctas * Lag<T, K>::LAG * K * TILE_THREADS * sizeof(T) : 0;
}
// upper bound over (element size, order) for the workspace: states > 16 B only
inline size_t pend_bytes(int w, int k, int num_ctas) {
    return (SAM_GPEND && w * k > 16) ? (size_t)num_ctas * SAM_LAGG * k * TILE_THREADS * w : 0;
}

template <typename T, int K, bool VEC>
cudaError_t launch_scan_impl(const LaunchArgs& a, uint64_t* launches) {
    using S = Smem<T, K, VEC>;
    using CT = typename Coef<T>::type;
    constexpr int ITEMS = Items<T, VEC>::V;
    constexpr int V = LB<T, K>::V;
    static KernelInfo<T, K, VEC> info;
    static std::map<ShapeKey, Params<T, K>*> tables;  // guarded by info.mu
    const Knobs& kn = knobs();
    const int dev = a.dev;
    if (dev < 0 || dev >= MAX_DEVICES) return cudaErrorInvalidDevice;
    int maxb;
    {
        std::lock_guard<std::mutex> lk(info.mu);
        if (!info.ready[dev]) {
            cudaError_t e = cudaFuncSetAttribute(sam_scan_kernel<T, K, VEC>,
                                                 cudaFuncAttributeMaxDynamicSharedMemorySize, S::BYTES);
            if (e != cudaSuccess) return e;
            int nb = 0;
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sam_scan_kernel<T, K, VEC>, Threads<T, K, VEC>::VALUE, S::BYTES);
            if (e != cudaSuccess) return e;
            info.max_blocks_per_sm[dev] = nb > 0 ? nb : 1;
            info.ready[dev] = true;
        }
        maxb = info.max_blocks_per_sm[dev];
    }
    const Geom geo = make_geom(a.s, ITEMS);
    const uint64_t h = a.g % (uint64_t)a.s;
    // pipeline depth: knob, else the autotune table, else the built-in LAG
    const TuneEntry* te = tune_lookup<T>(K, a.s, a.n);
    const int lag_rt = (kn.lag >= 1 && kn.lag <= S::LAG) ? kn.lag
                       : ((te && te->lag >= 1 && te->lag <= S::LAG) ? te->lag : S::LAG);
    const uint64_t num_tiles = (h + a.n + geo.T - 1) / geo.T;
    // super-tile size: up to MMAX tiles per carry unit, but keep >= 2 super-tiles per SM
    uint64_t M;
    {
        M = num_tiles / (2ull * (uint64_t)(a.num_sms > 0 ? a.num_sms : 148));
        if (M < 1) M = 1;
        // measured: tuple 1: 3 (4-byte) / 2 (8-byte) tiles; tuples (more carry-team work per unit):
        // 3, or 4 for odd tuples of 4-byte elements (~1.5% better there)
        const uint64_t mmax = a.s == 1 ? (uint64_t)Lag<T, K>::MMAX : ((sizeof(T) == 4 && (a.s & 1)) ? 4u : 3u);
        if (M > mmax) M = mmax;
        if (te && te->M > 0) M = (uint64_t)te->M;
        if (kn.super_tile) M = (uint64_t)kn.super_tile;
        // a super-tile is aggregated before its carry is known: at most LAG/2 tiles per unit
        // keep two units in flight per CTA (LAG bounds the tiles between load and carry application)
        const uint64_t mlag = lag_rt / 2 > 1 ? (uint64_t)lag_rt / 2 : 1;
        if (M > mlag) M = mlag;
    }
    const uint64_t num_super = (num_tiles + M - 1) / M;
    // measured: the full register budget per round trip beats spreading window rows over warps
    int Vr = V;
    if (kn.vr >= 1 && kn.vr <= V) Vr = kn.vr;
    // Static schedule (CTA b owns super-tiles b, b+P, ...): every CTA waits on aggregates of the
    // others, so all P CTAs must be co-resident -- a cooperative launch guarantees it or fails; on
    // failure the grid shrinks (the schedule is correct for any P) and the cap is remembered.
    uint64_t P = grid_of(maxb, a.num_sms, num_super);
    for (;;) {
        {
            uint64_t cap = grid_cap(dev);
            const uint64_t dcap = debug_grid_limit() ? debug_grid_cap(dev) : 0;
            if (dcap && (!cap || dcap < cap)) cap = dcap;
            if (cap && P > cap) P = cap;
        }
        // carry teams: one team of 4 warps per super-tile.  Two teams folding successive super-tiles
        // concurrently measured 5-20% slower on every config (profiles/r2_teams_ab.txt) and the team
        // split is not kept as an option.
        const int teams = 1;
        Params<T, K> p;
        {
            std::lock_guard<std::mutex> lk(info.mu);
            const ShapeKey key{dev, a.s, (int)M, Vr, teams, P};
            auto it = tables.find(key);
            if (it == tables.end()) {
                Params<T, K>* t = new Params<T, K>;
                memset(t, 0, sizeof(*t));
                t->s = geo.s; t->G = geo.G; t->logG = geo.logG; t->sp = geo.sp; t->c = geo.c; t->logc = geo.logc;
                t->Pw = geo.Pw; t->W = geo.W; t->Wn = geo.Wn; t->U = geo.U; t->T_ = geo.T; t->Uw = geo.Uw;
                t->M = (int)M;
                t->Vr = Vr;
                t->coop = kn.coop >= 0 ? kn.coop : 1;  // measured faster for every config tried
                const int64_t US = (int64_t)M * geo.U;  // lane length of a super-tile
                mcol<T>(ITEMS, K, t->bc);
                mcol<T>(geo.Uw, K, t->bw);
                mcol<T>(geo.U, K, t->bu);
                mcol<CT>(US, K, t->bus);
                for (int j = 0; j <= NCARRY; ++j) mcol<CT>((int64_t)j * geo.Wn * Vr * US, K, t->bwinj[j]);
                mcol<CT>((int64_t)(P - 1) * US, K, t->bprev);
                mcol<T>((int64_t)teams * P * US, K, t->bposP);  // one team step = `teams` rounds
                mcol<T>(-(int64_t)P * US, K, t->bnegP);
                mcol<CT>((int64_t)geo.Wn * US, K, t->bwn);
                for (int v = 0; v < 32; ++v) {
                    T b[K];
                    mcol<T>((int64_t)v * ITEMS, K, b);
                    for (int d = 0; d < K; ++d) t->bt[d][v] = b[d];
                    mcol<T>(-(int64_t)(v + 1) * ITEMS, K, b);
                    for (int d = 0; d < K; ++d) t->bn[d][v] = b[d];
                }
                for (int q = 0; q < 8; ++q) mcol<T>((int64_t)q * geo.Uw, K, t->bq[q]);
                for (int q = 0; q < 8; ++q) mcol<T>(-(int64_t)q * geo.Uw, K, t->bqn[q]);
                for (int j = 0; j < 32; ++j) mcol<CT>((int64_t)j * US, K, t->bl[j]);
                for (int j = 0; j < 8; ++j) mcol<CT>((int64_t)j * geo.U, K, t->bsub[j]);
                for (int l = 0; l < 5; ++l) mcol<T>((int64_t)(1 << l) * ITEMS, K, t->bks[l]);
                for (int l = 0; l < 3; ++l) mcol<T>((int64_t)(1 << l) * geo.Uw, K, t->bkw[l]);
                it = tables.emplace(key, t).first;
            }
            memcpy(&p, it->second, sizeof(p));
        }
        // per-call fields
        p.in = (const T*)a.in;
        p.out = (T*)a.out;
        p.n = a.n;
        p.h = h;
        p.num_tiles = num_tiles;
        p.num_super = num_super;
        p.delta = (uint32_t)(((uintptr_t)a.in - h * sizeof(T)) & 15);
        p.inclusive = a.inclusive;
        p.store_mode = a.store_mode;
        p.claim_slack = kn.claim_slack;
        p.seed = (const T*)a.seed;
        p.final_state = (T*)a.final_state;
        for (int m = 0; m < MAXS; ++m) {
            p.last_e[m] = -1;
            if (m < a.s && a.n > 0) {
                const int64_t eend = (int64_t)(h + a.n - 1);
                const int64_t le = eend - ((eend - m) % a.s + a.s) % a.s;
                if (le >= (int64_t)h && le >= 0) p.last_e[m] = le;
            }
        }
        p.carry = a.carry;
        p.ring_log2 = ring_log2_of((int)P);
        p.ring = 1ull << p.ring_log2;
        p.rec_words = rec_words_of((int)sizeof(T), K, a.s);
        p.carry_words = p.ring * p.rec_words;
        if (p.carry_words > a.carry_words) return cudaErrorInvalidValue;  // workspace too small for this grid
        p.tile_ctr = a.tile_ctr;
        p.done_ctr = a.done_ctr;
        p.epoch_ptr = a.epoch_ptr;
        p.reset_ctr = a.reset_ctr;
        p.pend = (T*)a.pend;
        const TuneEntry* tl = te;
        p.lag = lag_rt;
        p.teams = teams;
        p.land = kn.land >= 0 ? kn.land : ((tl && tl->land > 0) ? tl->land - 1 : 1);
        // measured (profiles/r2_ab_ring.txt): with the ring the value-parallel fold wins or ties on every
        // config (C2 +7%, int64 k=2 +10%, C5 +16%); the windowed fold stays for floats of order >= 2
        p.vfold = kn.vfold >= 0 ? kn.vfold : ((tl && tl->vfold > 0) ? tl->vfold - 1 : 1);
        p.dyn = kn.dyn >= 0 ? kn.dyn : SAM_DEFAULT_DYN;
        p.trace = a.trace;
        p.stress = debug_stress();

        cudaLaunchConfig_t cfg;
        memset(&cfg, 0, sizeof(cfg));
        cfg.gridDim = dim3((unsigned)P);
        cfg.blockDim = dim3((Threads<T, K, VEC>::GROUPS * geo.W + 2 + Threads<T, K, VEC>::NC) * 32);
        cfg.dynamicSmemBytes = S::BYTES;
        cfg.stream = a.stream;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeCooperative;
        attr[0].val.cooperative = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        const bool simulated = debug_grid_limit() && P > debug_grid_limit();
        cudaError_t e = simulated ? cudaErrorCooperativeLaunchTooLarge : cudaLaunchKernelEx(&cfg, sam_scan_kernel<T, K, VEC>, p);
        if (e == cudaErrorCooperativeLaunchTooLarge && P > 1) {
            if (!simulated) cudaGetLastError();  // clear, retry with a smaller co-resident grid
            P = P - (P + 3) / 4;
            (simulated ? debug_grid_cap(dev) : grid_cap(dev)) = P;
            continue;
        }
        if (e == cudaSuccess) {
            int* ls = last_shape();
            ls[0] = p.M; ls[1] = p.lag; ls[2] = p.vfold; ls[3] = p.land; ls[4] = (int)P; ls[5] = ITEMS;
        }
        if (launches && e == cudaSuccess) ++*launches;
        return e != cudaSuccess ? e : cudaGetLastError();
    }
}

// tuple 1 with a 16-B aligned input: the 128-bit shared-memory variant
template <typename T, int K>
cudaError_t launch_scan_tk(const LaunchArgs& a, uint64_t* launches) {
    const bool vec = a.s == 1 && ((uintptr_t)a.in & 15) == 0 && !knobs().no_vec;
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
cudaError_t launch_cyclic_fold(const void* payloads, size_t payload_bytes, int rank, int nranks, int k, int s,
                               const void* base_in, void* seed_out, void* base_out, cudaStream_t st,
                               uint64_t* launches) {
    sam_cyclic_fold_kernel<T><<<1, 32, 0, st>>>((const unsigned char*)payloads, payload_bytes, rank, nranks, k, s,
                                                (const T*)base_in, (T*)seed_out, (T*)base_out);
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

#include "sam_state.cuh"

#define SAM_INSTANTIATE(T)                                                                             \
    namespace sam {                                                                                    \
    template cudaError_t launch_state<T>(const void*, uint64_t, uint64_t, int, int, void*, void*, size_t, \
                                         unsigned int*, int, cudaStream_t, uint64_t*);                  \
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
    template cudaError_t launch_cyclic_fold<T>(const void*, size_t, int, int, int, int, const void*, void*,   \
                                               void*, cudaStream_t, uint64_t*);                        \
    template cudaError_t launch_payload_init<T>(void*, uint64_t, uint64_t, int, int, const void*, int, \
                                                void*, cudaStream_t, uint64_t*);                       \
    }
