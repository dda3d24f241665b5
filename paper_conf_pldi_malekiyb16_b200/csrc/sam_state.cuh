// sam_state.cuh -- the shard state pass (SURVEY §2.2 K*2, §8(e)): a pure reduction.
//
// sam_shard_state needs only the zero-seeded order-k state of every tuple lane at its last element
// of the stream, i.e. per lane m the k-vector  y_t(end) = sum_r C(E_m-1-r + t-1, t-1) x_r  over the
// lane positions r < E_m (P:1187-1197 iterated k times; the weights are the columns of M(L),
// DESIGN.md §2).  Unlike the scan it has no inter-tile carry chain: partial states combine with
// the carry operator in any grouping (M(a)M(b) = M(a+b)), so the pass streams the input once at
// read bandwidth:
//
//   * CTA c owns a contiguous range of tiles (same tile geometry as the scan: a warp holds G
//     lanes, thread <-> (lane m, ITEMS consecutive lane positions), strided smem reads conflict
//     free); tiles arrive by 1-D cp.async.bulk into a ring of 3 smem buffers;
//   * a thread runs the zero-seeded recurrence over its ITEMS positions (k adds per element) and
//     moves its state to the tile's end with the constant column b(U - (u+1) ITEMS) (k(k-1)/2
//     multiplies per thread per tile); the lane's threads sum (shuffles, then smem across warps);
//   * the CTA folds its tiles in order, S <- M(U) S + A_tile, then moves S to the lane's end of
//     the stream, M(E_m - end of range) S, and the last CTA to finish sums the CTAs' parts in
//     CTA order (deterministic for floats; integers are exact mod 2^w in any order).
// Floats accumulate the cross-thread / cross-tile terms in double (Coef<float> = double), with
// non-negative binomial weights only (no M(-L), no cancellation beyond the data's own).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "sam_kernel.cuh"

namespace sam {

template <typename T, int K>
struct StateParams {
    using CT = typename Coef<T>::type;
    const T* in;
    uint64_t n, h;          // elements; virtual index of in[0] (lane phase)
    uint64_t num_tiles;     // ceil((h + n) / T)
    uint64_t tiles_per_cta;
    uint32_t delta;         // byte offset of virtual element 0 inside its 16-B chunk
    int keep;               // L2::evict_last loads (a stream small enough to be re-read from L2)
    int s, G, logG, sp, c, Pw, W, U, T_;
    int64_t E[MAXS];        // per lane: positions up to and including its last element (0: none)
    CT bu[K];               // b(U): one tile
    CT* part;               // [grid][s][K] each CTA's state moved to the lanes' ends
    unsigned int* ticket;   // last-CTA election (reset by the last CTA)
    T* out;                 // [s][K] final state
};

template <typename T, int K>
struct StateSmem {
    using CT = typename Coef<T>::type;
    static constexpr int ITEMS = Cfg<T>::ITEMS;
    static constexpr int NB = 3;
    static constexpr int BUFB = ((TILE_THREADS * ITEMS * (int)sizeof(T) + 32) + 127) / 128 * 128;
    static constexpr int OFF_BAR = NB * BUFB;
    static constexpr int OFF_PART = OFF_BAR + 64;                          // [2][8 warps][8 lanes of a warp][K]
    static constexpr int BYTES = OFF_PART + 2 * 8 * 8 * K * (int)sizeof(CT);
};

template <typename T, int K>
__global__ void __launch_bounds__(TILE_THREADS) sam_state_kernel(const __grid_constant__ StateParams<T, K> p) {
    using CT = typename Coef<T>::type;
    using SM = StateSmem<T, K>;
    constexpr int ITEMS = SM::ITEMS;
    constexpr int NB = SM::NB;
    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* bar = (uint64_t*)(smem + SM::OFF_BAR);
    CT* wpart = (CT*)(smem + SM::OFF_PART);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int s = p.s, G = p.G, Pw = p.Pw, Tt = p.T_;
    const bool active = warp < p.W;
    const int g = warp % p.sp, q = warp / p.sp;
    const int a = lane & (G - 1), v = lane >> p.logG;
    const int m = g * G + a;            // this thread's lane
    const int u = q * Pw + v;           // its block of ITEMS lane positions inside a tile
    const int base_loc = u * ITEMS * s + m;

    const uint64_t t0 = (uint64_t)blockIdx.x * p.tiles_per_cta;
    uint64_t t1 = t0 + p.tiles_per_cta;
    if (t1 > p.num_tiles) t1 = p.num_tiles;

    if (tid == 0) {
        for (int b = 0; b < NB; ++b) mbar_init(&bar[b], 1);
        fence_mbar_init();
    }
    __syncthreads();
    auto issue = [&](uint64_t tile, int b) {  // tile -> buffer b (the scan's aligned-superset copy)
        const uint64_t e0 = tile * (uint64_t)Tt;
        const uint64_t lo = e0 > p.h ? e0 : p.h;
        const uint64_t hi = (e0 + Tt < p.h + p.n) ? e0 + Tt : p.h + p.n;
        const uintptr_t src_lo = (uintptr_t)p.in + (lo - p.h) * sizeof(T);
        const uintptr_t src_hi = (uintptr_t)p.in + (hi - p.h) * sizeof(T);
        const uintptr_t a16 = src_lo & ~(uintptr_t)15;
        const uintptr_t b16 = (src_hi + 15) & ~(uintptr_t)15;
        unsigned char* dst = smem + b * SM::BUFB + p.delta + (lo - e0) * sizeof(T) - (src_lo - a16);
        mbar_arrive_expect_tx(&bar[b], (uint32_t)(b16 - a16));
        bulk_g2s(dst, (const void*)a16, (uint32_t)(b16 - a16), &bar[b], p.keep ? policy_evict_last() : policy_evict_first());
    };
    if (tid == 0) {
        for (uint64_t t = t0; t < t1 && t < t0 + NB - 1; ++t) issue(t, (int)((t - t0) % NB));
    }

    // per-thread constant column of full tiles: b(U - (u+1) ITEMS)
    CT colv[K];
    mcol<CT>((int64_t)p.U - (int64_t)(u + 1) * ITEMS, K, colv);
    CT S[K];  // thread m < s: this CTA's running state of lane m (positions from t0*U)
#pragma unroll
    for (int t = 0; t < K; ++t) S[t] = CT(0);
    const int npl = p.c;  // warps per lane group

    for (uint64_t tile = t0; tile < t1; ++tile) {
        const int it = (int)(tile - t0);
        const int b = it % NB;
        // the previous tile is consumed: its buffer is refilled, its partials (smem, parity it-1)
        // folded by thread m; this tile's partials go to the other parity
        __syncthreads();
        if (tid == 0 && tile + NB - 1 < t1) {
            fence_proxy_async_smem();
            issue(tile + NB - 1, (int)((it + NB - 1) % NB));
        }
        if (it > 0 && tid < s) {
            const CT* wp = wpart + ((it - 1) & 1) * 64 * K;
            const int gm = tid / G, am = tid - gm * G;
            CT A[K];
#pragma unroll
            for (int t = 0; t < K; ++t) A[t] = CT(0);
            for (int qq = 0; qq < npl; ++qq) {
                const int wsrc = qq * p.sp + gm;
#pragma unroll
                for (int t = 0; t < K; ++t) A[t] += wp[(wsrc * 8 + am) * K + t];
            }
            // S <- M(U_m) S + A with U_m the lane's positions in that tile
            const uint64_t tp = tile - 1;
            int64_t Um = p.E[tid] - (int64_t)tp * p.U;
            Um = Um < 0 ? 0 : (Um > p.U ? p.U : Um);
            CT bcol[K];
            if (Um == p.U) {
#pragma unroll
                for (int t = 0; t < K; ++t) bcol[t] = p.bu[t];
            } else {
                mcol<CT>(Um, K, bcol);
            }
            if (Um > 0) {
#pragma unroll
                for (int t = K - 1; t >= 0; --t) {
                    CT acc = S[t] + A[t];
#pragma unroll
                    for (int j = 0; j < t; ++j) acc += bcol[t - j] * S[j];
                    S[t] = acc;
                }
            }
        }
        mbar_wait(&bar[b], (uint32_t)((it / NB) & 1));
        if (active) {
            const T* xs = (const T*)(smem + b * SM::BUFB + p.delta);
            const uint64_t e0 = tile * (uint64_t)Tt;
            const bool full = (e0 >= p.h) && (e0 + Tt <= p.h + p.n);
            T acc[K];
#pragma unroll
            for (int t = 0; t < K; ++t) acc[t] = T(0);
            CT cv[K];
            if (full) {
                T xv[ITEMS];
#pragma unroll
                for (int i = 0; i < ITEMS; ++i) xv[i] = xs[base_loc + i * s];
#pragma unroll
                for (int i = 0; i < ITEMS; ++i) {
                    acc[0] += xv[i];
#pragma unroll
                    for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
                }
#pragma unroll
                for (int t = 0; t < K; ++t) cv[t] = colv[t];
            } else {
                // edge tile: phantom elements before the stream are zeros, positions at or after
                // the lane's end are not stepped over
                int64_t Um = p.E[m] - (int64_t)tile * p.U;
                Um = Um < 0 ? 0 : (Um > p.U ? p.U : Um);
                int cnt = (int)(Um - (int64_t)u * ITEMS);
                cnt = cnt < 0 ? 0 : (cnt > ITEMS ? ITEMS : cnt);
                for (int i = 0; i < cnt; ++i) {
                    const int el = base_loc + i * s;
                    const uint64_t ve = e0 + el;
                    const T x = (ve >= p.h) ? xs[el] : T(0);
                    acc[0] += x;
#pragma unroll
                    for (int t = 1; t < K; ++t) acc[t] += acc[t - 1];
                }
                mcol<CT>(Um - (int64_t)u * ITEMS - cnt, K, cv);  // cnt == 0: acc is 0 anyway
            }
            // move to the tile's end: c = M(cv) acc, then sum over the lane's threads of this warp
            CT cst[K];
#pragma unroll
            for (int t = 0; t < K; ++t) {
                CT r = CT(acc[t]);
#pragma unroll
                for (int j = 0; j < t; ++j) r += cv[t - j] * CT(acc[j]);
                cst[t] = r;
            }
#pragma unroll
            for (int off = 16; off >= 1; off >>= 1) {
                if (off >= G) {
#pragma unroll
                    for (int t = 0; t < K; ++t) cst[t] += __shfl_xor_sync(0xffffffffu, cst[t], off);
                }
            }
            if (v == 0) {
                CT* wp = wpart + (it & 1) * 64 * K + (warp * 8 + a) * K;
#pragma unroll
                for (int t = 0; t < K; ++t) wp[t] = cst[t];
            }
        }
    }
    // the last tile's partials
    __syncthreads();
    const int nt = (int)(t1 > t0 ? t1 - t0 : 0);
    if (tid < s && nt > 0) {
        const CT* wp = wpart + ((nt - 1) & 1) * 64 * K;
        const int gm = tid / G, am = tid - gm * G;
        CT A[K];
#pragma unroll
        for (int t = 0; t < K; ++t) A[t] = CT(0);
        for (int qq = 0; qq < npl; ++qq) {
            const int wsrc = qq * p.sp + gm;
#pragma unroll
            for (int t = 0; t < K; ++t) A[t] += wp[(wsrc * 8 + am) * K + t];
        }
        const uint64_t tp = t1 - 1;
        int64_t Um = p.E[tid] - (int64_t)tp * p.U;
        Um = Um < 0 ? 0 : (Um > p.U ? p.U : Um);
        CT bcol[K];
        mcol<CT>(Um, K, bcol);
        if (Um > 0) {
#pragma unroll
            for (int t = K - 1; t >= 0; --t) {
                CT acc = S[t] + A[t];
#pragma unroll
                for (int j = 0; j < t; ++j) acc += bcol[t - j] * S[j];
                S[t] = acc;
            }
        }
    }
    // this CTA's state, moved over the lane positions after its range: M(E_m - min(t1 U, E_m)) S
    if (tid < s) {
        const int64_t end = (int64_t)t1 * p.U;
        int64_t D = p.E[tid] - end;
        D = D < 0 ? 0 : D;
        CT bcol[K], o[K];
        mcol<CT>(D, K, bcol);
#pragma unroll
        for (int t = 0; t < K; ++t) {
            CT r = S[t];
#pragma unroll
            for (int j = 0; j < t; ++j) r += bcol[t - j] * S[j];
            o[t] = r;
        }
        CT* dst = p.part + ((size_t)blockIdx.x * s + tid) * K;
#pragma unroll
        for (int t = 0; t < K; ++t) dst[t] = o[t];
    }
    // the last CTA sums the parts in CTA order
    __shared__ unsigned int last;
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        last = atomicAdd(p.ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (last) {
        __threadfence();
        if (tid < s) {
            CT acc[K];
#pragma unroll
            for (int t = 0; t < K; ++t) acc[t] = CT(0);
            for (unsigned cc = 0; cc < gridDim.x; ++cc) {
                const volatile CT* src = p.part + ((size_t)cc * s + tid) * K;
#pragma unroll
                for (int t = 0; t < K; ++t) acc[t] += src[t];
            }
#pragma unroll
            for (int t = 0; t < K; ++t) p.out[tid * K + t] = T(acc[t]);
        }
        if (tid == 0) *(volatile unsigned int*)p.ticket = 0u;
    }
}

// host launch: grid = min(tiles, SMs x resident CTAs), contiguous tile ranges per CTA
template <typename T, int K>
cudaError_t launch_state_impl(const T* in, uint64_t n, uint64_t gofs, int s, T* out_state, void* part,
                              size_t part_bytes, unsigned int* ticket, int num_sms, cudaStream_t st,
                              uint64_t* launches) {
    using SM = StateSmem<T, K>;
    using CT = typename Coef<T>::type;
    static int nb_cache[MAX_DEVICES] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= MAX_DEVICES) return cudaErrorInvalidDevice;
    if (!nb_cache[dev]) {
        cudaError_t e = cudaFuncSetAttribute(sam_state_kernel<T, K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             SM::BYTES);
        if (e != cudaSuccess) return e;
        int nb = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sam_state_kernel<T, K>, TILE_THREADS, SM::BYTES);
        if (e != cudaSuccess) return e;
        nb_cache[dev] = nb > 0 ? nb : 1;
    }
    const Geom geo = make_geom(s, Cfg<T>::ITEMS);
    StateParams<T, K> p;
    memset(&p, 0, sizeof(p));
    p.in = in;
    p.n = n;
    p.h = gofs % (uint64_t)s;
    p.s = s; p.G = geo.G; p.logG = geo.logG; p.sp = geo.sp; p.c = geo.c; p.Pw = geo.Pw; p.W = geo.W;
    p.U = geo.U; p.T_ = geo.T;
    p.num_tiles = (p.h + n + geo.T - 1) / geo.T;
    uint64_t grid = (uint64_t)nb_cache[dev] * (uint64_t)(num_sms > 0 ? num_sms : 148);
    if (grid > p.num_tiles) grid = p.num_tiles;
    if (grid < 1) grid = 1;
    p.tiles_per_cta = (p.num_tiles + grid - 1) / grid;
    grid = (p.num_tiles + p.tiles_per_cta - 1) / p.tiles_per_cta;
    if (grid < 1) grid = 1;
    if (grid * (uint64_t)s * K * sizeof(CT) > part_bytes) return cudaErrorInvalidValue;
    p.delta = (uint32_t)(((uintptr_t)in - p.h * sizeof(T)) & 15);
    p.keep = n * sizeof(T) <= ((uint64_t)48 << 20);
    for (int m = 0; m < MAXS; ++m) {
        p.E[m] = 0;
        if (m < s && n > 0) {
            const int64_t eend = (int64_t)(p.h + n - 1);
            const int64_t le = eend - ((eend - m) % s + s) % s;  // virtual index of lane m's last element
            if (le >= (int64_t)p.h && le >= 0) p.E[m] = (le - m) / s + 1;
        }
    }
    mcol<CT>(geo.U, K, p.bu);
    p.part = (CT*)part;
    p.ticket = ticket;
    p.out = out_state;
    sam_state_kernel<T, K><<<(unsigned)grid, TILE_THREADS, SM::BYTES, st>>>(p);
    if (launches) ++*launches;
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_state(const void* in, uint64_t n, uint64_t gofs, int k, int s, void* out_state, void* part,
                         size_t part_bytes, unsigned int* ticket, int num_sms, cudaStream_t st, uint64_t* launches) {
    const T* x = (const T*)in;
    T* o = (T*)out_state;
    switch (k) {
        case 1: return launch_state_impl<T, 1>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 2: return launch_state_impl<T, 2>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 3: return launch_state_impl<T, 3>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 4: return launch_state_impl<T, 4>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 5: return launch_state_impl<T, 5>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 6: return launch_state_impl<T, 6>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        case 7: return launch_state_impl<T, 7>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
        default: return launch_state_impl<T, 8>(x, n, gofs, s, o, part, part_bytes, ticket, num_sms, st, launches);
    }
}

}  // namespace sam
