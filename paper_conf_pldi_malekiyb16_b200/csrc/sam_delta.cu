// sam_delta.cu -- the k-th order, stride-s delta ENCODER: the step before the
// decoder (the scan of sam_kernel.cuh) in the compression pipeline that motivates the paper.
//
//   out[i] = sum_{t=0..k} (-1)^t C(k,t) in[i - t*s]        ("missing" values, i - t*s < 0, are 0)
//
// P:1155-1162 (Sec. 2.4): "There are closed-form solutions for generating higher-order difference
// sequences in a single step and in parallel ... out_k = in_k - 2 in_{k-1} + in_{k-2}"; for s-tuples
// the previous value of a lane is s positions back.  Delta encoding "is embarrassingly
// parallel when not done in place": no carries, one read and one write of HBM.
//
// Kernel: one CTA per tile of TILE elements.  The tile is staged in shared memory with 128-bit
// coalesced loads (evict-first: every element is read from HBM once) behind a halo of the k*s <= 64
// preceding elements (plain loads: the previous tile's bytes, likely still in L2).  Each thread
// then evaluates the stencil for elements j = e*THREADS + tid (conflict-free 32-bit LDS, stride 1
// across a warp) and writes them with coalesced streaming stores; for s = 1 it instead slides a
// register window of 128-bit vectors, and for s > 1 with k*s >= 24 each thread walks one lane of
// a chunk with the lane's last k values in a shift register (k + 1 smem reads per element would
// make high orders bound by shared-memory bandwidth rather than HBM).  Integers: unsigned arithmetic
// mod 2^w (the identity holds in the ring Z/2^w, so the result equals k passes of first-order
// differencing bit for bit); fp32: accumulated in double, rounded once; fp64: accumulated in double.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

namespace sam {
namespace {

constexpr int D_THREADS = 256;
constexpr int D_HALO = 64;  // >= max k*s = 8*8
constexpr int D_LANE_MIN_KS = 24;  // k*s from which s > 1 takes the lane-strided register path
                                   // (SAM_DELTA_LANE_MIN_KS overrides: measurement knob)

template <typename T> struct DeltaAcc { using type = T; };
template <> struct DeltaAcc<float> { using type = double; };

template <typename T> struct DeltaGeom {
    static constexpr int V = 16 / (int)sizeof(T);      // scalars per 128-bit vector
    static constexpr int VPT = 4;                      // vectors per thread
    static constexpr int PER_THREAD = V * VPT;         // 16 (4-byte) / 8 (8-byte)
    static constexpr int TILE = D_THREADS * PER_THREAD;
};

template <typename T> __device__ __forceinline__ T zero_of() { return T(0); }

template <typename T, int K>
__global__ void __launch_bounds__(D_THREADS) delta_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                           uint64_t n, int s, int vec_ok /* bit0 in, bit1 out 16-B aligned */,
                                                           const T* __restrict__ halo, int lane_min_ks) {
    using G = DeltaGeom<T>;
    using A = typename DeltaAcc<T>::type;
    __shared__ __align__(16) T sm[D_HALO + G::TILE];
    const int tid = threadIdx.x;
    const uint64_t b = (uint64_t)blockIdx.x * (uint64_t)G::TILE;
    const uint64_t rem = n - b;
    const int cnt = rem < (uint64_t)G::TILE ? (int)rem : G::TILE;
    const int ks = K * s;

    // (-1)^t C(K,t) by the Pascal recurrence C(K,t) = C(K,t-1) (K-t+1) / t
    A c[K + 1];
    {
        long long m = 1;
#pragma unroll
        for (int t = 0; t <= K; ++t) {
            if (t > 0) m = m * (K - t + 1) / t;
            c[t] = (t & 1) ? (A)(0 - (A)m) : (A)m;
        }
    }

    if (tid < ks) {
        const uint64_t q = (uint64_t)tid + 1;
        // before in[0]: the caller's halo (halo[ks-1] adjacent to in[0]) or "missing" = 0
        sm[D_HALO - (int)q] = (b >= q) ? in[b - q] : (halo ? halo[ks - (int)(q - b)] : zero_of<T>());
    }
    if ((vec_ok & 1) && cnt == G::TILE) {
        const int4* src = reinterpret_cast<const int4*>(in + b);
        int4* dst = reinterpret_cast<int4*>(sm + D_HALO);
        int4 v[G::VPT];
#pragma unroll
        for (int u = 0; u < G::VPT; ++u) v[u] = __ldcs(src + u * D_THREADS + tid);
#pragma unroll
        for (int u = 0; u < G::VPT; ++u) dst[u * D_THREADS + tid] = v[u];
    } else {
        for (int j = tid; j < cnt; j += D_THREADS) sm[D_HALO + j] = __ldcs(in + b + j);
    }
    __syncthreads();

    if (s == 1 && (vec_ok & 2) && cnt == G::TILE) {
        // s = 1, full tile: thread tid owns the 128-bit vectors u*THREADS + tid and reads each one
        // with the NH vectors before it (LDS.128, consecutive threads on consecutive vectors:
        // conflict free) into a register window; the stencil then runs on registers, so shared
        // memory carries (NH + 1) * 16 B per V outputs instead of (K + 1) * w per output.
        constexpr int V = G::V;
        constexpr int NH = (K + V - 1) / V;  // <= D_HALO / V, so the window stays inside sm
        const int4* sv = reinterpret_cast<const int4*>(sm + D_HALO);
        int4* ov = reinterpret_cast<int4*>(out + b);
#pragma unroll
        for (int u = 0; u < G::VPT; ++u) {
            const int vi = u * D_THREADS + tid;
            T win[(NH + 1) * V];
#pragma unroll
            for (int h = 0; h <= NH; ++h) {
                const int4 q = sv[vi - NH + h];
                const T* qt = reinterpret_cast<const T*>(&q);
#pragma unroll
                for (int e = 0; e < V; ++e) win[h * V + e] = qt[e];
            }
            T r[V];
#pragma unroll
            for (int e = 0; e < V; ++e) {
                A acc = (A)win[NH * V + e];
#pragma unroll
                for (int t = 1; t <= K; ++t) acc = acc + c[t] * (A)win[NH * V + e - t];
                r[e] = (T)acc;
            }
            __stcs(ov + vi, *reinterpret_cast<const int4*>(r));
        }
        return;
    }

    if (s > 1 && ks >= lane_min_ks) {
        // large k*s: lane-strided register path.  Unit u = (chunk c, lane m) owns the R positions
        // c*s*R + m + i*s (i < R) of one lane and keeps the K previous values of that lane in a
        // shift register, so a unit reads R + K smem values for R outputs instead of (K + 1) * R.
        // R odd (17 / 9) keeps the warp's reads on distinct banks for even s, and
        // ceil(TILE / (s R)) * s <= 248 (4-byte) / 232 (8-byte) units for every s <= 8: one unit
        // per thread covers the tile.
        constexpr int R = sizeof(T) == 4 ? 17 : 9;
        const int span = s * R;
        const int nunits = ((cnt + span - 1) / span) * s;  // <= D_THREADS (see above)
        const int u = tid;
        const int cc = u / s;
        const int p0 = cc * span + (u - cc * s);
        // A unit's only reads of other units' values are its K history values (the previous chunk
        // of its lane): take them, then after one barrier each unit owns its R positions alone and
        // overwrites them in place with its outputs, which then leave through coalesced 128-bit
        // stores (a warp's direct stores would be s-element groups at stride s*R: partial sectors).
        A h[K];  // h[t-1] = x[p - t*s]
        if (u < nunits) {
#pragma unroll
            for (int t = 1; t <= K; ++t) h[t - 1] = (A)sm[D_HALO + p0 - t * s];
        }
        __syncthreads();
        if (u < nunits) {
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const int p = p0 + i * s;
                if (p < cnt) {
                    const A xv = (A)sm[D_HALO + p];
                    A acc = xv;
#pragma unroll
                    for (int t = 1; t <= K; ++t) acc = acc + c[t] * h[t - 1];
                    sm[D_HALO + p] = (T)acc;
#pragma unroll
                    for (int t = K - 1; t > 0; --t) h[t] = h[t - 1];
                    h[0] = xv;
                }
            }
        }
        __syncthreads();
        if ((vec_ok & 2) && cnt == G::TILE) {
            const int4* src = reinterpret_cast<const int4*>(sm + D_HALO);
            int4* dst = reinterpret_cast<int4*>(out + b);
#pragma unroll
            for (int v = 0; v < G::VPT; ++v) __stcs(dst + v * D_THREADS + tid, src[v * D_THREADS + tid]);
        } else {
            for (int j = tid; j < cnt; j += D_THREADS) __stcs(out + b + j, sm[D_HALO + j]);
        }
        return;
    }

#pragma unroll 4
    for (int e = 0; e < G::PER_THREAD; ++e) {
        const int j = e * D_THREADS + tid;
        if (j < cnt) {
            const T* p = sm + D_HALO + j;
            A acc = (A)p[0];
#pragma unroll
            for (int t = 1; t <= K; ++t) acc = acc + c[t] * (A)p[-t * s];
            __stcs(out + b + j, (T)acc);
        }
    }
}

int lane_min_ks() {
    static const int v = [] {
        const char* e = getenv("SAM_DELTA_LANE_MIN_KS");
        return e ? atoi(e) : D_LANE_MIN_KS;
    }();
    return v;
}

template <typename T, int K>
cudaError_t launch_k(const T* in, T* out, uint64_t n, int s, const T* halo, cudaStream_t st) {
    using G = DeltaGeom<T>;
    const uint64_t tiles = (n + G::TILE - 1) / G::TILE;
    const int vec_ok = (((uintptr_t)in % 16) == 0 ? 1 : 0) | (((uintptr_t)out % 16) == 0 ? 2 : 0);
    delta_kernel<T, K><<<(unsigned)tiles, D_THREADS, 0, st>>>(in, out, n, s, vec_ok, halo, lane_min_ks());
    return cudaGetLastError();
}

}  // namespace

// One launch of the delta encoder (halo: NULL or k*s elements preceding in[0]; n > 0, 1 <= k, s <= 8, in/out non-overlapping, validated by
// the caller).  *launches is incremented by the number of kernels launched.
template <typename T>
cudaError_t launch_delta(const void* in_, void* out_, uint64_t n, int k, int s, const void* halo_,
                         cudaStream_t st, uint64_t* launches) {
    const T* halo = (const T*)halo_;
    const T* in = (const T*)in_;
    T* out = (T*)out_;
    if (n == 0) return cudaSuccess;
    if ((n + DeltaGeom<T>::TILE - 1) / DeltaGeom<T>::TILE > 0x7fffffffull) return cudaErrorInvalidValue;
    cudaError_t e = cudaErrorInvalidValue;
    switch (k) {
        case 1: e = launch_k<T, 1>(in, out, n, s, halo, st); break;
        case 2: e = launch_k<T, 2>(in, out, n, s, halo, st); break;
        case 3: e = launch_k<T, 3>(in, out, n, s, halo, st); break;
        case 4: e = launch_k<T, 4>(in, out, n, s, halo, st); break;
        case 5: e = launch_k<T, 5>(in, out, n, s, halo, st); break;
        case 6: e = launch_k<T, 6>(in, out, n, s, halo, st); break;
        case 7: e = launch_k<T, 7>(in, out, n, s, halo, st); break;
        case 8: e = launch_k<T, 8>(in, out, n, s, halo, st); break;
    }
    if (e == cudaSuccess) *launches += 1;
    return e;
}

template cudaError_t launch_delta<uint32_t>(const void*, void*, uint64_t, int, int, const void*, cudaStream_t, uint64_t*);
template cudaError_t launch_delta<uint64_t>(const void*, void*, uint64_t, int, int, const void*, cudaStream_t, uint64_t*);
template cudaError_t launch_delta<float>(const void*, void*, uint64_t, int, int, const void*, cudaStream_t, uint64_t*);
template cudaError_t launch_delta<double>(const void*, void*, uint64_t, int, int, const void*, cudaStream_t, uint64_t*);

}  // namespace sam
