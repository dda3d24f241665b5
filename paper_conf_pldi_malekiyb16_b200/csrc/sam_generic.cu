// sam_generic.cu -- host launch of the generic-operator / selectable-carry scan kernel
// (sam_generic.cuh): instantiations per (element type, operator, order) and the cooperative ->
// look-back fallback of the static schedule.  Called by the C ABI (sam_api.cu).
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <mutex>

#include "sam_generic.cuh"
#include "sam_generic_launch.h"

namespace sam {
namespace gen {

constexpr int MAXDEV = 64;

template <typename T, int OP, int K>
cudaError_t launch_t(const GenArgs& a) {
    using S = GSmem<T, OP, K>;
    static std::mutex mu;
    static bool attr_set[MAXDEV] = {};
    static int occ[MAXDEV][9] = {};
    const size_t smem = S::bytes(a.s);
    {
        std::lock_guard<std::mutex> lk(mu);
        if (!attr_set[a.dev]) {
            size_t mx = 0;
            for (int ss = 1; ss <= 8; ++ss) mx = S::bytes(ss) > mx ? S::bytes(ss) : mx;
            cudaError_t e = cudaFuncSetAttribute(sam_generic_kernel<T, OP, K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                 (int)mx);
            if (e != cudaSuccess) return e;
            attr_set[a.dev] = true;
        }
        if (!occ[a.dev][a.s]) {
            int nb = 0;
            cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sam_generic_kernel<T, OP, K>, TB, smem);
            if (e != cudaSuccess) return e;
            occ[a.dev][a.s] = nb > 0 ? nb : 1;
        }
    }
    GParams<T, K> p;
    memset(&p, 0, sizeof(p));
    p.in = (const T*)a.in;
    p.out = (T*)a.out;
    p.n = a.n;
    const uint64_t TT = (uint64_t)TB * Ips<T>::of(a.s) * a.s;
    p.num_tiles = (a.n + TT - 1) / TT;
    p.s = a.s;
    p.k = a.k;
    p.inclusive = a.inclusive;
    p.words = a.words;
    p.tile_ctr = a.tile_ctr;
    p.done_ctr = a.done_ctr;
    p.epoch_ptr = a.epoch_ptr;
    int mode = a.mode;
    if (mode == GEN_STATIC) {
        uint64_t P = (uint64_t)occ[a.dev][a.s] * (uint64_t)a.num_sms;
        if (P > p.num_tiles) P = p.num_tiles;
        for (;;) {
            p.mode = GEN_STATIC;
            cudaLaunchConfig_t cfg;
            memset(&cfg, 0, sizeof(cfg));
            cfg.gridDim = dim3((unsigned)P);
            cfg.blockDim = dim3(TB);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = a.stream;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeCooperative;
            attr[0].val.cooperative = 1;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            cudaError_t e = cudaLaunchKernelEx(&cfg, sam_generic_kernel<T, OP, K>, p);
            if (e == cudaErrorCooperativeLaunchTooLarge && P > 1) {
                cudaGetLastError();
                P = P - (P + 3) / 4;
                continue;
            }
            if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
                cudaGetLastError();
                mode = GEN_LOOKBACK;  // no co-resident grid at all: the look-back form needs none
                break;
            }
            if (a.mode_used) *a.mode_used = GEN_STATIC;
            return e != cudaSuccess ? e : cudaGetLastError();
        }
    }
    p.mode = mode;
    sam_generic_kernel<T, OP, K><<<(unsigned)p.num_tiles, TB, smem, a.stream>>>(p);
    if (a.mode_used) *a.mode_used = mode;
    return cudaGetLastError();
}

template <typename T, int OP>
cudaError_t launch_k(const GenArgs& a) {
    switch (a.k) {
        case 1: return launch_t<T, OP, 1>(a);
        case 2: return launch_t<T, OP, 2>(a);
        case 3: return launch_t<T, OP, 3>(a);
        case 4: return launch_t<T, OP, 4>(a);
        case 5: return launch_t<T, OP, 5>(a);
        case 6: return launch_t<T, OP, 6>(a);
        case 7: return launch_t<T, OP, 7>(a);
        default: return launch_t<T, OP, 8>(a);
    }
}

// elem: 0 i32, 1 i64, 2 f32, 3 f64, 4 u32, 5 u64 (sam_dtype); op: OP_*
cudaError_t launch_generic(int elem, int op, const GenArgs& a) {
    const bool isf = elem == 2 || elem == 3;
    if (op == OP_ADD) {
        switch (elem) {
            case 0: case 4: return launch_k<uint32_t, OP_ADD>(a);
            case 1: case 5: return launch_k<uint64_t, OP_ADD>(a);
            case 2: return launch_k<float, OP_ADD>(a);
            default: return launch_k<double, OP_ADD>(a);
        }
    }
    if (op == OP_XOR) {
        if (isf) return cudaErrorInvalidValue;
        return (elem == 0 || elem == 4) ? launch_k<uint32_t, OP_XOR>(a) : launch_k<uint64_t, OP_XOR>(a);
    }
    // max / min: order k = order 1 with a k-position exclusive shift (runtime k <= 8)
    if (op == OP_MAX) {
        switch (elem) {
            case 0: return launch_t<int32_t, OP_MAX, 8>(a);
            case 4: return launch_t<uint32_t, OP_MAX, 8>(a);
            case 1: return launch_t<int64_t, OP_MAX, 8>(a);
            case 5: return launch_t<uint64_t, OP_MAX, 8>(a);
            case 2: return launch_t<float, OP_MAX, 8>(a);
            default: return launch_t<double, OP_MAX, 8>(a);
        }
    }
    switch (elem) {
        case 0: return launch_t<int32_t, OP_MIN, 8>(a);
        case 4: return launch_t<uint32_t, OP_MIN, 8>(a);
        case 1: return launch_t<int64_t, OP_MIN, 8>(a);
        case 5: return launch_t<uint64_t, OP_MIN, 8>(a);
        case 2: return launch_t<float, OP_MIN, 8>(a);
        default: return launch_t<double, OP_MIN, 8>(a);
    }
}

// workspace bytes of tagged words for n elements
size_t generic_words_bytes(int elem, int k, int s, uint64_t n) {
    const int w = (elem == 0 || elem == 2 || elem == 4) ? 4 : 8;
    const uint64_t TT = (uint64_t)TB * (w == 4 ? Ips<uint32_t>::of(s) : Ips<uint64_t>::of(s)) * s;
    const uint64_t tiles = (n + TT - 1) / TT + 1;
    return (size_t)tiles * s * 8 /* K <= 8 */ * 2 * (w / 4) * 8;
    (void)k;
}

}  // namespace gen
}  // namespace sam
