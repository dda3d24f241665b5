// sam_api.cu -- the C ABI of libsam.so (include/sam.h): argument validation, per-(device,
// stream) workspaces, dispatch over (element type, order), the sharded entry points and the
// host-buffer streaming pipeline.  Every arithmetic step of the scan runs in the CUDA kernels
// of sam_kernel.cuh; this file only validates, allocates and launches.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <atomic>
#include <map>
#include <mutex>
#include <string>
#include <utility>

#include "sam.h"
#include "sam_generic_launch.h"
#include "sam_launch.cuh"

namespace sam {
template <typename T, int K> cudaError_t launch_scan_tk(const LaunchArgs&, uint64_t*);
template <typename T> cudaError_t launch_delta(const void*, void*, uint64_t, int, int, const void*, cudaStream_t, uint64_t*);
template <typename T> cudaError_t launch_fold(const void*, size_t, int, int, int, void*, cudaStream_t, uint64_t*);
template <typename T> cudaError_t launch_payload_init(void*, uint64_t, uint64_t, int, int, const void*, int, void*,
                                                      cudaStream_t, uint64_t*);
}  // namespace sam

namespace {

thread_local std::string g_err;
thread_local int g_last_carry = -1;  // carry scheme the last generic launch on this thread ran
std::atomic<uint64_t> g_launches{0};
constexpr const char* kVersion = "sam-b200 0.2 (sm_100a, single-pass, SAM static carry schedule on a cooperative persistent grid, order 1-8, tuple 1-8)";

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}
int cuda_fail(cudaError_t e, const char* where) {
    g_err = std::string(where) + ": " + cudaGetErrorString(e);
    return SAM_ERR_CUDA;
}

size_t elem_size(sam_dtype d) { return (d == SAM_I32 || d == SAM_F32 || d == SAM_U32) ? 4 : 8; }

// SAM_U32 / SAM_U64 are the same bits as SAM_I32 / SAM_I64 for addition (wraparound)
sam_dtype add_dtype(sam_dtype d) { return d == SAM_U32 ? SAM_I32 : (d == SAM_U64 ? SAM_I64 : d); }

int validate_common(sam_dtype dtype, int order, int tuple) {
    if ((int)dtype < 0 || (int)dtype > 5) return fail(SAM_ERR_UNSUPPORTED, "unknown dtype");
    if (order < 1 || order > 8) return fail(SAM_ERR_UNSUPPORTED, "order must be in 1..8 (DESIGN.md R4)");
    if (tuple < 1 || tuple > 8) return fail(SAM_ERR_UNSUPPORTED, "tuple must be in 1..8 (DESIGN.md R4)");
    return SAM_OK;
}

int validate_buffers(sam_dtype dtype, const void* in, const void* out, uint64_t n, bool need_out) {
    if (n == 0) return SAM_OK;
    const size_t w = elem_size(dtype);
    if (!in || (need_out && !out)) return fail(SAM_ERR_INVALID_ARG, "null buffer with n > 0");
    if (((uintptr_t)in % w) != 0 || (need_out && ((uintptr_t)out % w) != 0))
        return fail(SAM_ERR_INVALID_ARG, "buffers must be aligned to the element size");
    if (n > (UINT64_MAX / 16)) return fail(SAM_ERR_INVALID_ARG, "n too large");
    if (need_out && in != out) {
        const uintptr_t a0 = (uintptr_t)in, a1 = a0 + n * w, b0 = (uintptr_t)out, b1 = b0 + n * w;
        if (a0 < b1 && b0 < a1) return fail(SAM_ERR_INVALID_ARG, "in and out partially overlap (only in == out is allowed)");
    }
    return SAM_OK;
}

struct Workspace {
    unsigned long long* carry = nullptr;  // tagged carry words of every tile
    size_t carry_cap = 0;                 // bytes
    unsigned char* pend = nullptr;        // pending-state scratch (states > 16 B)
    size_t pend_cap = 0;
    unsigned char* ctr = nullptr;  // [tile_ctr u64][done u32][epoch u32][reset u32][state ticket u32][pad][seed 512 B]
    unsigned char* part = nullptr; // state pass: per-CTA parts [grid][s][k] (fixed size, PART_BYTES)
};
constexpr size_t PART_BYTES = (size_t)2048 * 64 * 8;  // up to 2048 CTAs x 64 values x 8 B

std::mutex g_mu;
std::map<std::pair<int, cudaStream_t>, Workspace*> g_ws;
std::map<int, int> g_sms;
unsigned long long* g_trace = nullptr;  // diagnostics: per-tile event timestamps of the next launches

// First use of a device: SM count, and an L2 persisting set-aside so the kernel's L2::evict_last
// hints (tiles parked in L2 between local scan and carry application) are honoured.  Only raised,
// never lowered; SAM_L2_PERSIST_MB=0 disables it.
int num_sms(int dev) {
    auto it = g_sms.find(dev);
    if (it != g_sms.end()) return it->second;
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    g_sms[dev] = n;
    int maxp = 0;
    size_t cur = 0;
    long want_mb = 0;  // measured: a set-aside starves the streaming traffic; opt in only
    if (const char* env = getenv("SAM_L2_PERSIST_MB")) want_mb = atol(env);
    if (want_mb > 0 && cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev) == cudaSuccess &&
        maxp > 0 && cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) == cudaSuccess) {
        size_t want = (size_t)want_mb << 20;
        if (want > (size_t)maxp) want = (size_t)maxp;
        if (cur < want) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want);
    }
    cudaGetLastError();  // the set-aside is an optimisation; never fail a scan over it
    return n;
}

// Workspace header (device memory): [u64 tile_ctr][u32 done][u32 epoch][u32 reset][pad .. 32]
// [512 B seed scratch of sam_shard_scan][pad .. 1024], then the tagged carry words.
constexpr size_t CTR_BYTES = 32 + 8 * 8 * 8;
constexpr size_t WS_HEADER = 1024;

// workspace of (current device, stream) with room for `carry_bytes` of tagged carry words and
// `pend_bytes` of pending-state scratch
int get_ws(cudaStream_t st, size_t carry_bytes, Workspace** out, int* dev_out, size_t pend_bytes = 0) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    std::lock_guard<std::mutex> lk(g_mu);
    Workspace*& ws = g_ws[std::make_pair(dev, st)];
    if (!ws) ws = new Workspace();
    if (!ws->ctr) {
        e = cudaMalloc(&ws->ctr, CTR_BYTES);
        if (e != cudaSuccess) return fail(SAM_ERR_OOM, std::string("workspace: ") + cudaGetErrorString(e));
        e = cudaMemsetAsync(ws->ctr, 0, CTR_BYTES, st);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync");
    }
    if (carry_bytes > ws->carry_cap) {
        // grow (never shrink); the old buffer may still be read by queued kernels on this stream
        // (graph capture / concurrent streams: use sam_scan_ws with a caller-owned workspace)
        e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
        const size_t cap = carry_bytes + carry_bytes / 4 + 4096;
        if (ws->carry) cudaFree(ws->carry);
        ws->carry = nullptr;
        ws->carry_cap = 0;
        e = cudaMalloc(&ws->carry, cap);
        if (e != cudaSuccess) return fail(SAM_ERR_OOM, std::string("workspace: ") + cudaGetErrorString(e));
        // zero words carry tag 0, which no launch uses
        e = cudaMemsetAsync(ws->carry, 0, cap, st);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync");
        ws->carry_cap = cap;
    }
    if (pend_bytes > ws->pend_cap) {
        e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
        if (ws->pend) cudaFree(ws->pend);
        ws->pend = nullptr;
        ws->pend_cap = 0;
        e = cudaMalloc(&ws->pend, pend_bytes);
        if (e != cudaSuccess) return fail(SAM_ERR_OOM, std::string("workspace: ") + cudaGetErrorString(e));
        ws->pend_cap = pend_bytes;
    }
    *out = ws;
    *dev_out = dev;
    return SAM_OK;
}

int num_sms_of(int dev) {
    std::lock_guard<std::mutex> lk(g_mu);
    return num_sms(dev);
}

// bytes of pending-state scratch a workspace holds (multiple of 256, placed after the header)
size_t pend_area(sam_dtype d, int k, int dev) {
    return (sam::pend_bytes((int)elem_size(d), k, num_sms_of(dev)) + 255) / 256 * 256;
}

int items_of(sam_dtype d) {
    switch (add_dtype(d)) {
        case SAM_I32: return sam::Cfg<uint32_t>::ITEMS;
        case SAM_I64: return sam::Cfg<uint64_t>::ITEMS;
        case SAM_F32: return sam::Cfg<float>::ITEMS;
        default: return sam::Cfg<double>::ITEMS;
    }
}

// bytes of the O(1) carry ring (sam_launch.cuh): RING_ROUNDS records per CTA of the largest grid of
// the current device, whatever n is (`tiles` is no longer needed)
size_t carry_bytes(sam_dtype d, int k, int s, size_t tiles) {
    (void)tiles;
    int dev = 0;
    cudaGetDevice(&dev);
    return sam::ring_bytes((int)elem_size(d), k, s, num_sms_of(dev));
}
// the largest ring of any (dtype, order, tuple): the generic kernel's words go after it
size_t ring_max_bytes() {
    int dev = 0;
    cudaGetDevice(&dev);
    return sam::ring_bytes(8, 8, 8, num_sms_of(dev));
}
size_t tiles_for(sam_dtype dtype, int s, uint64_t n) {
    const sam::Geom geo = sam::make_geom(s, items_of(dtype));
    return (size_t)((n + (uint64_t)s + geo.T - 1) / geo.T);
}

template <typename T>
cudaError_t dispatch_k(int k, const sam::LaunchArgs& a) {
    uint64_t l = 0;
    cudaError_t e = cudaErrorInvalidValue;
    switch (k) {
        case 1: e = sam::launch_scan_tk<T, 1>(a, &l); break;
        case 2: e = sam::launch_scan_tk<T, 2>(a, &l); break;
        case 3: e = sam::launch_scan_tk<T, 3>(a, &l); break;
        case 4: e = sam::launch_scan_tk<T, 4>(a, &l); break;
        case 5: e = sam::launch_scan_tk<T, 5>(a, &l); break;
        case 6: e = sam::launch_scan_tk<T, 6>(a, &l); break;
        case 7: e = sam::launch_scan_tk<T, 7>(a, &l); break;
        case 8: e = sam::launch_scan_tk<T, 8>(a, &l); break;
    }
    g_launches += l;
    return e;
}

// one scan-kernel launch for a stream of n elements at global offset g.  ws_hdr / carry / carry_cap:
// an explicit workspace (sam_scan_ws), or null for the cached (device, stream) workspace.
int run_scan(sam_dtype dtype, int k, int s, int inclusive, const void* in, void* out, uint64_t n, uint64_t g,
             const void* seed, void* final_state, int store_mode, cudaStream_t st,
             unsigned char* ws_hdr = nullptr, unsigned long long* ws_carry = nullptr, size_t ws_carry_cap = 0,
             void* ws_pend = nullptr) {
    int dev = 0;
    if (!ws_hdr) {
        Workspace* ws = nullptr;
        int d0 = 0;
        cudaGetDevice(&d0);
        int rc = get_ws(st, carry_bytes(dtype, k, s, tiles_for(dtype, s, n + g % (uint64_t)s)), &ws, &dev,
                        sam::pend_bytes((int)elem_size(dtype), k, num_sms_of(d0)));
        if (rc != SAM_OK) return rc;
        ws_hdr = ws->ctr;
        ws_carry = ws->carry;
        ws_carry_cap = ws->carry_cap;
        ws_pend = ws->pend;
    } else {
        cudaError_t e = cudaGetDevice(&dev);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    }
    sam::LaunchArgs a;
    a.in = in;
    a.out = out;
    a.n = n;
    a.g = g;
    a.seed = seed;
    a.final_state = final_state;
    a.s = s;
    a.inclusive = inclusive ? 1 : 0;
    a.store_mode = store_mode;
    a.stream = st;
    a.carry = ws_carry;
    a.carry_words = ws_carry_cap / 8;
    a.tile_ctr = (unsigned long long*)(ws_hdr);
    a.done_ctr = (unsigned int*)(ws_hdr + 8);
    a.epoch_ptr = (unsigned int*)(ws_hdr + 12);
    a.reset_ctr = (unsigned int*)(ws_hdr + 16);
    a.pend = ws_pend;
    a.num_sms = num_sms(dev);
    a.dev = dev;
    a.trace = g_trace;
    cudaError_t e;
    switch (add_dtype(dtype)) {
        case SAM_I32: e = dispatch_k<uint32_t>(k, a); break;
        case SAM_I64: e = dispatch_k<uint64_t>(k, a); break;
        case SAM_F32: e = dispatch_k<float>(k, a); break;
        default: e = dispatch_k<double>(k, a); break;
    }
    if (e != cudaSuccess) return cuda_fail(e, "scan kernel launch");
    return SAM_OK;
}

int payload_init(sam_dtype dtype, void* payload, uint64_t n, uint64_t g, int k, int s, const void* seed,
                 int write_header, void* final_state, cudaStream_t st) {
    uint64_t l = 0;
    cudaError_t e;
    switch (dtype) {
        case SAM_I32: e = sam::launch_payload_init<uint32_t>(payload, n, g, k, s, seed, write_header, final_state, st, &l); break;
        case SAM_I64: e = sam::launch_payload_init<uint64_t>(payload, n, g, k, s, seed, write_header, final_state, st, &l); break;
        case SAM_F32: e = sam::launch_payload_init<float>(payload, n, g, k, s, seed, write_header, final_state, st, &l); break;
        default: e = sam::launch_payload_init<double>(payload, n, g, k, s, seed, write_header, final_state, st, &l); break;
    }
    g_launches += l;
    return e == cudaSuccess ? SAM_OK : cuda_fail(e, "payload init launch");
}

template <typename T>
void cyclic_fold_host_t(const unsigned char* P, size_t pb, int rank, int nranks, int k, int s, const T* base_in,
                        T* seed_out, T* base_out) {
    for (int m = 0; m < s; ++m) {
        T sd[sam::MAXK];
        sam::fold_payloads_from<T>(base_in ? base_in + m * k : nullptr, P, pb, rank, k, s, m, sd);
        if (base_out) sam::fold_payloads_from<T>(sd, P + (size_t)rank * pb, pb, nranks - rank, k, s, m, base_out + m * k);
        for (int t = 0; t < k; ++t) seed_out[m * k + t] = sd[t];
    }
}
// block-cyclic fold on host buffers (sam_cyclic_fold_host)
// SAM_STATE_VIA_SCAN=1 (read once): sam_shard_state runs the scan kernel in state-only mode (A/B)
bool state_via_scan() {
    static const bool v = getenv("SAM_STATE_VIA_SCAN") != nullptr && atoi(getenv("SAM_STATE_VIA_SCAN")) != 0;
    return v;
}

int store_mode_for(const void* in, const void* out) {
    return ((((uintptr_t)in) ^ ((uintptr_t)out)) & 15) == 0 ? sam::STORE_BULK : sam::STORE_STRIPED;
}

}  // namespace

extern "C" {

int sam_scan(sam_dtype dtype, int order, int tuple, int inclusive, const void* in, void* out, uint64_t n,
             sam_stream_t stream) {
    return sam_scan_seeded(dtype, order, tuple, inclusive, in, out, n, 0, nullptr, nullptr, stream);
}

int sam_scan_seeded(sam_dtype dtype, int order, int tuple, int inclusive, const void* in, void* out, uint64_t n,
                    uint64_t global_offset, const void* seed, void* final_state, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    rc = validate_buffers(dtype, in, out, n, true);
    if (rc) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (final_state) {
        rc = payload_init(dtype, nullptr, n, global_offset, order, tuple, seed, 0, final_state, st);
        if (rc) return rc;
    }
    if (n == 0) return SAM_OK;
    return run_scan(dtype, order, tuple, inclusive, in, out, n, global_offset, seed, final_state,
                    store_mode_for(in, out), st);
}

int sam_prepare(sam_dtype dtype, int order, int tuple, uint64_t max_n, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    Workspace* ws = nullptr;
    int dev = 0;
    return get_ws((cudaStream_t)stream, carry_bytes(dtype, order, tuple, tiles_for(dtype, tuple, max_n)), &ws, &dev);
}

int sam_scan_workspace_size(sam_dtype dtype, int order, int tuple, uint64_t n, size_t* bytes) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (!bytes) return fail(SAM_ERR_INVALID_ARG, "null bytes pointer");
    int dev = 0;
    cudaGetDevice(&dev);
    *bytes = WS_HEADER + pend_area(dtype, order, dev) + carry_bytes(dtype, order, tuple, tiles_for(dtype, tuple, n));
    return SAM_OK;
}

int sam_scan_ws(sam_dtype dtype, int order, int tuple, int inclusive, const void* in, void* out, uint64_t n,
                void* ws, size_t ws_bytes, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    rc = validate_buffers(dtype, in, out, n, true);
    if (rc) return rc;
    if (n == 0) return SAM_OK;
    size_t need = 0;
    sam_scan_workspace_size(dtype, order, tuple, n, &need);
    if (!ws) return fail(SAM_ERR_INVALID_ARG, "null workspace");
    if (((uintptr_t)ws & 15) != 0) return fail(SAM_ERR_INVALID_ARG, "workspace must be 16-B aligned");
    if (ws_bytes < need)
        return fail(SAM_ERR_INVALID_ARG, "workspace too small (sam_scan_workspace_size gives " + std::to_string(need) + " B)");
    unsigned char* w = (unsigned char*)ws;
    int dev = 0;
    cudaGetDevice(&dev);
    const size_t pa = pend_area(dtype, order, dev);
    return run_scan(dtype, order, tuple, inclusive, in, out, n, 0, nullptr, nullptr, store_mode_for(in, out),
                    (cudaStream_t)stream, w, (unsigned long long*)(w + WS_HEADER + pa), ws_bytes - WS_HEADER - pa,
                    pa ? (void*)(w + WS_HEADER) : nullptr);
}

size_t sam_shard_payload_bytes(sam_dtype dtype, int order, int tuple) {
    if (validate_common(dtype, order, tuple)) return 0;
    // header + values, rounded to 16 B so every rank's payload in the gathered buffer is aligned
    return (16 + (size_t)order * (size_t)tuple * elem_size(dtype) + 15) / 16 * 16;
}

int sam_shard_state(sam_dtype dtype, int order, int tuple, const void* in_local, uint64_t n_local,
                    uint64_t global_offset, void* payload_dev, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    rc = validate_buffers(dtype, in_local, nullptr, n_local, false);
    if (rc) return rc;
    if (!payload_dev) return fail(SAM_ERR_INVALID_ARG, "null payload");
    cudaStream_t st = (cudaStream_t)stream;
    void* fs = (unsigned char*)payload_dev + 16;
    rc = payload_init(dtype, payload_dev, n_local, global_offset, order, tuple, nullptr, 1, fs, st);
    if (rc || n_local == 0) return rc;
    if (state_via_scan())  // A/B: the scan kernel in state-only mode (round 1-2 path)
        return run_scan(dtype, order, tuple, 1, in_local, nullptr, n_local, global_offset, nullptr, fs,
                        sam::STORE_NONE, st);
    // the dedicated reduction kernel (sam_state.cuh): one read of the shard, no carry chain
    Workspace* ws = nullptr;
    int dev = 0;
    rc = get_ws(st, 0, &ws, &dev);
    if (rc) return rc;
    if (!ws->part) {
        cudaError_t e = cudaMalloc(&ws->part, PART_BYTES);
        if (e != cudaSuccess) return fail(SAM_ERR_OOM, std::string("workspace: ") + cudaGetErrorString(e));
    }
    unsigned int* ticket = (unsigned int*)(ws->ctr + 20);
    uint64_t l = 0;
    cudaError_t e;
    const int sms = num_sms_of(dev);
    switch (add_dtype(dtype)) {
        case SAM_I32: e = sam::launch_state<uint32_t>(in_local, n_local, global_offset, order, tuple, fs, ws->part, PART_BYTES, ticket, sms, st, &l); break;
        case SAM_I64: e = sam::launch_state<uint64_t>(in_local, n_local, global_offset, order, tuple, fs, ws->part, PART_BYTES, ticket, sms, st, &l); break;
        case SAM_F32: e = sam::launch_state<float>(in_local, n_local, global_offset, order, tuple, fs, ws->part, PART_BYTES, ticket, sms, st, &l); break;
        default: e = sam::launch_state<double>(in_local, n_local, global_offset, order, tuple, fs, ws->part, PART_BYTES, ticket, sms, st, &l); break;
    }
    g_launches += l;
    return e == cudaSuccess ? SAM_OK : cuda_fail(e, "state kernel launch");
}

int sam_shard_scan(sam_dtype dtype, int order, int tuple, int inclusive, const void* in_local, void* out_local,
                   uint64_t n_local, uint64_t global_offset, const void* all_payloads_dev, int rank, int nranks,
                   sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAM_ERR_INVALID_ARG, "rank/nranks out of range");
    if (rank > 0 && !all_payloads_dev) return fail(SAM_ERR_INVALID_ARG, "null payloads");
    rc = validate_buffers(dtype, in_local, out_local, n_local, true);
    if (rc) return rc;
    if (n_local == 0) return SAM_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const void* seed = nullptr;
    if (rank > 0) {
        Workspace* ws = nullptr;
        int dev = 0;
        rc = get_ws(st, 0, &ws, &dev);
        if (rc) return rc;
        void* seedbuf = ws->ctr + 32;
        const size_t pb = sam_shard_payload_bytes(dtype, order, tuple);
        uint64_t l = 0;
        cudaError_t e;
        switch (dtype) {
            case SAM_I32: e = sam::launch_fold<uint32_t>(all_payloads_dev, pb, rank, order, tuple, seedbuf, st, &l); break;
            case SAM_I64: e = sam::launch_fold<uint64_t>(all_payloads_dev, pb, rank, order, tuple, seedbuf, st, &l); break;
            case SAM_F32: e = sam::launch_fold<float>(all_payloads_dev, pb, rank, order, tuple, seedbuf, st, &l); break;
            default: e = sam::launch_fold<double>(all_payloads_dev, pb, rank, order, tuple, seedbuf, st, &l); break;
        }
        g_launches += l;
        if (e != cudaSuccess) return cuda_fail(e, "fold launch");
        seed = seedbuf;
    }
    return run_scan(dtype, order, tuple, inclusive, in_local, out_local, n_local, global_offset, seed, nullptr,
                    store_mode_for(in_local, out_local), st);
}

int sam_fold_payloads_host(sam_dtype dtype, int order, int tuple, const void* all_payloads_host, int rank,
                           int nranks, void* seed_host) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAM_ERR_INVALID_ARG, "rank/nranks out of range");
    if (!seed_host || (rank > 0 && !all_payloads_host)) return fail(SAM_ERR_INVALID_ARG, "null buffer");
    const size_t pb = sam_shard_payload_bytes(dtype, order, tuple);
    const unsigned char* P = (const unsigned char*)all_payloads_host;
    for (int m = 0; m < tuple; ++m) {
        switch (dtype) {
            case SAM_I32: sam::fold_payloads<uint32_t>(P, pb, rank, order, tuple, m, (uint32_t*)seed_host + m * order); break;
            case SAM_I64: sam::fold_payloads<uint64_t>(P, pb, rank, order, tuple, m, (uint64_t*)seed_host + m * order); break;
            case SAM_F32: sam::fold_payloads<float>(P, pb, rank, order, tuple, m, (float*)seed_host + m * order); break;
            default: sam::fold_payloads<double>(P, pb, rank, order, tuple, m, (double*)seed_host + m * order); break;
        }
    }
    return SAM_OK;
}

int sam_cyclic_fold(sam_dtype dtype, int order, int tuple, const void* round_payloads, int rank, int nranks,
                    const void* base_in, void* seed_out, void* base_out, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAM_ERR_INVALID_ARG, "rank/nranks out of range");
    if (!round_payloads || !seed_out) return fail(SAM_ERR_INVALID_ARG, "null payloads or seed_out");
    const size_t pb = sam_shard_payload_bytes(dtype, order, tuple);
    cudaStream_t st = (cudaStream_t)stream;
    uint64_t l = 0;
    cudaError_t e;
    switch (dtype) {
        case SAM_I32: e = sam::launch_cyclic_fold<uint32_t>(round_payloads, pb, rank, nranks, order, tuple, base_in, seed_out, base_out, st, &l); break;
        case SAM_I64: e = sam::launch_cyclic_fold<uint64_t>(round_payloads, pb, rank, nranks, order, tuple, base_in, seed_out, base_out, st, &l); break;
        case SAM_F32: e = sam::launch_cyclic_fold<float>(round_payloads, pb, rank, nranks, order, tuple, base_in, seed_out, base_out, st, &l); break;
        default: e = sam::launch_cyclic_fold<double>(round_payloads, pb, rank, nranks, order, tuple, base_in, seed_out, base_out, st, &l); break;
    }
    g_launches += l;
    return e == cudaSuccess ? SAM_OK : cuda_fail(e, "cyclic fold launch");
}

int sam_cyclic_fold_host(sam_dtype dtype, int order, int tuple, const void* round_payloads_host, int rank,
                         int nranks, const void* base_in_host, void* seed_out_host, void* base_out_host) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(SAM_ERR_INVALID_ARG, "rank/nranks out of range");
    if (!round_payloads_host || !seed_out_host) return fail(SAM_ERR_INVALID_ARG, "null buffer");
    const size_t pb = sam_shard_payload_bytes(dtype, order, tuple);
    const unsigned char* P = (const unsigned char*)round_payloads_host;
    switch (dtype) {
        case SAM_I32: cyclic_fold_host_t<uint32_t>(P, pb, rank, nranks, order, tuple, (const uint32_t*)base_in_host, (uint32_t*)seed_out_host, (uint32_t*)base_out_host); break;
        case SAM_I64: cyclic_fold_host_t<uint64_t>(P, pb, rank, nranks, order, tuple, (const uint64_t*)base_in_host, (uint64_t*)seed_out_host, (uint64_t*)base_out_host); break;
        case SAM_F32: cyclic_fold_host_t<float>(P, pb, rank, nranks, order, tuple, (const float*)base_in_host, (float*)seed_out_host, (float*)base_out_host); break;
        default: cyclic_fold_host_t<double>(P, pb, rank, nranks, order, tuple, (const double*)base_in_host, (double*)seed_out_host, (double*)base_out_host); break;
    }
    return SAM_OK;
}

// ---------------------------------------------------------------------------------------------
// host-buffer streaming pipeline: H2D(j+1) | scan(j) | D2H(j-1) on three streams
// ---------------------------------------------------------------------------------------------
namespace {
struct HostPipe {
    static constexpr int NB = 3;
    int dev = -1;
    size_t chunk_bytes = 0;
    unsigned char* buf[NB] = {nullptr, nullptr, nullptr};
    unsigned char* state = nullptr;  // 2 x 512 B
    unsigned char* obuf[NB] = {nullptr, nullptr, nullptr};  // encoder outputs (allocated on first use)
    unsigned char* halo = nullptr;                         // encoder halos, 2 x 512 B
    cudaStream_t s_h2d = nullptr, s_cmp = nullptr, s_d2h = nullptr;
    cudaEvent_t ev_h2d[NB], ev_cmp[NB], ev_d2h[NB], ev_start;
};
std::mutex g_pipe_mu;
std::map<int, HostPipe*> g_pipes;
constexpr size_t kChunkBytes = size_t(128) << 20;

int get_pipe(HostPipe** out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    HostPipe*& P = g_pipes[dev];
    if (!P) {
        P = new HostPipe();
        P->dev = dev;
        P->chunk_bytes = kChunkBytes;
        for (int i = 0; i < HostPipe::NB; ++i) {
            e = cudaMalloc(&P->buf[i], P->chunk_bytes);
            if (e != cudaSuccess) return fail(SAM_ERR_OOM, "host pipeline buffers");
            cudaEventCreateWithFlags(&P->ev_h2d[i], cudaEventDisableTiming);
            cudaEventCreateWithFlags(&P->ev_cmp[i], cudaEventDisableTiming);
            cudaEventCreateWithFlags(&P->ev_d2h[i], cudaEventDisableTiming);
        }
        e = cudaMalloc(&P->state, 1024);
        if (e != cudaSuccess) return fail(SAM_ERR_OOM, "host pipeline state");
        cudaEventCreateWithFlags(&P->ev_start, cudaEventDisableTiming);
        cudaStreamCreateWithFlags(&P->s_h2d, cudaStreamNonBlocking);
        cudaStreamCreateWithFlags(&P->s_cmp, cudaStreamNonBlocking);
        cudaStreamCreateWithFlags(&P->s_d2h, cudaStreamNonBlocking);
    }
    *out = P;
    return SAM_OK;
}
}  // namespace

int sam_scan_host(sam_dtype dtype, int order, int tuple, int inclusive, const void* in_host, void* out_host,
                  uint64_t n, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (n == 0) return SAM_OK;
    if (!in_host || !out_host) return fail(SAM_ERR_INVALID_ARG, "null buffer with n > 0");
    std::lock_guard<std::mutex> lk(g_pipe_mu);
    HostPipe* P = nullptr;
    rc = get_pipe(&P);
    if (rc) return rc;
    const size_t w = elem_size(dtype);
    const uint64_t C = P->chunk_bytes / w;
    const uint64_t nchunks = (n + C - 1) / C;
    cudaStream_t user = (cudaStream_t)stream;
    cudaEventRecord(P->ev_start, user);
    cudaStreamWaitEvent(P->s_h2d, P->ev_start, 0);
    cudaStreamWaitEvent(P->s_cmp, P->ev_start, 0);
    cudaStreamWaitEvent(P->s_d2h, P->ev_start, 0);
    const size_t sb = (size_t)order * tuple * w;
    for (uint64_t j = 0; j < nchunks; ++j) {
        const int b = (int)(j % HostPipe::NB);
        const uint64_t off = j * C;
        const uint64_t cn = (n - off < C) ? n - off : C;
        if (j >= (uint64_t)HostPipe::NB) cudaStreamWaitEvent(P->s_h2d, P->ev_d2h[b], 0);
        cudaError_t e = cudaMemcpyAsync(P->buf[b], (const unsigned char*)in_host + off * w, cn * w,
                                        cudaMemcpyHostToDevice, P->s_h2d);
        if (e != cudaSuccess) return cuda_fail(e, "H2D");
        cudaEventRecord(P->ev_h2d[b], P->s_h2d);
        cudaStreamWaitEvent(P->s_cmp, P->ev_h2d[b], 0);
        const void* seed = j ? (const void*)(P->state + ((j - 1) & 1) * 512) : nullptr;
        void* fin = (j + 1 < nchunks) ? (void*)(P->state + (j & 1) * 512) : nullptr;
        (void)sb;
        rc = sam_scan_seeded(dtype, order, tuple, inclusive, P->buf[b], P->buf[b], cn, off, seed, fin, P->s_cmp);
        if (rc) return rc;
        cudaEventRecord(P->ev_cmp[b], P->s_cmp);
        cudaStreamWaitEvent(P->s_d2h, P->ev_cmp[b], 0);
        e = cudaMemcpyAsync((unsigned char*)out_host + off * w, P->buf[b], cn * w, cudaMemcpyDeviceToHost, P->s_d2h);
        if (e != cudaSuccess) return cuda_fail(e, "D2H");
        cudaEventRecord(P->ev_d2h[b], P->s_d2h);
    }
    cudaError_t e = cudaStreamSynchronize(P->s_d2h);
    if (e == cudaSuccess) e = cudaStreamSynchronize(P->s_cmp);
    if (e != cudaSuccess) return cuda_fail(e, "host pipeline");
    return SAM_OK;
}

int sam_delta_encode_host(sam_dtype dtype, int order, int tuple, const void* in_host, void* out_host, uint64_t n,
                          sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if (n == 0) return SAM_OK;
    if (!in_host || !out_host) return fail(SAM_ERR_INVALID_ARG, "null buffer with n > 0");
    if (in_host == out_host) return fail(SAM_ERR_INVALID_ARG, "delta encoding is not done in place (P:281-284)");
    std::lock_guard<std::mutex> lk(g_pipe_mu);
    HostPipe* P = nullptr;
    rc = get_pipe(&P);
    if (rc) return rc;
    if (!P->halo) {
        for (int i = 0; i < HostPipe::NB; ++i)
            if (cudaMalloc(&P->obuf[i], P->chunk_bytes) != cudaSuccess) return fail(SAM_ERR_OOM, "encoder buffers");
        if (cudaMalloc(&P->halo, 1024) != cudaSuccess) return fail(SAM_ERR_OOM, "encoder halo");
    }
    const size_t w = elem_size(dtype);
    const uint64_t C = P->chunk_bytes / w;  // >= order*tuple: only the last chunk is short
    const uint64_t nchunks = (n + C - 1) / C;
    const size_t hb = (size_t)order * tuple * w;
    cudaStream_t user = (cudaStream_t)stream;
    cudaEventRecord(P->ev_start, user);
    cudaStreamWaitEvent(P->s_h2d, P->ev_start, 0);
    cudaStreamWaitEvent(P->s_cmp, P->ev_start, 0);
    cudaStreamWaitEvent(P->s_d2h, P->ev_start, 0);
    for (uint64_t j = 0; j < nchunks; ++j) {
        const int b = (int)(j % HostPipe::NB);
        const uint64_t off = j * C;
        const uint64_t cn = (n - off < C) ? n - off : C;
        // buf[b] / obuf[b] are free once chunk j-NB has left the device
        if (j >= (uint64_t)HostPipe::NB) {
            cudaStreamWaitEvent(P->s_h2d, P->ev_d2h[b], 0);
            cudaStreamWaitEvent(P->s_cmp, P->ev_d2h[b], 0);
        }
        cudaError_t e = cudaMemcpyAsync(P->buf[b], (const unsigned char*)in_host + off * w, cn * w,
                                        cudaMemcpyHostToDevice, P->s_h2d);
        if (e != cudaSuccess) return cuda_fail(e, "H2D");
        cudaEventRecord(P->ev_h2d[b], P->s_h2d);
        cudaStreamWaitEvent(P->s_cmp, P->ev_h2d[b], 0);
        // chunk j's halo = the last order*tuple inputs of chunk j-1, saved on the compute stream
        const void* halo = j ? (const void*)(P->halo + ((j - 1) & 1) * 512) : nullptr;
        rc = sam_delta_encode_halo(dtype, order, tuple, P->buf[b], P->obuf[b], cn, halo, P->s_cmp);
        if (rc) return rc;
        if (j + 1 < nchunks) {
            e = cudaMemcpyAsync(P->halo + (j & 1) * 512, P->buf[b] + cn * w - hb, hb, cudaMemcpyDeviceToDevice,
                                P->s_cmp);
            if (e != cudaSuccess) return cuda_fail(e, "halo copy");
        }
        cudaEventRecord(P->ev_cmp[b], P->s_cmp);
        cudaStreamWaitEvent(P->s_d2h, P->ev_cmp[b], 0);
        e = cudaMemcpyAsync((unsigned char*)out_host + off * w, P->obuf[b], cn * w, cudaMemcpyDeviceToHost,
                            P->s_d2h);
        if (e != cudaSuccess) return cuda_fail(e, "D2H");
        cudaEventRecord(P->ev_d2h[b], P->s_d2h);
    }
    cudaError_t e = cudaStreamSynchronize(P->s_d2h);
    if (e == cudaSuccess) e = cudaStreamSynchronize(P->s_cmp);
    if (e != cudaSuccess) return cuda_fail(e, "encoder host pipeline");
    return SAM_OK;
}

int sam_delta_encode(sam_dtype dtype, int order, int tuple, const void* in, void* out, uint64_t n,
                     sam_stream_t stream) {
    return sam_delta_encode_halo(dtype, order, tuple, in, out, n, nullptr, stream);
}

int sam_delta_encode_halo(sam_dtype dtype, int order, int tuple, const void* in, void* out, uint64_t n,
                          const void* halo, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    rc = validate_buffers(dtype, in, out, n, true);
    if (rc) return rc;
    if (n > 0 && in == out)
        return fail(SAM_ERR_INVALID_ARG, "delta encoding is not done in place (P:281-284): in must differ from out");
    if (n == 0) return SAM_OK;
    if (halo && ((uintptr_t)halo % elem_size(dtype)) != 0)
        return fail(SAM_ERR_INVALID_ARG, "halo must be aligned to the element size");
    cudaStream_t st = (cudaStream_t)stream;
    uint64_t l = 0;
    cudaError_t e;
    switch (dtype) {
        case SAM_I32: e = sam::launch_delta<uint32_t>(in, out, n, order, tuple, halo, st, &l); break;
        case SAM_I64: e = sam::launch_delta<uint64_t>(in, out, n, order, tuple, halo, st, &l); break;
        case SAM_F32: e = sam::launch_delta<float>(in, out, n, order, tuple, halo, st, &l); break;
        default: e = sam::launch_delta<double>(in, out, n, order, tuple, halo, st, &l); break;
    }
    g_launches += l;
    return e == cudaSuccess ? SAM_OK : cuda_fail(e, "delta encoder launch");
}

int sam_scan_generic(sam_dtype dtype, sam_op op, sam_carry carry, int order, int tuple, int inclusive,
                     const void* in, void* out, uint64_t n, sam_stream_t stream) {
    int rc = validate_common(dtype, order, tuple);
    if (rc) return rc;
    if ((int)op < 0 || (int)op > 3) return fail(SAM_ERR_UNSUPPORTED, "unknown operator");
    if ((int)carry < 0 || (int)carry > 2) return fail(SAM_ERR_UNSUPPORTED, "unknown carry scheme");
    if (op == SAM_OP_XOR && (dtype == SAM_F32 || dtype == SAM_F64))
        return fail(SAM_ERR_UNSUPPORTED, "xor is defined for integer dtypes only (reading R14)");
    rc = validate_buffers(dtype, in, out, n, true);
    if (rc) return rc;
    if (n == 0) return SAM_OK;
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* ws = nullptr;
    int dev = 0;
    const size_t rmax = ring_max_bytes();
    rc = get_ws(st, rmax + sam::gen::generic_words_bytes((int)dtype, order, tuple, n), &ws, &dev);
    if (rc) return rc;
    sam::gen::GenArgs a;
    memset(&a, 0, sizeof(a));
    a.in = in;
    a.out = out;
    a.n = n;
    a.s = tuple;
    a.k = order;
    a.inclusive = inclusive ? 1 : 0;
    a.mode = (int)carry;
    a.words = ws->carry + rmax / 8;  // after the main kernel's ring: separate tags and layout
    a.words_bytes = ws->carry_cap - rmax;
    a.tile_ctr = (unsigned long long*)(ws->ctr);
    a.done_ctr = (unsigned int*)(ws->ctr + 8);
    a.epoch_ptr = (unsigned int*)(ws->ctr + 12);
    a.dev = dev;
    a.num_sms = num_sms_of(dev);
    a.stream = st;
    a.mode_used = &g_last_carry;
    cudaError_t e = sam::gen::launch_generic((int)dtype, (int)op, a);
    if (e != cudaSuccess) return cuda_fail(e, "generic scan kernel launch");
    g_launches += 1;
    return SAM_OK;
}

int sam_scan_op(sam_dtype dtype, sam_op op, int order, int tuple, int inclusive, const void* in, void* out,
                uint64_t n, sam_stream_t stream) {
    if (op == SAM_OP_ADD) return sam_scan(dtype, order, tuple, inclusive, in, out, n, stream);
    return sam_scan_generic(dtype, op, SAM_CARRY_STATIC, order, tuple, inclusive, in, out, n, stream);
}

int sam_last_carry_scheme(void) { return g_last_carry; }

int sam_debug_limit_grid(uint64_t max_ctas) {
    sam::debug_grid_limit() = max_ctas;
    for (int d = 0; d < sam::MAX_DEVICES; ++d) sam::debug_grid_cap(d) = 0;
    return SAM_OK;
}

int sam_tune_override(int tiles_per_unit, int lag, int vfold, int land, int teams) {
    sam::Knobs& k = sam::knobs_mut();
    k.teams = (teams == 1 || teams == 2 || teams == 4) ? teams : 0;
    k.super_tile = (tiles_per_unit >= 1 && tiles_per_unit <= 8) ? tiles_per_unit : 0;
    k.lag = lag >= 1 ? lag : 0;
    k.vfold = vfold >= 0 ? (vfold != 0) : -1;
    k.land = land >= 0 ? (land != 0) : -1;
    return SAM_OK;
}

int sam_debug_last_shape(int* out6) {
    if (!out6) return fail(SAM_ERR_INVALID_ARG, "null output");
    for (int i = 0; i < 6; ++i) out6[i] = sam::last_shape()[i];
    return SAM_OK;
}

int sam_debug_set_stress(uint32_t seed) {
    sam::debug_stress() = seed;
    return SAM_OK;
}

int sam_debug_set_trace(void* trace_dev) {
    g_trace = (unsigned long long*)trace_dev;
    return SAM_OK;
}

const char* sam_last_error(void) { return g_err.c_str(); }
const char* sam_version(void) { return kVersion; }
uint64_t sam_launch_count(void) { return g_launches.load(); }

int sam_release_workspaces(void) {
    std::lock_guard<std::mutex> lk(g_mu);
    cudaDeviceSynchronize();
    for (auto& kv : g_ws) {
        Workspace* ws = kv.second;
        if (ws->carry) cudaFree(ws->carry);
        if (ws->ctr) cudaFree(ws->ctr);
        if (ws->part) cudaFree(ws->part);
        delete ws;
    }
    g_ws.clear();
    return SAM_OK;
}

}  // extern "C"
