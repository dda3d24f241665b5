/*
 * sam.h -- C ABI of libsam.so: single-pass higher-order (order k) and tuple-based (tuple s)
 * prefix sums on NVIDIA B200 (sm_100a).
 *
 * Method: Maleki, Yang & Burtscher, "Higher-Order and Tuple-Based Massively-Parallel Prefix
 * Sums", PLDI'16.  Citations "P:<line>" are lines of the paper text.
 *
 * SEMANTICS (what every entry point computes)
 *   Tuple s: element i of a stream belongs to lane m = (g + i) mod s, g being the
 *   global index of the stream's first element (0 for sam_scan); the s lanes are independent.
 *   Order 1, inclusive: y[i] = x[i] + y[previous element of the same lane].
 *   Order 1, exclusive: y[i] = sum of the lane's elements strictly before i.
 *   Order k: the order-1 operator applied k times; exclusive order k is the
 *   order-1 exclusive operator applied k times, i.e. the inclusive result shifted by k lane
 *   positions (reading R1).
 *   Integers: two's-complement wraparound mod 2^w (reading R2) -- results are bit-exact and
 *   independent of association order; SAM_I32/SAM_I64 may equally hold unsigned data.
 *   Floats: IEEE arithmetic in the element type; association order follows the tile geometry
 *   (reading R6); accuracy contract in DESIGN.md reading R7.
 *
 * MEMORY AND OWNERSHIP
 *   `in`, `out`, payload buffers: device pointers (cudaMalloc / torch CUDA tensors) on the
 *   current device, owned by the caller, aligned to the element size.  `in == out` (in-place)
 *   is allowed; any other overlap is SAM_ERR_INVALID_ARG.  Scratch (epoch-tagged carry words,
 *   a few counters) lives either in a workspace the library caches per (device, stream), grown
 *   lazily -- growing synchronises the stream -- and kept for the life of the process
 *   (sam_release_workspaces frees it), or, with sam_scan_ws, in a caller-owned workspace
 *   (no allocation, no synchronisation: the form for graph capture and concurrent streams).
 *   Calls on one stream are ordered; calls on different streams use different workspaces and
 *   may run concurrently.  The kernel resets its own counters and validates carry words by a
 *   per-launch epoch tag, so CUDA-graph replays need no host work (with the cached workspace,
 *   create it before capture: one un-captured call, or sam_prepare).
 *
 * EXECUTION MODEL
 *   One kernel launch per scan: a persistent grid of P co-resident CTAs (one per SM, launched
 *   cooperatively) runs SAM's static carry schedule: CTA b owns super-tiles b,
 *   b+P, b+2P, ...; the carry into super-tile S is the CTA's own inclusive state after S-P
 *   combined with the aggregates the other P-1 CTAs published in between.  This needs all P
 *   CTAs resident at once.  If the driver refuses the cooperative grid (MPS SM limits, a green
 *   context, an SM-partitioned device), the launch retries with a smaller grid -- the schedule
 *   is correct for any P -- and the reduced size is remembered for the device.
 *
 * ERRORS
 *   Every entry point returns a sam_status.  Argument validation happens synchronously before
 *   any CUDA call.  SAM_ERR_CUDA reports a launch/allocation failure; asynchronous device
 *   faults surface at the caller's next synchronisation.  sam_last_error() returns a
 *   thread-local description of the last failure on the calling thread.
 */
#ifndef SAM_H_
#define SAM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* SAM_U32 / SAM_U64: unsigned integers -- the same bits as SAM_I32 / SAM_I64 for add and xor, and the
 * unsigned order for max / min (SAM_I32 / SAM_I64 are signed there). */
typedef enum { SAM_I32 = 0, SAM_I64 = 1, SAM_F32 = 2, SAM_F64 = 3, SAM_U32 = 4, SAM_U64 = 5 } sam_dtype;

/* Associative operators ("prefix scans"). */
typedef enum { SAM_OP_ADD = 0, SAM_OP_XOR = 1, SAM_OP_MAX = 2, SAM_OP_MIN = 3 } sam_op;

/* Inter-tile carry schemes (the paper's Sec. 5.4). */
typedef enum {
    SAM_CARRY_STATIC = 0,   /* SAM's persistent-block schedule, P:783-832 (cooperative grid) */
    SAM_CARRY_LOOKBACK = 1, /* decoupled look-back over dynamically claimed tiles (no co-residency) */
    SAM_CARRY_CHAINED = 2   /* each tile waits for its predecessor's inclusive state */
} sam_carry;

typedef enum {
    SAM_OK = 0,
    SAM_ERR_INVALID_ARG = -1,  /* null pointer with n > 0, partial overlap, bad rank/nranks, misaligned */
    SAM_ERR_UNSUPPORTED = -2,  /* order or tuple outside 1..8, unknown dtype */
    SAM_ERR_CUDA = -3,         /* CUDA launch / runtime failure */
    SAM_ERR_OOM = -4,          /* workspace allocation failed */
    SAM_ERR_INTERNAL = -5
} sam_status;

/* `stream` is a cudaStream_t passed as an opaque pointer (NULL = legacy default stream). */
typedef void* sam_stream_t;

/*
 * sam_scan -- single-GPU order-k, tuple-s, inclusive/exclusive scan of n scalars.
 * One kernel launch, one read of `in` and one write of `out`, the
 * inter-tile carries propagated by SAM's static persistent-block schedule (see
 * EXECUTION MODEL above).
 *   dtype      element type of in/out (n elements each)
 *   order      k, 1..8          tuple  s, 1..8          inclusive  nonzero = inclusive
 *   n          number of scalars (not tuples); n = 0 is a no-op returning SAM_OK
 * Asynchronous on `stream`.
 */
int sam_scan(sam_dtype dtype, int order, int tuple, int inclusive, const void* in, void* out,
             uint64_t n, sam_stream_t stream);

/*
 * sam_scan_seeded -- sam_scan of a stream that continues an earlier one:
 *   global_offset  g = global index of in[0] (lane of in[0] is g mod s)
 *   seed           device pointer to order*tuple values of dtype, laid out [lane][order], the
 *                  state (y_1..y_k) of each global lane at its last element BEFORE this stream
 *                  (NULL = all zero, i.e. the stream starts the array)
 *   final_state    optional device pointer (order*tuple values, [lane][order]) receiving the
 *                  state of each lane at its last element of this stream (lanes with no
 *                  element in the stream receive their seed), NULL = not wanted.
 */
int sam_scan_seeded(sam_dtype dtype, int order, int tuple, int inclusive, const void* in,
                    void* out, uint64_t n, uint64_t global_offset, const void* seed,
                    void* final_state, sam_stream_t stream);

/* Make sure the workspace for (current device, stream) exists (optional; useful before graph
 * capture).  `max_n` sizes it for streams of up to max_n elements. */
int sam_prepare(sam_dtype dtype, int order, int tuple, uint64_t max_n, sam_stream_t stream);

/*
 * Explicit-workspace form (CUB-style), for graph capture and concurrent streams: no allocation,
 * no synchronisation, no library state per stream.
 *   sam_scan_workspace_size  *bytes = workspace bytes sam_scan_ws needs for (dtype, order, tuple,
 *                            n); a workspace sized for n serves any n' <= n.
 *   sam_scan_ws              sam_scan with the caller's workspace `ws` (device memory, 16-B
 *                            aligned, ws_bytes >= the size above).  The caller ZERO-FILLS the
 *                            workspace once before its first use (cudaMemsetAsync); afterwards the
 *                            kernel maintains it (epoch tags, counters reset by the last CTA of
 *                            each launch, a full reset when the 32-bit epoch wraps).  One
 *                            workspace serves one scan at a time: calls ordered on one stream may
 *                            share it, concurrent calls need distinct workspaces.
 *   Errors: as sam_scan; null/misaligned ws or ws_bytes too small -> SAM_ERR_INVALID_ARG.
 */
int sam_scan_workspace_size(sam_dtype dtype, int order, int tuple, uint64_t n, size_t* bytes);
int sam_scan_ws(sam_dtype dtype, int order, int tuple, int inclusive, const void* in, void* out,
                uint64_t n, void* ws, size_t ws_bytes, sam_stream_t stream);

/*
 * Host-buffer entry point (end-to-end path): `in_host` / `out_host` are host pointers
 * (pinned memory recommended; pageable works but is slower).  The array is streamed through
 * the GPU in chunks: H2D copy, seeded scan and D2H copy of consecutive chunks overlap on
 * separate streams, the carry of chunk j seeding chunk j+1 on the device.  Synchronous:
 * returns after out_host holds the result.  `stream` orders the work after prior work on it.
 */
int sam_scan_host(sam_dtype dtype, int order, int tuple, int inclusive, const void* in_host,
                  void* out_host, uint64_t n, sam_stream_t stream);

/* ---------------------------------------------------------------------------------------
 * Sharded (multi-GPU) scan: contiguous shards in rank order.
 *   1. sam_shard_state: read-only pass over the local shard (a dedicated reduction kernel, no
 *      carry chain: partial lane states combine with the carry operator in any grouping) -> payload (device memory,
 *      sam_shard_payload_bytes bytes): [u64 n_local][u64 global_offset][order*tuple values,
 *      [lane][order]], padded to a multiple of 16 B] = the zero-seeded state of each global lane at its last element of the
 *      shard.
 *   2. the caller all-gathers the payloads of all ranks (NCCL all_gather over NVLink), in
 *      rank order, into one device buffer of nranks * payload_bytes bytes.
 *   3. sam_shard_scan: folds the payloads of ranks < rank with the carry operator (lanes
 *      with no element in a shard pass the state through) into this shard's seed and runs
 *      the seeded single-pass scan (the binomial fix-up C(r+t-j, t-j) is fused into the
 *      carry application).
 * --------------------------------------------------------------------------------------- */
size_t sam_shard_payload_bytes(sam_dtype dtype, int order, int tuple);

int sam_shard_state(sam_dtype dtype, int order, int tuple, const void* in_local,
                    uint64_t n_local, uint64_t global_offset, void* payload_dev,
                    sam_stream_t stream);

int sam_shard_scan(sam_dtype dtype, int order, int tuple, int inclusive, const void* in_local,
                   void* out_local, uint64_t n_local, uint64_t global_offset,
                   const void* all_payloads_dev, int rank, int nranks, sam_stream_t stream);

/* Host-side fold of gathered payloads (host memory, same layout) into the seed of `rank`
 * (host memory, order*tuple values [lane][order], lanes of global index mod s).  This is the
 * same routine the device fold runs; exposed for CPU-side orchestration and tests. */
int sam_fold_payloads_host(sam_dtype dtype, int order, int tuple, const void* all_payloads_host,
                           int rank, int nranks, void* seed_host);

/* ---------------------------------------------------------------------------------------
 * Block-cyclic multi-GPU scan: SAM's carry scheme with the GPUs as the
 * persistent blocks ("each block ... only needs to read the local sums of the
 * previous P-1 chunks and its own carry from the previous iteration").  The global array is cut
 * into chunks of C elements; chunk c lives on rank c mod p, so round r holds chunks r*p .. r*p+p-1
 * (one per rank).  Per round each rank (1) runs sam_shard_state on its chunk (global offset
 * c*C) while the chunk stays in L2, (2) all ranks exchange the p payloads of the round, (3)
 * sam_cyclic_fold gives the carry into its chunk, (4) sam_scan_seeded scans the chunk (its re-read
 * an L2 hit when the chunk fits there), so each element costs one HBM read and one write on every
 * GPU -- contiguous shards cost 1.5x that (state pass over the whole shard, then the scan).  Each
 * round is three kernel launches, so chunks must be large enough to amortise them.
 *
 * sam_cyclic_fold: `round_payloads` (device, nranks * sam_shard_payload_bytes, rank order) = the
 * payloads of one round; `base_in` (device, [tuple][order], or NULL = zero state) = the state of
 * every global lane before the round (the stream seed before round 0).  Writes `seed_out`
 * (device, [tuple][order]) = base (+) payloads of ranks < rank, the carry operator (+) of
 * DESIGN.md §2 applied in rank order (lanes absent from a chunk pass through), and, if `base_out`
 * is not NULL, base (+) all nranks payloads = the next round's base.  base_out may alias base_in.
 * Every rank folds the same bytes in the same order: the bases are bit-identical on all ranks
 * (floats included).  Errors: UNSUPPORTED for order/tuple outside 1..8, INVALID_ARG for null
 * payloads/seed_out or rank outside [0, nranks).  One one-warp kernel, asynchronous on `stream`.
 * --------------------------------------------------------------------------------------- */
int sam_cyclic_fold(sam_dtype dtype, int order, int tuple, const void* round_payloads, int rank,
                    int nranks, const void* base_in, void* seed_out, void* base_out,
                    sam_stream_t stream);

/* The same fold on host buffers (CPU orchestration and tests). */
int sam_cyclic_fold_host(sam_dtype dtype, int order, int tuple, const void* round_payloads_host,
                         int rank, int nranks, const void* base_in_host, void* seed_out_host,
                         void* base_out_host);

/*
 * sam_delta_encode -- the k-th order, tuple-s difference sequence (delta ENCODER), the inverse of
 * the inclusive sam_scan with the same (order, tuple):
 *     out[i] = sum_{t=0..k} (-1)^t C(k,t) in[i - t*s],   in[j] = 0 for j < 0   ("missing" = 0)
 * = first-order differencing out_i = in_i - in_{i-s} applied k times (Sec. 2.4; the
 * paper's worked examples P:298-302; tuples P:349-355).  Embarrassingly parallel,
 * one read and one write of HBM, one kernel launch.
 *   dtype/order/tuple as for sam_scan; in, out: device pointers of n elements each.
 *   Integers: exact mod 2^w.  fp32: accumulated in double, rounded once; fp64: double.
 *   in == out (in place) or any overlap -> SAM_ERR_INVALID_ARG ("embarrassingly parallel when
 *   not done in place").  n = 0 is a no-op.  Asynchronous on `stream`.
 */
int sam_delta_encode(sam_dtype dtype, int order, int tuple, const void* in, void* out, uint64_t n,
                     sam_stream_t stream);

/* sam_delta_encode of a chunk / shard that continues an earlier stream: `halo` is a device
 * pointer to the order*tuple elements immediately preceding in[0] (halo[order*tuple - 1] is
 * adjacent to in[0]; zero-padded on the left when fewer precede), NULL = none ("missing" values
 * zero).  Encoding the shards of an array with their halos gives exactly the
 * whole-array result.  Misaligned halo -> SAM_ERR_INVALID_ARG. */
int sam_delta_encode_halo(sam_dtype dtype, int order, int tuple, const void* in, void* out, uint64_t n,
                          const void* halo, sam_stream_t stream);

/* Host-buffer encoder (end-to-end path): like sam_scan_host, the array is streamed through the GPU
 * in chunks, H2D | encode | D2H overlapping on separate streams; chunk j's halo is the last
 * order*tuple inputs of chunk j-1 (kept on the device).  Synchronous.  in_host == out_host ->
 * SAM_ERR_INVALID_ARG. */
int sam_delta_encode_host(sam_dtype dtype, int order, int tuple, const void* in_host, void* out_host,
                          uint64_t n, sam_stream_t stream);

/*
 * sam_scan_op -- order-k, tuple-s scan under operator `op` (NEXT-4).
 *   SAM_OP_ADD  = sam_scan (the production single-pass kernel).
 *   SAM_OP_XOR  integers only (floats -> SAM_ERR_UNSUPPORTED): addition in GF(2)^w, so the order-k
 *               carry algebra is the additive one with binomials reduced mod 2.
 *   SAM_OP_MAX / SAM_OP_MIN: every dtype; signed or unsigned order by dtype; floats use IEEE
 *               maxNum/minNum (a NaN operand is ignored; an all-NaN prefix yields the identity).
 *               Idempotent, so order k inclusive = order 1, and order k exclusive = the inclusive
 *               scan shifted by k lane positions (identity -inf/+inf/INT_MIN/... in front).
 *   Exclusive (all ops): the order-1 exclusive operator applied k times (reading R1), identity-seeded.
 *   Runs the generic kernel (sam_generic.cuh) with SAM's static carry schedule, falling back to the
 *   look-back form when no cooperative grid can form.  Arguments as sam_scan.
 */
int sam_scan_op(sam_dtype dtype, sam_op op, int order, int tuple, int inclusive, const void* in,
                void* out, uint64_t n, sam_stream_t stream);

/*
 * sam_scan_generic -- the generic kernel with an explicit carry scheme (NEXT-3 ablation: the same
 * intra-tile code under SAM's static schedule, decoupled look-back, or the chained scheme; the
 * look-back and chained forms need no co-resident grid).  `op` as sam_scan_op (ADD included).
 * sam_last_carry_scheme() returns the scheme the last call on this thread actually ran.
 */
int sam_scan_generic(sam_dtype dtype, sam_op op, sam_carry carry, int order, int tuple, int inclusive,
                     const void* in, void* out, uint64_t n, sam_stream_t stream);
int sam_last_carry_scheme(void);

/* Diagnostics */
const char* sam_last_error(void);
const char* sam_version(void);
int sam_release_workspaces(void);
/* Kernel launches issued by this library on the calling process since load (for bench). */
uint64_t sam_launch_count(void);
/* Testing: treat persistent grids above max_ctas CTAs as refused by the driver (0 = off), so the
 * cooperative-launch fallback shrinks the grid (to <= max_ctas) exactly as it does under MPS. */
int sam_debug_limit_grid(uint64_t max_ctas);
/* Tuning (tools/autotune.py): override, for subsequent scans of this process, the carry unit
 * (tiles per super-tile, 1..8), the pipeline depth (tiles between local scan and carry application),
 * the value-parallel integer fold (0/1), the landing-buffer fold (0/1) and the number of carry teams
 * (1, 2 or 4 teams of 4, 2 or 1 carry warps); -1 / 0 = no override.
 * The measured choices go to lib/sam_tune.txt, which the library reads once at first use (SAM's
 * install-time auto-tuner). */
int sam_tune_override(int tiles_per_unit, int lag, int vfold, int land, int teams);
/* Diagnostics: the launch shape of the last scan on this thread: out6 = {tiles per super-tile,
 * pipeline depth, value-parallel fold, landing fold, grid CTAs, items per thread}. */
int sam_debug_last_shape(int* out6);
/* Testing: nonzero seed = pseudo-random delays (up to ~16 us, 1 in 8 events) at every pipeline
 * hand-over of subsequent scan launches (loads, aggregate publication, carry folds, hand-offs,
 * local scans, carry applications), so the warps and CTAs meet in shuffled orders; 0 = off. */
int sam_debug_set_stress(uint32_t seed);
/* Diagnostics: when trace_dev (device memory, >= 16 * tiles u64, zeroed) is non-NULL, subsequent
 * scan launches record %globaltimer at pipeline events of every tile: [tile][claim, P1 start,
 * P1 done, aggregate published, look-back start, inclusive published, carry applied, stored,
 * first poll issued, first poll returned, look-back done, #polls, stop = own previous unit, ...]
 * (look-back fields on the first tile of each look-back unit).  NULL turns tracing off. */
int sam_debug_set_trace(void* trace_dev);

#ifdef __cplusplus
}
#endif
#endif /* SAM_H_ */
