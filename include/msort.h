/*
 * msort.h - C ABI of the B200-native multi-GPU P2P sort (libmsort.so).
 *
 * Method: Maltenberger, Ilic, Tolovski, Rabl, "Evaluating Multi-GPU Sorting
 * with Modern Interconnects", SIGMOD '22.  Citations "P:n" are lines of the
 * paper text (/root/reference/PAPER.md at build time; the sections are named
 * beside each citation so the header stands on its own).
 *
 * What the library computes (§5, §5.1, §5.2
 * P:1588-1854): n keys are split into g = 1, 2, 4 or 8 equal chunks, one per
 * GPU; every GPU radix-sorts its chunk (LSD, 8-bit digits, onesweep); then
 * g-1 merge stages (Alg.2), each a pivot search (Alg.1
 * P:1613-1625), an exchange of the pivot-split key ranges between mirrored GPU
 * pairs and a local two-run merge,
 * leave GPU i holding global ranks [i*c, (i+1)*c).
 *
 * Order: ascending by the unsigned value of T(key): T = identity for
 * u32/u64; for f32/f64 T flips all bits of negative keys and the sign bit of
 * the others (IEEE-754 totalOrder: -NaN < -inf < ... < -0.0 < +0.0 < ... <
 * +inf < +NaN).  The paper sorts "integers, floats, longs and doubles"
 * (§6.3) and is silent on -0.0/NaN; reading Q1.
 * Keys are never modified bitwise; the output is a permutation of the input.
 *
 * Conventions for every function:
 *   - returns an msort_status (0 = MSORT_OK); no C++ exception crosses the ABI;
 *     msort_last_error() returns a thread-local detail string;
 *   - "stream" arguments are cudaStream_t passed as void* (NULL = legacy
 *     default stream); device pointers are CUDA device addresses; "host"
 *     pointers are CPU addresses (pinned memory gives full PCIe rate);
 *   - the caller owns every buffer it passes in; the library never frees them.
 *     A context (msort_ctx) owns all device buffers, streams and events it
 *     allocates; nothing is allocated inside a sort call after the first call
 *     at a given capacity (all device memory is
 *     pre-allocated);
 *   - there is NO CPU fallback: without a usable GPU every compute entry point
 *     fails with MSORT_ERR_DEVICE or MSORT_ERR_CUDA.
 */
#ifndef MSORT_H
#define MSORT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MSORT_MAX_GPUS 8
#define MSORT_MAX_STAGES 7          /* g - 1 stages for g = 8 */
#define MSORT_RADIX_BITS 8          /* DESIGN.md reading Q10 */
#define MSORT_DIST_HANDLE_BYTES 512 /* opaque per-rank bytes exchanged by msort_dist_* */

typedef enum {
    MSORT_U32 = 0,   /* unsigned 32-bit integers ("integers") */
    MSORT_U64 = 1,   /* unsigned 64-bit integers ("longs")    */
    MSORT_F32 = 2,   /* IEEE binary32 ("floats")                          */
    MSORT_F64 = 3    /* IEEE binary64 ("doubles")                         */
} msort_key_type;

typedef enum {
    MSORT_OK = 0,
    MSORT_ERR_INVALID_ARGUMENT = 1, /* NULL pointer with n > 0, bad key_type, g not in {1,2,4,8}, c >= 2^32 */
    MSORT_ERR_DEVICE = 2,           /* too few GPUs, no peer access, no CUDA device                        */
    MSORT_ERR_OUT_OF_MEMORY = 3,    /* device or pinned allocation failed (no CPU fallback)                */
    MSORT_ERR_CUDA = 4,             /* a CUDA runtime call or kernel failed                                */
    MSORT_ERR_NCCL = 5,             /* reserved                                                            */
    MSORT_ERR_INTERNAL = 6,         /* invariant violated inside the library                               */
    MSORT_ERR_TIMEOUT = 7           /* a cross-GPU device barrier did not complete (dist mode)             */
} msort_status;

/* ------------------------------------------------------------------------ */
/* Whole sort                                                               */
/* ------------------------------------------------------------------------ */

/* msort_sort - sort n keys in place (the north_star entry point).
 *   keys     host pointer (pinned or pageable) or device pointer (detected with
 *            cudaPointerGetAttributes). Device pointers must live on device 0
 *            when n_gpus > 1, or on the current device when n_gpus == 1.
 *   n        number of keys; n <= 1 is a no-op.
 *   key_type msort_key_type.
 *   n_gpus   g in {1,2,4,8}: GPUs 0..g-1 each sort c = ceil(n/g) (rounded up
 *            to a multiple of 4) keys; the tail is padded with the largest key
 *            under T and the padding is dropped (reading Q3).
 *   stream   the sort is ordered after work already queued on `stream`; the call
 *            BLOCKS until the sorted result is in `keys` (NCCL-free host round
 *            trips per merge stage make the call synchronous anyway).
 * A per-(device set, key type) context is cached and grown on demand. */
int msort_sort(void* keys, uint64_t n, int key_type, int n_gpus, void* stream);

/* ------------------------------------------------------------------------ */
/* Context: pre-allocated buffers, streams, events (single process, g GPUs) */
/* ------------------------------------------------------------------------ */

typedef struct msort_ctx msort_ctx;

/* msort_create - allocate a context for n_gpus chunks of up to
 * ceil(max_keys/n_gpus) keys each.
 *   device_ids  NULL -> 0..n_gpus-1.  Entries may REPEAT a device: several
 *               "virtual ranks" on one GPU run the identical algorithm with
 *               peer loads becoming local loads (used to test g > 1 on 1 GPU).
 * Per chunk the context allocates two internal chunk buffers (B0, B1), one
 * chunk staging buffer for host sorts, and the radix workspace.  Peer access is
 * enabled between distinct devices (MSORT_ERR_DEVICE if impossible). */
int msort_create(msort_ctx** out, int n_gpus, const int* device_ids, uint64_t max_keys, int key_type);
int msort_destroy(msort_ctx* ctx);

/* Options (msort_set_option). */
enum {
    MSORT_OPT_TIMING = 0,        /* 1: record CUDA events per phase / per radix pass / per merge (default 1) */
    MSORT_OPT_EXCHANGE = 1,      /* 0: fused exchange+merge, the merge kernel loads the partner's block over
                                       NVLink directly (default); 1: swap first (peer copy into a receive
                                       buffer), then a local merge;
                                       2: NEXT-1, the paper's future work: exact multi-sequence
                                       splitters over all g sorted chunks, ONE all-to-all exchange fused into
                                       a log2(g)-round merge tree whose first round reads the g runs straight
                                       from the peers' chunks over NVLink;
                                       3: NEXT-1 with the exchange as separate pulls (every GPU copies its run
                                       from every chunk into a local buffer), then the merge tree            */
    MSORT_OPT_SKIP_TRIVIAL = 2,  /* 1: skip radix passes whose digit is constant (identity permutation)   */
    MSORT_OPT_HOST_PIPELINE = 3, /* 1 (default): host sorts overlap the transfers with the sort (chunks of
                                       at least 2^20 keys) - the chunk arrives in 4 pieces, each radix sorted
                                       while the next is in flight, and the sorted pieces merge.  One GPU
                                       (msort_sort_host, g = 1): the final merge runs in slices, each copied
                                       back while the next one merges.  msort_dist_sort_host: the merged
                                       chunk enters the merge phase, D2H follows it.  0: H2D, sort, D2H
                                       one after the other                                                */
    MSORT_OPT_SMALL_GRAPH = 4    /* 1 (default): a one-GPU device sort of <= 2^22 keys repeated on the same
                                       buffer and size replays the whole radix sort as one CUDA graph
                                       (captured on the second call; all passes run, no host round trip on
                                       the histogram); 0: always the launch-by-launch path              */
};
int msort_set_option(msort_ctx* ctx, int option, int64_t value);

/* msort_sort_host - end-to-end sort of n keys at host address host_keys, in
 * place: H2D of chunk i to GPU i, per-GPU radix sort, merge phase, D2H
 * (P:2244-2250).  Blocks until done. */
int msort_sort_host(msort_ctx* ctx, void* host_keys, uint64_t n);

/* msort_sort_device - device-resident sort.  chunks[i] is a device pointer on
 * the context's i-th device holding keys_per_gpu keys (16-byte aligned).  On
 * return chunk i holds global ranks [i*c, (i+1)*c) of the union, sorted.
 * streams: NULL or an array of n_gpus cudaStream_t; the sort is ordered after
 * them (NULL: after each device's legacy default stream) and they are ordered
 * after the sort.  Blocks until done. */
int msort_sort_device(msort_ctx* ctx, void* const* chunks, uint64_t keys_per_gpu, void* const* streams);

typedef struct {
    double   h2d_ms, sort_ms, merge_ms, d2h_ms, total_ms; /* phases; a phase ends when the last GPU ends */
    double   hist_ms;                 /* S2 upfront histogram, max over GPUs                    */
    double   pass_ms_sum;             /* S3 sum of onesweep pass durations, max over GPUs       */
    int      passes_run;              /* S3 onesweep passes executed per GPU                    */
    int      passes_total;            /* P = 8*K/8                                              */
    int      n_gpus;
    int      n_stages;
    uint64_t keys_per_gpu;
    int      stage_label[MSORT_MAX_STAGES];             /* chunks per group (Alg.2 merge stage i)  */
    uint64_t stage_pivot[MSORT_MAX_STAGES][MSORT_MAX_GPUS / 2]; /* p per group                     */
    uint64_t stage_max_x[MSORT_MAX_STAGES];             /* busiest mirrored pair's x_d             */
    uint64_t stage_keys_exchanged[MSORT_MAX_STAGES];    /* sum of x_d over pairs, one direction    */
    double   stage_ms[MSORT_MAX_STAGES];                /* barrier..merge end, max over GPUs       */
    double   stage_exchange_ms[MSORT_MAX_STAGES];       /* merge (fused) or swap+merge kernels     */
    int      kernel_launches;                           /* libmsort kernels launched by this process */
} msort_timings;

int msort_get_timings(const msort_ctx* ctx, msort_timings* out);

/* Ranking used by the onesweep passes on `device`: 1 = one shared-memory atomic
 * per key (the GPU passed the lane-order self-test, radix.cu), 0 = peer-match
 * ranking, -1 = no such device. */
int msort_rank_mode(int device);
const char* msort_status_string(int status);
const char* msort_last_error(void);
int msort_version(void);

/* ------------------------------------------------------------------------ */
/* Step-level entry points (one per SURVEY §8(a) row; used by parity tests) */
/* ------------------------------------------------------------------------ */

/* Bytes of device workspace msort_radix_sort / msort_step_radix_pass need for n keys. */
uint64_t msort_radix_workspace_bytes(uint64_t n, int key_type);

/* S1+S2: P = 8*sizeof(key)/8 histograms of the 8-bit digits of T(keys)
 * ("calculating the histogram once").  d_hist: device uint32
 * [P][256], overwritten.  n < 2^32. */
int msort_step_histogram(const void* d_keys, uint64_t n, int key_type, uint32_t* d_hist, void* stream);

/* S3: one stable onesweep pass on digit `pass` (0 = least significant):
 * out[base[d] + rank] = key, base = exclusive prefix of d_hist[pass].
 * flags: MSORT_PASS_ENCODE_IN (d_in holds raw keys: apply T when loading),
 *        MSORT_PASS_DECODE_OUT (write raw keys: apply T^-1 when storing);
 * otherwise d_in/d_out hold T-codes.  d_ws: >= msort_radix_workspace_bytes. */
#define MSORT_PASS_ENCODE_IN 1
#define MSORT_PASS_DECODE_OUT 2
int msort_step_radix_pass(const void* d_in, void* d_out, uint64_t n, int key_type, int pass,
                          const uint32_t* d_hist, int flags, void* d_ws, uint64_t ws_bytes, void* stream);

/* S1-S3: sort n keys at d_keys in place (d_aux: n keys of scratch). */
int msort_radix_sort(void* d_keys, void* d_aux, uint64_t n, int key_type, void* d_ws, uint64_t ws_bytes, void* stream);

/* S4: Alg.1 for the group of n_chunks sorted chunks of c keys
 * each: A = chunks[0 .. n_chunks/2), B = chunks[n_chunks/2 .. n_chunks) as
 * concatenated arrays (|A| = |B|, reading Q3).  Writes the leftmost pivot p
 * = #{i : B[i] < A[|A|-1-i]} (reading Q5) as uint64 to d_pivot.
 * d_chunks is a HOST array of device pointers (peer pointers allowed). */
int msort_step_pivot(const void* const* d_chunks, int n_chunks, uint64_t c, int key_type,
                     uint64_t* d_pivot, void* stream);

/* S6: merge two sorted runs a[0..a_len) and b[0..b_len) (either may be a peer
 * pointer) into out[0..a_len+b_len).  d_ws >=
 * msort_merge_workspace_bytes(a_len + b_len). */
uint64_t msort_merge_workspace_bytes(uint64_t total, int key_type);
int msort_step_merge(const void* d_a, uint64_t a_len, const void* d_b, uint64_t b_len, void* d_out,
                     int key_type, void* d_ws, uint64_t ws_bytes, void* stream);

/* NEXT-1 splitters (DESIGN reading Q15): for n_chunks sorted
 * chunks of c keys (HOST array of device pointers, peers allowed) writes the
 * device uint64 matrix d_s[(n_chunks+1) x n_chunks]: d_s[j*n_chunks + r] = how
 * many keys of chunk r are among the j*c smallest of the union (ties go to
 * lower r).  n_chunks in 2..8. */
int msort_step_splitters(const void* const* d_chunks, int n_chunks, uint64_t c, int key_type, uint64_t* d_s,
                         void* stream);

/* ------------------------------------------------------------------------ */
/* Host-side plan (no GPU needed): Alg.2 stage schedule and swap mapping     */
/* ------------------------------------------------------------------------ */

/* Number of sequential merge stages for g chunks: g-1 (reading Q7). */
int msort_plan_num_stages(int g);
/* Stage s (0-based) of g: *label = chunks per group; groups are [j*label, (j+1)*label). */
int msort_plan_stage(int g, int s, int* label);
/* For stage s with pivots[j] for group j: per chunk r: partner[r] (-1 if none),
 * x[r] = keys exchanged with the partner, side[r] = 0 (left half, sends its last
 * x) or 1 (right half, sends its first x).  Mirrored pairs d: L = mid-1-d,
 * R = mid+d, x_d = clamp(p - d*c, 0, c) (reading Q6, Fig.9). */
int msort_plan_exchange(int g, int s, uint64_t c, const uint64_t* pivots, int* partner, uint64_t* x, int* side);

/* ------------------------------------------------------------------------ */
/* Multi-process mode: one process per GPU (torchrun), peers via CUDA IPC    */
/* ------------------------------------------------------------------------ */

/* msort_dist_create - this process is `rank` of `world` (g = world), using
 * `device`.  Allocates B0/B1/signal buffers for up to max_keys_per_rank keys. */
int msort_dist_create(msort_ctx** out, int rank, int world, int device, uint64_t max_keys_per_rank, int key_type);
/* Writes MSORT_DIST_HANDLE_BYTES opaque bytes (IPC handles of this rank's
 * shared buffers) to handle_out; the caller all-gathers them (e.g. with
 * torch.distributed) into a world x MSORT_DIST_HANDLE_BYTES array. */
int msort_dist_export(msort_ctx* ctx, void* handle_out);
/* Maps every peer's shared buffers from the gathered handles. */
int msort_dist_import(msort_ctx* ctx, const void* all_handles);
/* Sort: d_chunk (device pointer on this rank's device, c keys); all ranks call
 * with the same c.  On return rank r holds global ranks [r*c, (r+1)*c).
 * Cross-GPU ordering uses device-side barriers on IPC-mapped flags (timeout ->
 * MSORT_ERR_TIMEOUT).  Blocks until done. */
int msort_dist_sort(msort_ctx* ctx, void* d_chunk, uint64_t c, void* stream);

/* End-to-end dist sort: host_keys (this rank's c keys, pinned for full PCIe
 * rate) -> H2D -> msort_dist_sort -> D2H, in place.  Blocks until done. */
int msort_dist_sort_host(msort_ctx* ctx, void* host_keys, uint64_t c);

#ifdef __cplusplus
}
#endif
#endif /* MSORT_H */
