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
    MSORT_ERR_NCCL = 5,             /* libnccl missing, or an NCCL call failed (exchange mode 4)            */
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
 *            BLOCKS until the sorted result is in `keys` (the statistics of the
 *            merge stages are read back at the end).
 * A per-(device set, key type) context is cached and grown on demand
 * (msort_release_cached drops them). */
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
                                       from every chunk into a local buffer), then the merge tree;
                                       4: the swap as grouped ncclSend/ncclRecv per mirrored pair into a
                                       receive buffer, then a local merge (north_star S5).  Single process:
                                       one NCCL communicator per distinct device, created here (ranks sharing
                                       a device use NCCL self send/recv); dist mode: call
                                       msort_dist_nccl_init on every rank first.  libnccl.so.2 is loaded at
                                       run time (MSORT_NCCL_LIB overrides); MSORT_ERR_NCCL if unavailable.
                                       Modes 1 and 4 read each stage's pivots on the host (the NCCL counts
                                       are host arguments); mode 0 keeps every stage on the GPUs            */
    MSORT_OPT_SKIP_TRIVIAL = 2,  /* 1: skip radix passes whose digit is constant (identity permutation)   */
    MSORT_OPT_HOST_PIPELINE = 3, /* 1 (default): host sorts overlap the transfers with the sort (chunks of
                                       at least 2^20 keys) - the chunk arrives in 4 pieces, each radix sorted
                                       while the next is in flight, and the sorted pieces merge.  One GPU
                                       (msort_sort_host, g = 1): the final merge runs in slices, each copied
                                       back while the next one merges.  msort_dist_sort_host: the merged
                                       chunk enters the merge phase, D2H follows it.  0: H2D, sort, D2H
                                       one after the other                                                */
    MSORT_OPT_SMALL_GRAPH = 4,   /* 1 (default): a one-GPU device sort of <= 2^22 keys repeated on the same
                                       buffer and size replays the whole radix sort as one CUDA graph
                                       (captured on the second call; all passes run, no host round trip on
                                       the histogram); 0: always the launch-by-launch path              */
    MSORT_OPT_STOP_AFTER_STAGE = 101, /* testing only: end the Alg.2 merge phase (modes 0, 1, 4) after stage
                                       `value` (-1: all stages); every chunk then holds what the paper's
                                       stage model holds after that stage (per-stage parity)*/
    MSORT_OPT_RADIX_EPOCH = 100  /* testing only: set the radix workspace epoch (0..511) so that the next
                                       sort runs at epoch value+1; the look-back words carry the epoch as a
                                       tag and the whole workspace is zeroed when it wraps to 0            */
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
    int      exchange_mode;                             /* MSORT_OPT_EXCHANGE as run: 0 / 2 fall back to 1 / 3
                                                           when peer_bulk_ok == 0                      */
    int      peer_bulk_ok;                              /* 1: TMA bulk copies from peer memory passed the
                                                           self-test msort_create / msort_dist_import run
                                                           between distinct devices (or none needed)   */
    double   stage_swap_ms[MSORT_MAX_STAGES];           /* the transfer alone (modes 1 / 4: copy or NCCL
                                                           send/recv; fused modes: = stage_exchange_ms) */
    double   stage_pivot_ms[MSORT_MAX_STAGES];          /* stage start .. exchange start: the pivot search
                                                           (S4; modes 1 / 4 include its host read-back) */
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
/* msort_plan_chunk - the chunking rule ("equally sized chunks",
 * DESIGN.md reading Q3), host only: for n keys on g GPUs, rank `rank` owns the
 * input keys [offset, offset + valid) in a chunk of c keys, where
 *   c      = ceil(n / g) rounded up to a multiple of 4 keys (16-byte alignment),
 *   offset = min(rank * c, n),   valid = min(max(n - rank * c, 0), c).
 * The library pads [valid, c) with the largest key under T; the pads sort to
 * the global end and are dropped, so after a sort rank r's first `valid` keys
 * are global ranks [offset, offset + valid) of the sorted output.
 * Outputs may be NULL.  INVALID_ARGUMENT for g not in {1,2,4,8} or rank out of range. */
int msort_plan_chunk(uint64_t n, int g, int rank, uint64_t* c, uint64_t* offset, uint64_t* valid);

/* msort_dist_sort - device-resident sort of n_total keys spread over the
 * `world` ranks by msort_plan_chunk: d_chunk (device pointer on this rank's
 * device, room for c keys, 16-byte aligned) holds this rank's `valid` input
 * keys; every rank calls with the same n_total.  The library pads the chunk
 * (reading Q3), sorts, and leaves this rank's `valid` sorted keys (global ranks
 * [offset, offset + valid)) in d_chunk[0, valid).  Cross-GPU ordering uses
 * device-side barriers on IPC-mapped flags (timeout -> MSORT_ERR_TIMEOUT).
 * Ordered after `stream`; blocks until done. */
int msort_dist_sort(msort_ctx* ctx, void* d_chunk, uint64_t n_total, void* stream);

/* End-to-end dist sort: host_keys holds this rank's `valid` keys
 * (msort_plan_chunk; pinned for full PCIe rate) -> H2D -> pad -> msort_dist_sort
 * -> D2H of the `valid` sorted keys, in place.  Blocks until done. */
int msort_dist_sort_host(msort_ctx* ctx, void* host_keys, uint64_t n_total);

/* Exchange mode 4 in dist mode: rank 0 creates an NCCL unique id
 * (MSORT_NCCL_ID_BYTES bytes), the caller broadcasts it (e.g. with
 * torch.distributed), and every rank joins the communicator of `world` ranks.
 * MSORT_ERR_NCCL on failure (no libnccl, or NCCL refused the ranks - e.g. two
 * ranks on one GPU). */
#define MSORT_NCCL_ID_BYTES 128
int msort_nccl_unique_id(void* out);
int msort_dist_nccl_init(msort_ctx* ctx, const void* unique_id);

/* ------------------------------------------------------------------------ */
/* Interconnect peaks (the denominators of the NVLink / PCIe fractions)      */
/* ------------------------------------------------------------------------ */

typedef struct {
    double   p2p_ce_gbs;     /* per GPU and direction: mirrored pairs GPU i <-> GPU g-1-i copying concurrently
                                in both directions (§4.3), copy engines (peer cudaMemcpyAsync) */
    double   p2p_sm_gbs;     /* same pattern, SM loads through the peer mapping (the fused merge's access)  */
    double   h2d_gbs;        /* per GPU, all of this context's GPUs copying host->device concurrently (§4.2) */
    double   d2h_gbs;        /* per GPU, all GPUs device->host concurrently                                  */
    double   bidir_gbs;      /* per GPU and direction, H2D and D2H at the same time             */
    uint64_t bytes;          /* bytes per copy (<= one chunk buffer)                                        */
    int      pairs;          /* mirrored pairs measured (g/2; 0 when g == 1)                                */
    int      same_device;    /* 1: a pair shares one GPU (virtual ranks): the P2P numbers are HBM copies    */
} msort_link_peaks;

/* msort_measure_links - time the interconnect patterns above with the
 * context's own buffers (their contents are overwritten: do not overlap a
 * sort).  Single process: every rank of the context; the result is the
 * slowest GPU's rate.  Dist mode: collective (every rank calls it; device
 * barriers line the ranks up), the result is THIS rank's rate (reduce the
 * minimum across ranks).  Pinned host buffers of `bytes` per GPU are allocated
 * and freed inside.  `reps` timed repetitions (mean), after one warm-up. */
int msort_measure_links(msort_ctx* ctx, uint64_t bytes, int reps, msort_link_peaks* out);

/* msort_release_cached - destroy every context msort_sort cached (device
 * buffers of about 3 chunk copies per GPU stay allocated between msort_sort
 * calls otherwise).  Safe to call at any time no msort_sort is running; the
 * next msort_sort re-creates what it needs. */
int msort_release_cached(void);

#ifdef __cplusplus
}
#endif
#endif /* MSORT_H */
