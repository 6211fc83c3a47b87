// msort.cpp - C ABI, contexts and the stage scheduler of the P2P sort.
//
// Orchestration of PAPER.md §5.2 on B200s:
//   chunking -> per-GPU radix sort (§5.1, radix.cu) ->
//   g-1 merge stages of Alg.2: barrier, Alg.1 pivots of every
//   group (merge.cu), exchange + local merge of each mirrored GPU pair
//    -> result chunk i = global ranks
//   [i*c, (i+1)*c).
// Two execution modes share the plan and the kernels:
//   * single process (msort_create): one host thread drives g "ranks"; ranks
//     may be distinct GPUs (peer access over NVLink) or repeated devices
//     (virtual ranks on one GPU); cross-rank ordering by CUDA events;
//   * one process per GPU (msort_dist_*): peers' buffers are mapped with CUDA
//     IPC; cross-rank ordering by a device-side barrier on IPC-mapped flags.
// Every rank knows every pivot of every stage (each rank computes all of them
// from peer memory), so the buffer rotation of all ranks is replicated
// deterministically without extra messages.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <condition_variable>
#include <mutex>
#include <string>
#include <thread>

#include <unistd.h>
#include <tuple>
#include <vector>

#include "../../include/msort.h"
#include "kernels.h"
#include "nccl_shim.h"

using namespace msort;

namespace {

thread_local std::string g_last_error;

int set_error(int status, const std::string& msg) {
    g_last_error = msg;
    return status;
}

int cuda_status(cudaError_t e) {
    switch (e) {
        case cudaErrorMemoryAllocation: return MSORT_ERR_OUT_OF_MEMORY;
        case cudaErrorNoDevice:
        case cudaErrorInsufficientDriver:
        case cudaErrorInvalidDevice:
        case cudaErrorPeerAccessUnsupported: return MSORT_ERR_DEVICE;
        default: return MSORT_ERR_CUDA;
    }
}

#define CUDA_TRY(expr)                                                                                  \
    do {                                                                                                \
        cudaError_t e_ = (expr);                                                                        \
        if (e_ != cudaSuccess) {                                                                        \
            cudaGetLastError(); /* clear a non-sticky error (e.g. a failed allocation) for later calls */ \
            return set_error(cuda_status(e_), std::string(#expr) + " -> " + cudaGetErrorString(e_) +   \
                                                  " (" + __FILE__ + ":" + std::to_string(__LINE__) + ")"); \
        }                                                                                               \
    } while (0)

#define MSORT_TRY(expr)             \
    do {                            \
        int s_ = (expr);            \
        if (s_ != MSORT_OK) return s_; \
    } while (0)

bool valid_kt(int kt) { return kt >= 0 && kt <= 3; }
bool valid_g(int g) { return g == 1 || g == 2 || g == 4 || g == 8; }

// ---------------------------------------------------------------------------
// Plan (host only): Alg.2 stage labels, reading Q7.
// ---------------------------------------------------------------------------
void stage_labels(int g, std::vector<int>& out) {
    if (g < 2) return;
    if (g == 2) {
        out.push_back(2);
        return;
    }
    std::vector<int> half;
    stage_labels(g / 2, half);
    out.insert(out.end(), half.begin(), half.end());
    out.push_back(g);
    out.insert(out.end(), half.begin(), half.end());
}

struct Exchange {
    int partner[MSORT_MAX_GPUS];
    uint64_t x[MSORT_MAX_GPUS];
    int side[MSORT_MAX_GPUS];
};

// Reading Q6 (Fig.9).
void plan_exchange(int g, int label, uint64_t c, const uint64_t* pivots, Exchange& ex) {
    for (int r = 0; r < g; ++r) {
        ex.partner[r] = -1;
        ex.x[r] = 0;
        ex.side[r] = 0;
    }
    for (int j = 0; j < g / label; ++j) {
        const int lo = j * label, mid = lo + label / 2;
        const uint64_t p = pivots[j];
        for (int d = 0; d < label / 2; ++d) {
            const int L = mid - 1 - d, R = mid + d;
            const uint64_t dc = uint64_t(d) * c;
            const uint64_t x = p <= dc ? 0 : std::min<uint64_t>(p - dc, c);
            ex.partner[L] = R;
            ex.partner[R] = L;
            ex.x[L] = ex.x[R] = x;
            ex.side[L] = 0;
            ex.side[R] = 1;
        }
    }
}

uint64_t chunk_size(uint64_t n, int g) {
    const uint64_t c = (n + g - 1) / g;
    return (c + 3) / 4 * 4;  // reading Q3
}

// ---------------------------------------------------------------------------
// Per-rank state
// ---------------------------------------------------------------------------
constexpr int kPieces = 4;   // pipelined host sort: H2D pieces, each sorted while the next one arrives
constexpr int kSlices = 4;   // ... and final-merge slices, each copied back while the next one merges
constexpr uint32_t kEpochs = 512;  // radix tag cycle (RadixWs::epoch)

struct Rank {
    int dev = 0;
    cudaStream_t st = nullptr;
    void* buf[3] = {nullptr, nullptr, nullptr};  // B0, B1 (rotating chunk buffers), B2 (swap-mode receive)
    void* stage = nullptr;                       // chunk staging buffer for host / single-pointer sorts
    void* rws = nullptr;
    size_t rws_bytes = 0;
    void* mws = nullptr;
    size_t mws_bytes = 0;
    uint64_t* d_pivot = nullptr;   // [128] pivots (Alg.2) or splitters (all-to-all)
    uint64_t* h_pivot = nullptr;   // pinned [128]
    uint32_t* h_trivial = nullptr; // pinned [kTrivialWords]: trivial flags, largest bin, hot digits per pass
    DevStage* d_stage = nullptr;   // device-resident Alg.2 state (exchange mode 0): buffer rotation, pivots
    DevStage* h_stage = nullptr;   // pinned copy read after the sort (stage statistics)
    MergeDesc* d_desc = nullptr;   // this rank's exchange+merge of the current stage, resolved on the GPU
    int* d_err = nullptr;          // barrier timeout flag
    int* h_err = nullptr;          // pinned
    cudaEvent_t e_begin = nullptr, e_hist = nullptr, e_sorted = nullptr, e_end = nullptr;
    cudaEvent_t e_h2d0 = nullptr, e_h2d1 = nullptr, e_d2h0 = nullptr, e_d2h1 = nullptr;
    cudaEvent_t e_pass[8][2] = {};
    // pipelined host sort (g == 1): copy stream, piece arrivals, merged slices
    cudaStream_t cst = nullptr;
    cudaEvent_t e_piece[kPieces] = {};
    cudaEvent_t e_slice[kSlices] = {};
    cudaEvent_t e_merged = nullptr;
    // small one-GPU sorts (<= kGraphMaxKeys): the whole radix sort as one CUDA
    // graph, captured when the same (buffer, size) is sorted a second time
    cudaGraphExec_t small_exec = nullptr;
    const void* small_user = nullptr;
    uint64_t small_c = 0;
    int small_timing = -1;
    bool small_seen = false;
    cudaEvent_t e_sync[MSORT_MAX_STAGES + 1] = {};
    cudaEvent_t e_nccl[2] = {};  // exchange mode 4: ranks sharing a device hand their stream to one NCCL stream
    // pageable host memory (S0/S8): pinned bounce buffers, allocated on first use
    void* bounce[3] = {nullptr, nullptr, nullptr};
    cudaEvent_t e_bounce[3] = {};
    cudaEvent_t e_stage[MSORT_MAX_STAGES][2] = {};
    cudaEvent_t e_xch[MSORT_MAX_STAGES][2] = {};
    cudaEvent_t e_swp[MSORT_MAX_STAGES] = {};  // modes 1 / 4: end of the transfer (the merge follows)
    bool xch_rec[MSORT_MAX_STAGES] = {};  // e_xch[s] recorded in this sort
    // per sort
    void* user = nullptr;
    int cur = -1;  // -1: user buffer, 0..2: buf[]
    int passes_run = 0;
    int pass_ids[8] = {};
    // radix workspace epoch (RadixWs::epoch); starts so that the first sort
    // zeroes the whole workspace, and wraps to 0 (the whole allocation zeroed
    // again) every kEpochs sorts
    uint32_t radix_epoch = kEpochs - 1;

    void* ptr(int which) const { return which < 0 ? user : buf[which]; }
};

struct DeviceGuard {
    int prev = 0;
    DeviceGuard() { cudaGetDevice(&prev); }
    ~DeviceGuard() { cudaSetDevice(prev); }
};

}  // namespace

struct msort_ctx {
    int g = 1;
    int kt = 0;
    uint64_t cap = 0;  // keys per rank
    bool dist = false;
    int rank = 0;      // dist: this process's rank
    int nlocal = 1;    // ranks driven by this process
    Rank r[MSORT_MAX_GPUS];
    // dist mode: buffers and flags of every rank as seen from this process
    void* peer_buf[MSORT_MAX_GPUS][2] = {};
    unsigned long long* peer_flags[MSORT_MAX_GPUS] = {};
    unsigned long long* my_flags = nullptr;
    unsigned long long epoch = 0;
    bool imported = false;
    std::vector<void*> opened;
    // options
    int timing = 1;
    int exchange = 0;       // MSORT_OPT_EXCHANGE as requested
    int xmode = 0;          // as run: 0 / 2 fall back to 1 / 3 when bulk copies from peer memory failed the
                            // self-test (peer_bulk_ok)
    bool peer_bulk_ok = true;
    int skip_trivial = 1;
    int host_pipeline = 1;
    int small_graph = 1;
    bool stats_on_device = false;  // the sort's stage statistics are in r[0].h_stage (device-resident Alg.2)
    // exchange mode 4 (NCCL send/recv swap): single process - one comm per distinct device (ncclCommInitAll),
    // rank i uses comm nccl_comm[i] with comm rank nccl_rank[i]; dist - one comm of `g` ranks
    int stop_after = -1;  // testing (MSORT_OPT_STOP_AFTER_STAGE): end the Alg.2 merge phase after this stage
    NcclState nccl;
    int nccl_comm[MSORT_MAX_GPUS] = {};
    int nccl_rank[MSORT_MAX_GPUS] = {};
    msort_timings tm{};
};

namespace {

int stages_to_run(const msort_ctx* ctx, int S) {
    return ctx->stop_after >= 0 ? std::min(S, ctx->stop_after + 1) : S;
}

int alloc_rank(msort_ctx* ctx, Rank& R, bool need_b1, bool need_stage) {
    const size_t K = key_bytes(ctx->kt);
    CUDA_TRY(cudaSetDevice(R.dev));
    atomic_rank_ok(nullptr);  // one-time per-device probe, outside any sort
    CUDA_TRY(cudaStreamCreateWithFlags(&R.st, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&R.cst, cudaStreamNonBlocking));
    for (auto& e : R.e_piece) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto& e : R.e_slice) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreate(&R.e_merged));
    const size_t bytes = std::max<size_t>(ctx->cap * K, 256);
    CUDA_TRY(cudaMalloc(&R.buf[0], bytes));
    if (need_b1) CUDA_TRY(cudaMalloc(&R.buf[1], bytes));
    if (need_stage) CUDA_TRY(cudaMalloc(&R.stage, bytes));
    R.rws_bytes = radix_ws_bytes(ctx->cap, ctx->kt);
    CUDA_TRY(cudaMalloc(&R.rws, R.rws_bytes));
    R.mws_bytes = merge_ws_bytes(ctx->cap, ctx->kt);
    CUDA_TRY(cudaMalloc(&R.mws, R.mws_bytes));
    CUDA_TRY(cudaMalloc(&R.d_pivot, 128 * sizeof(uint64_t)));
    CUDA_TRY(cudaMalloc(&R.d_err, sizeof(int)));
    CUDA_TRY(cudaMemset(R.d_err, 0, sizeof(int)));
    CUDA_TRY(cudaMalloc(&R.d_stage, sizeof(DevStage)));
    CUDA_TRY(cudaMalloc(&R.d_desc, sizeof(MergeDesc)));
    CUDA_TRY(cudaMallocHost(&R.h_stage, sizeof(DevStage)));
    CUDA_TRY(cudaMallocHost(&R.h_pivot, 128 * sizeof(uint64_t)));
    CUDA_TRY(cudaMallocHost(&R.h_trivial, kTrivialWords * sizeof(uint32_t)));
    CUDA_TRY(cudaMallocHost(&R.h_err, sizeof(int)));
    *R.h_err = 0;
    cudaEvent_t* evs[] = {&R.e_begin, &R.e_hist, &R.e_sorted, &R.e_end, &R.e_h2d0, &R.e_h2d1, &R.e_d2h0, &R.e_d2h1};
    for (auto* e : evs) CUDA_TRY(cudaEventCreate(e));
    for (auto& pe : R.e_pass)
        for (auto& e : pe) CUDA_TRY(cudaEventCreate(&e));
    for (auto& e : R.e_sync) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto& e : R.e_nccl) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto& se : R.e_stage)
        for (auto& e : se) CUDA_TRY(cudaEventCreate(&e));
    for (auto& xe : R.e_xch)
        for (auto& e : xe) CUDA_TRY(cudaEventCreate(&e));
    for (auto& e : R.e_swp) CUDA_TRY(cudaEventCreate(&e));
    return MSORT_OK;
}

void free_rank(Rank& R) {
    if (!R.st) return;
    cudaSetDevice(R.dev);
    cudaStreamSynchronize(R.st);
    for (void* p : R.buf)
        if (p) cudaFree(p);
    if (R.stage) cudaFree(R.stage);
    if (R.rws) cudaFree(R.rws);
    if (R.mws) cudaFree(R.mws);
    if (R.d_pivot) cudaFree(R.d_pivot);
    if (R.d_err) cudaFree(R.d_err);
    if (R.d_stage) cudaFree(R.d_stage);
    if (R.d_desc) cudaFree(R.d_desc);
    if (R.h_stage) cudaFreeHost(R.h_stage);
    if (R.h_pivot) cudaFreeHost(R.h_pivot);
    if (R.h_trivial) cudaFreeHost(R.h_trivial);
    if (R.h_err) cudaFreeHost(R.h_err);
    cudaEvent_t evs[] = {R.e_begin, R.e_hist, R.e_sorted, R.e_end, R.e_h2d0, R.e_h2d1, R.e_d2h0, R.e_d2h1};
    for (auto e : evs)
        if (e) cudaEventDestroy(e);
    for (auto& pe : R.e_pass)
        for (auto e : pe)
            if (e) cudaEventDestroy(e);
    for (auto e : R.e_sync)
        if (e) cudaEventDestroy(e);
    for (auto e : R.e_nccl)
        if (e) cudaEventDestroy(e);
    for (auto& se : R.e_stage)
        for (auto e : se)
            if (e) cudaEventDestroy(e);
    for (auto& xe : R.e_xch)
        for (auto e : xe)
            if (e) cudaEventDestroy(e);
    for (auto e : R.e_swp)
        if (e) cudaEventDestroy(e);
    for (auto e : R.e_piece)
        if (e) cudaEventDestroy(e);
    for (auto e : R.e_slice)
        if (e) cudaEventDestroy(e);
    if (R.e_merged) cudaEventDestroy(R.e_merged);
    for (void* b : R.bounce)
        if (b) cudaFreeHost(b);
    for (auto e : R.e_bounce)
        if (e) cudaEventDestroy(e);
    if (R.small_exec) cudaGraphExecDestroy(R.small_exec);
    if (R.cst) {
        cudaStreamSynchronize(R.cst);
        cudaStreamDestroy(R.cst);
    }
    cudaStreamDestroy(R.st);
    R = Rank();
}

float elapsed(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return 0.f;
    }
    return ms;
}

// --- radix phase (S1-S3) -----------------------------------------------------

int radix_begin(msort_ctx* ctx, Rank& R, const void* src, uint64_t c) {
    CUDA_TRY(cudaSetDevice(R.dev));
    RadixWs ws = radix_ws_layout(R.rws, c, ctx->kt);
    R.radix_epoch = (R.radix_epoch + 1) % kEpochs;
    ws.epoch = R.radix_epoch;
    ws.alloc_bytes = R.rws_bytes;
    CUDA_TRY(radix_prologue(src, c, ctx->kt, ws, R.st));
    ctx->tm.kernel_launches += 2;
    if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_hist, R.st));
    if (ctx->skip_trivial) CUDA_TRY(cudaMemcpyAsync(R.h_trivial, ws.trivial, kTrivialWords * sizeof(uint32_t), cudaMemcpyDeviceToHost, R.st));
    return MSORT_OK;
}

// skewed-pass ranking (MSORT_SKEW_MODE, tuning only): 0 = peer match, 1 = one
// atomic per warp row for each of the 4 most frequent digit values, 2 (default)
// = 1 when one digit holds > 1/4 of the keys, else 0; 3 = plain atomic ranking
// (same-address lanes serialised) for every skewed pass
int skew_mode() {
    static int v = -1;
    if (v < 0) {
        const char* e = std::getenv("MSORT_SKEW_MODE");
        v = e ? std::atoi(e) : 2;
        if (v < 0 || v > 3) v = 2;
    }
    return v;
}

// src -> dst through tmp; an even number of executed passes, so the last write
// lands in dst and no pass reads and writes the same buffer.
int radix_passes(msort_ctx* ctx, Rank& R, const void* src, void* dst, void* tmp, uint64_t c) {
    CUDA_TRY(cudaSetDevice(R.dev));
    const int P = num_passes(ctx->kt);
    RadixWs ws = radix_ws_layout(R.rws, c, ctx->kt);
    ws.epoch = R.radix_epoch;
    bool run[8];
    int nrun = 0;
    for (int p = 0; p < P; ++p) {
        run[p] = !(ctx->skip_trivial && R.h_trivial[p]);
        nrun += run[p];
    }
    if (nrun % 2) {  // un-skip one trivial pass (an identity permutation) to keep the parity
        for (int p = 0; p < P; ++p)
            if (!run[p]) {
                run[p] = true;
                ++nrun;
                break;
            }
    }
    R.passes_run = 0;
    for (int p = 0; p < P; ++p)
        if (run[p]) R.pass_ids[R.passes_run++] = p;
    const int E = R.passes_run;
    if (E == 0) {
        if (src != dst) CUDA_TRY(cudaMemcpyAsync(dst, src, c * key_bytes(ctx->kt), cudaMemcpyDeviceToDevice, R.st));
        return MSORT_OK;
    }
    const void* in = src;
    for (int j = 0; j < E; ++j) {
        void* out = ((E - 1 - j) % 2 == 0) ? dst : tmp;
        // Ranking (flag 4 = one smem atomic per key): stable when the GPU passed
        // the lane-order self-test, and always valid for the first executed pass
        // (nothing has ordered the keys yet).  A skewed digit (one value holding
        // more than 1/16 of the keys) would make same-address atomics serialize:
        // its digit value goes to the kernel (flags bits 8.., value + 1), whose
        // lanes on that digit reserve their slots with one atomic per warp row
        // (host knows the histogram when skip_trivial synchronised on it).
        // Skewed passes (profiles/radix_tuning_r1.md): a dominant digit (largest
        // bin > 1/4 of the keys) -> the 4 most frequent digit values are ranked
        // with one atomic per warp row each (flag 8); moderate skew (zipf: ~100
        // elevated digits, the largest ~12%) -> peer match, which handles every
        // colliding digit.  MSORT_SKEW_MODE 0 / 1 forces peer match / flag 8.
        const int pid = R.pass_ids[j];
        const uint64_t maxbin = ctx->skip_trivial ? uint64_t(R.h_trivial[8 + pid]) : 0;
        const bool skewed = maxbin * 16 > c;
        const int mode = skew_mode();
        // (default: hot-4 when one digit holds > 1/4 of the keys or the 4 largest bins > 1/2 - e.g. the
        // exponent byte of floats; a long tail of elevated digits, as in zipf, ranks faster by peer match)
        const uint64_t top4 = ctx->skip_trivial ? uint64_t(R.h_trivial[24 + pid]) : 0;
        const bool dominant = mode == 1 ? skewed : (mode == 0 || mode == 3 ? false : maxbin * 4 > c || top4 * 2 > c);
        bool atomic_rank = j == 0 || atomic_rank_ok(R.st);
        if (skewed && !dominant && mode != 3) atomic_rank = false;  // peer match
        const bool hot = dominant && atomic_rank;
        const int flags = (j == 0 ? 1 : 0) | (j == E - 1 ? 2 : 0) | (atomic_rank ? 4 : 0) | (hot ? 8 : 0);
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_pass[j][0], R.st));
        CUDA_TRY(launch_onesweep(in, out, c, ctx->kt, pid, flags, ws, ws.base + pid * 256, R.st, R.h_trivial[16 + pid]));
        ctx->tm.kernel_launches += 1;
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_pass[j][1], R.st));
        in = out;
    }
    return MSORT_OK;
}

// --- merge phase (S4-S7) ------------------------------------------------------

// Launch this rank's exchange+merge for one stage. `own` is its current chunk,
// `peer` the partner's current chunk (peer pointer); returns the new cur index.
int launch_exchange(msort_ctx* ctx, Rank& R, int stage, bool last, uint64_t c, uint64_t x, int side, const void* own,
                    const void* peer, int& new_cur) {
    const size_t K = key_bytes(ctx->kt);
    const char* ownb = static_cast<const char*>(own);
    const char* peerb = static_cast<const char*>(peer);
    new_cur = R.cur;
    if (x == 0) return MSORT_OK;  // Alg.2 line 7 / reading Q8
    const int out_idx = last ? -1 : (R.cur == 0 ? 1 : 0);
    void* out = R.ptr(out_idx);
    // (mode 4 recorded the start before the NCCL swap)
    if (ctx->timing && ctx->xmode != 4) CUDA_TRY(cudaEventRecord(R.e_xch[stage][0], R.st));
    const bool swp = ctx->timing && (ctx->xmode == 1 || ctx->xmode == 4);
    if (x == c) {
        // the whole chunk moves: a pure P2P copy (one sorted run, reading Q8);
        // mode 4 received it into `out` already
        if (ctx->xmode != 4) CUDA_TRY(cudaMemcpyAsync(out, peer, c * K, cudaMemcpyDefault, R.st));
        if (swp) CUDA_TRY(cudaEventRecord(R.e_swp[stage], R.st));
    } else if (ctx->xmode == 4) {
        // NCCL swap done (nccl_stage_exchange): the partner's block is in B2
        if (swp) CUDA_TRY(cudaEventRecord(R.e_swp[stage], R.st));
        const char* recv = static_cast<const char*>(R.buf[2]);
        if (side == 0)
            CUDA_TRY(launch_merge(ownb, c - x, recv, x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
        else
            CUDA_TRY(launch_merge(recv, x, ownb + x * K, c - x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
    } else if (ctx->xmode == 0) {
        // fused: the merge kernel reads the partner's block over NVLink
        if (side == 0)
            CUDA_TRY(launch_merge(ownb, c - x, peerb, x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
        else
            CUDA_TRY(launch_merge(peerb + (c - x) * K, x, ownb + x * K, c - x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
    } else {
        // swap (P2P copy into the receive buffer), then local merge
        char* recv = static_cast<char*>(R.buf[2]);
        if (side == 0) {
            CUDA_TRY(cudaMemcpyAsync(recv, peerb, x * K, cudaMemcpyDefault, R.st));
            if (swp) CUDA_TRY(cudaEventRecord(R.e_swp[stage], R.st));
            CUDA_TRY(launch_merge(ownb, c - x, recv, x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
        } else {
            CUDA_TRY(cudaMemcpyAsync(recv, peerb + (c - x) * K, x * K, cudaMemcpyDefault, R.st));
            if (swp) CUDA_TRY(cudaEventRecord(R.e_swp[stage], R.st));
            CUDA_TRY(launch_merge(recv, x, ownb + x * K, c - x, out, ctx->kt, R.mws, R.st, &ctx->tm.kernel_launches));
        }
    }
    if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[stage][1], R.st));
    R.xch_rec[stage] = ctx->timing != 0;
    new_cur = out_idx;
    return MSORT_OK;
}

// --- exchange mode 4: the swap as NCCL send/recv (S5, north_star) -----------------

// Single process: one communicator per distinct device of the context
// (ncclCommInitAll); ranks sharing a device (virtual ranks) share its comm and
// exchange through NCCL's self send/recv.
int nccl_init_local(msort_ctx* ctx) {
    std::vector<int> devs;
    for (int i = 0; i < ctx->g; ++i) {
        const int d = ctx->r[i].dev;
        int idx = -1;
        for (int u = 0; u < int(devs.size()); ++u)
            if (devs[u] == d) idx = u;
        if (idx < 0) {
            idx = int(devs.size());
            devs.push_back(d);
        }
        ctx->nccl_comm[i] = idx;
        ctx->nccl_rank[i] = idx;
    }
    std::string err;
    DeviceGuard guard;
    if (!nccl_init_all(ctx->nccl, devs.data(), int(devs.size()), &err)) return set_error(MSORT_ERR_NCCL, err);
    return MSORT_OK;
}

// Post one stage's swap for the ranks this process drives: every rank with
// x != 0 sends its outgoing block (L: its last x keys, R: its first x keys,
// reading Q6) to its partner and receives the partner's block into its receive
// buffer B2 - or, when the whole chunk moves (x == c), straight into the
// buffer the stage writes.  Sends are posted in rank order, then the receives
// in the order of their senders, so matching pairs line up per comm pair.
// Ranks on one device run their NCCL calls on the first such rank's stream.
int nccl_stage_exchange(msort_ctx* ctx, const Exchange& ex, uint64_t c, bool last) {
    const size_t K = key_bytes(ctx->kt);
    const int nl = ctx->nlocal;
    auto me_of = [&](int i) { return ctx->dist ? ctx->rank : i; };
    auto lead_of = [&](int i) {
        for (int q = 0; q < nl; ++q)
            if (ctx->r[q].dev == ctx->r[i].dev) return q;
        return i;
    };
    // hand every rank's stream to its device's NCCL stream
    for (int i = 0; i < nl; ++i) {
        const int l = lead_of(i);
        if (l == i) continue;
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaEventRecord(ctx->r[i].e_nccl[0], ctx->r[i].st));
        CUDA_TRY(cudaStreamWaitEvent(ctx->r[l].st, ctx->r[i].e_nccl[0], 0));
    }
    std::vector<P2POp> ops;
    for (int i = 0; i < nl; ++i) {  // sends
        const int me = me_of(i);
        const uint64_t x = ex.x[me];
        if (x == 0) continue;
        const Rank& R = ctx->r[i];
        const char* own = static_cast<const char*>(R.ptr(R.cur));
        const int partner = ex.partner[me];
        const int peer_rank = ctx->dist ? partner : ctx->nccl_rank[partner];
        ops.push_back({true, own + (ex.side[me] == 0 ? (c - x) : 0) * K, x * K, peer_rank,
                       ctx->dist ? 0 : ctx->nccl_comm[i], ctx->r[lead_of(i)].st});
    }
    for (int sidx = 0; sidx < ctx->g; ++sidx) {  // receives, in the order of their senders
        const int recv_me = ex.partner[sidx];
        if (recv_me < 0 || ex.x[sidx] == 0) continue;
        int i = -1;  // local index of the receiving rank
        if (ctx->dist) {
            if (recv_me == ctx->rank) i = 0;
        } else {
            i = recv_me;
        }
        if (i < 0) continue;
        if (ctx->dist && ctx->rank != recv_me) continue;
        Rank& R = ctx->r[i];
        const uint64_t x = ex.x[recv_me];
        void* dst = x == c ? R.ptr(last ? -1 : (R.cur == 0 ? 1 : 0)) : R.buf[2];
        const int peer_rank = ctx->dist ? sidx : ctx->nccl_rank[sidx];
        ops.push_back({false, dst, x * K, peer_rank, ctx->dist ? 0 : ctx->nccl_comm[i], ctx->r[lead_of(i)].st});
    }
    std::string err;
    {
        DeviceGuard guard;
        if (!ops.empty() && !nccl_group(ctx->nccl, ops, &err)) return set_error(MSORT_ERR_NCCL, err);
    }
    for (int i = 0; i < nl; ++i) {
        const int l = lead_of(i);
        if (l == i) continue;
        CUDA_TRY(cudaSetDevice(ctx->r[l].dev));
        CUDA_TRY(cudaEventRecord(ctx->r[l].e_nccl[1], ctx->r[l].st));
        CUDA_TRY(cudaStreamWaitEvent(ctx->r[i].st, ctx->r[l].e_nccl[1], 0));
    }
    return MSORT_OK;
}

// --- pageable host memory (S0 / S8) -----------------------------------------------
// A copy from pageable memory makes the driver stage it through its own small
// pinned buffers one piece at a time (measured: 4e9 u32 keys, msort_sort on a
// numpy array 2.21 s vs 0.57 s pinned).  Pageable host keys go through a ring
// of pinned bounce buffers per GPU instead: host threads copy chunk k into a
// bounce buffer while the copy engine moves chunk k-1 (H2D), or the copy engine
// fills chunk k+1 while the threads drain chunk k (D2H), so PCIe stays busy.
constexpr size_t kBounceBytes = size_t(64) << 20;
constexpr int kBounce = 3;

class CopyPool {  // parallel memcpy on the host cores (persistent workers)
  public:
    static CopyPool& get() {
        // never destroyed (its detached workers wait on it until exit); a process forked after the
        // pool started has no workers, so it builds its own
        static std::mutex mu;
        static CopyPool* p = nullptr;
        static pid_t owner = 0;
        std::lock_guard<std::mutex> lk(mu);
        if (!p || owner != getpid()) {
            p = new CopyPool;
            owner = getpid();
        }
        return *p;
    }
    void copy(void* dst, const void* src, size_t bytes) {
        std::lock_guard<std::mutex> one(call_mu_);  // one copy at a time (contexts may live on several threads)
        const int parts = int(std::min<size_t>(workers_.size() + 1, std::max<size_t>(1, bytes >> 20)));
        if (parts <= 1) {
            std::memcpy(dst, src, bytes);
            return;
        }
        const size_t step = (bytes + parts - 1) / parts;
        {
            std::lock_guard<std::mutex> lk(mu_);
            dst_ = static_cast<char*>(dst);
            src_ = static_cast<const char*>(src);
            bytes_ = bytes;
            step_ = step;
            pending_ = parts - 1;
            jobs_ = parts - 1;
        }
        cv_.notify_all();
        std::memcpy(dst, src, std::min(step, bytes));  // the caller copies part 0
        std::unique_lock<std::mutex> lk(mu_);
        done_.wait(lk, [&] { return pending_ == 0; });
    }

  private:
    CopyPool() {
        const unsigned hw = std::thread::hardware_concurrency();
        const int n = int(std::min<unsigned>(15, hw > 1 ? hw - 1 : 1));
        for (int i = 0; i < n; ++i) workers_.emplace_back([this] { loop(); });
        for (auto& t : workers_) t.detach();  // (live for the process)
    }
    void loop() {
        for (;;) {
            std::unique_lock<std::mutex> lk(mu_);
            cv_.wait(lk, [&] { return jobs_ > 0; });
            const int part = jobs_--;  // parts P-1 .. 1 of the current copy
            char* d = dst_;
            const char* s = src_;
            const size_t step = step_, bytes = bytes_;
            lk.unlock();
            const size_t off = size_t(part) * step;
            if (off < bytes) std::memcpy(d + off, s + off, std::min(step, bytes - off));
            lk.lock();
            if (--pending_ == 0) done_.notify_all();
        }
    }
    std::vector<std::thread> workers_;
    std::mutex call_mu_, mu_;
    std::condition_variable cv_, done_;
    char* dst_ = nullptr;
    const char* src_ = nullptr;
    size_t bytes_ = 0, step_ = 0;
    int pending_ = 0, jobs_ = 0;
};

bool host_is_pageable(const void* p) {
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return true;
    }
    return a.type == cudaMemoryTypeUnregistered;
}

int bounce_alloc(Rank& R) {
    if (R.bounce[0]) return MSORT_OK;
    CUDA_TRY(cudaSetDevice(R.dev));
    for (int b = 0; b < kBounce; ++b) {
        CUDA_TRY(cudaMallocHost(&R.bounce[b], kBounceBytes));
        CUDA_TRY(cudaEventCreateWithFlags(&R.e_bounce[b], cudaEventDisableTiming));
    }
    return MSORT_OK;
}

// pageable host -> device through the bounce ring (returns when every chunk is queued)
int bounce_h2d(Rank& R, void* dst, const char* src, size_t bytes, cudaStream_t st) {
    MSORT_TRY(bounce_alloc(R));
    char* d = static_cast<char*>(dst);
    for (size_t off = 0, k = 0; off < bytes; off += kBounceBytes, ++k) {
        const int b = int(k % kBounce);
        const size_t len = std::min(kBounceBytes, bytes - off);
        // its last DMA is done (also one queued by an earlier call: the pipelined path stages piece by piece;
        // an event never recorded counts as complete)
        CUDA_TRY(cudaEventSynchronize(R.e_bounce[b]));
        CopyPool::get().copy(R.bounce[b], src + off, len);
        CUDA_TRY(cudaMemcpyAsync(d + off, R.bounce[b], len, cudaMemcpyHostToDevice, st));
        CUDA_TRY(cudaEventRecord(R.e_bounce[b], st));
    }
    return MSORT_OK;
}

// device -> pageable host through the bounce ring (returns when the data is in `dst`)
int bounce_d2h(Rank& R, char* dst, const void* src, size_t bytes, cudaStream_t st) {
    MSORT_TRY(bounce_alloc(R));
    const char* sp = static_cast<const char*>(src);
    const size_t nch = (bytes + kBounceBytes - 1) / kBounceBytes;
    auto issue = [&](size_t k) -> int {
        const int b = int(k % kBounce);
        const size_t off = k * kBounceBytes, len = std::min(kBounceBytes, bytes - off);
        CUDA_TRY(cudaMemcpyAsync(R.bounce[b], sp + off, len, cudaMemcpyDeviceToHost, st));
        CUDA_TRY(cudaEventRecord(R.e_bounce[b], st));
        return MSORT_OK;
    };
    for (size_t k = 0; k < std::min<size_t>(nch, kBounce); ++k) MSORT_TRY(issue(k));
    for (size_t k = 0; k < nch; ++k) {
        const int b = int(k % kBounce);
        const size_t off = k * kBounceBytes, len = std::min(kBounceBytes, bytes - off);
        CUDA_TRY(cudaEventSynchronize(R.e_bounce[b]));
        CopyPool::get().copy(dst + off, R.bounce[b], len);
        if (k + kBounce < nch) MSORT_TRY(issue(k + kBounce));
    }
    return MSORT_OK;
}

// --- exchange mode actually run ----------------------------------------------------

// The fused modes (0: Alg.2 merge reading the partner's block, 2: NEXT-1 merge
// reading the runs) move peer memory with TMA bulk copies (cp.async.bulk) in
// merge_pipe_kernel; if the self-test below found that this does not work
// between two of the context's GPUs, they fall back to the copy-engine modes
// 1 / 3 (peer copy into a local buffer, then a local merge).
int apply_exchange_mode(msort_ctx* ctx) {
    int m = ctx->exchange;
    if (!ctx->peer_bulk_ok) m = m == 0 ? 1 : (m == 2 ? 3 : m);
    if (m == 1 || m == 4)
        for (int i = 0; i < ctx->nlocal; ++i)
            if (!ctx->r[i].buf[2]) {
                CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
                CUDA_TRY(cudaMalloc(&ctx->r[i].buf[2], std::max<size_t>(ctx->cap * key_bytes(ctx->kt), 256)));
            }
    ctx->xmode = m;
    return MSORT_OK;
}

// Self-test of the fused exchange's access path: a merge on GPU `me` whose
// second run lives in a peer's buffer (read by cp.async.bulk through the peer
// mapping, starting one key past a 16-byte boundary) must equal the merge of
// the known patterns.  a: local even keys, b: peer odd keys.
constexpr uint32_t kSelfTestKeys = 4099;

void selftest_pattern(std::vector<uint32_t>& even, std::vector<uint32_t>& odd, uint32_t n) {
    even.resize(n);
    odd.resize(n);
    for (uint32_t k = 0; k < n; ++k) {
        even[k] = 2 * k;
        odd[k] = 2 * k + 1;
    }
}

// merge local even[0..n) with peer_odd[1..n) on rank R; true if the result is right
int selftest_merge(msort_ctx* ctx, Rank& R, const void* peer_odd, uint32_t n, bool* ok) {
    std::vector<uint32_t> even, odd, got(2 * n - 1);
    selftest_pattern(even, odd, n);
    CUDA_TRY(cudaSetDevice(R.dev));
    CUDA_TRY(cudaMemcpyAsync(R.stage, even.data(), n * 4, cudaMemcpyHostToDevice, R.st));
    CUDA_TRY(launch_merge(R.stage, n, static_cast<const uint32_t*>(peer_odd) + 1, n - 1, R.buf[1], 0, R.mws, R.st,
                          nullptr));
    CUDA_TRY(cudaMemcpyAsync(got.data(), R.buf[1], (2 * n - 1) * 4, cudaMemcpyDeviceToHost, R.st));
    CUDA_TRY(cudaStreamSynchronize(R.st));
    bool good = true;
    for (uint32_t k = 0; k < 2 * n - 1; ++k)  // expected: 0, 2, 3, 4, 5, ... (the odd 1 is skipped)
        good = good && got[k] == (k == 0 ? 0 : k + 1);
    *ok = good;
    return MSORT_OK;
}

int peer_bulk_selftest_local(msort_ctx* ctx) {
    const uint32_t n = kSelfTestKeys;
    if (ctx->cap < 2 * uint64_t(n)) return MSORT_OK;  // (tiny contexts: nothing to test with)
    std::vector<uint32_t> even, odd;
    selftest_pattern(even, odd, n);
    bool tested[MSORT_MAX_GPUS][MSORT_MAX_GPUS] = {};
    for (int i = 0; i < ctx->g; ++i)
        for (int j = 0; j < ctx->g; ++j) {
            Rank &A = ctx->r[i], &B = ctx->r[j];
            if (A.dev == B.dev || tested[i][j]) continue;
            for (int a = 0; a < ctx->g; ++a)
                for (int b = 0; b < ctx->g; ++b)
                    if (ctx->r[a].dev == A.dev && ctx->r[b].dev == B.dev) tested[a][b] = true;
            CUDA_TRY(cudaSetDevice(B.dev));
            CUDA_TRY(cudaMemcpy(B.buf[0], odd.data(), n * 4, cudaMemcpyHostToDevice));
            bool ok = false;
            const int st = selftest_merge(ctx, A, B.buf[0], n, &ok);
            if (st != MSORT_OK || !ok) ctx->peer_bulk_ok = false;
        }
    return MSORT_OK;
}

int check_c(msort_ctx* ctx, uint64_t c) {
    if (c > ctx->cap) return set_error(MSORT_ERR_INVALID_ARGUMENT, "keys per GPU exceed the context capacity");
    if (c >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "keys per GPU must be < 2^32");
    return MSORT_OK;
}

int sm_count_of(int dev) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
        cudaGetLastError();
        return 148;
    }
    return n > 0 ? n : 148;
}

void reset_timings(msort_ctx* ctx, uint64_t c) {
    ctx->stats_on_device = false;
    ctx->tm = msort_timings{};
    ctx->tm.exchange_mode = ctx->xmode;
    ctx->tm.peer_bulk_ok = ctx->peer_bulk_ok ? 1 : 0;
    ctx->tm.n_gpus = ctx->g;
    ctx->tm.keys_per_gpu = c;
    ctx->tm.passes_total = num_passes(ctx->kt);
}

// Single-process device-resident sort of r[i].user (c keys each).
// --- NEXT-1: one all-to-all exchange ----------------------------

// Runs received by rank j: run r = chunk r's keys [s[j][r], s[j+1][r]).
struct Runs {
    uint64_t off[MSORT_MAX_GPUS];
    uint64_t len[MSORT_MAX_GPUS];
};

Runs runs_of(const uint64_t* s, int g, int j) {
    Runs rr{};
    uint64_t o = 0;
    for (int r = 0; r < g; ++r) {
        rr.off[r] = o;
        rr.len[r] = s[(j + 1) * g + r] - s[j * g + r];
        o += rr.len[r];
    }
    return rr;
}

void record_alltoall_stats(msort_ctx* ctx, const uint64_t* s, int g) {
    uint64_t mx = 0, sum = 0;
    for (int j = 0; j < g; ++j) {
        const Runs rr = runs_of(s, g, j);
        uint64_t remote = 0;
        for (int r = 0; r < g; ++r)
            if (r != j) remote += rr.len[r];
        mx = std::max(mx, remote);
        sum += remote;
    }
    ctx->tm.n_stages = 1;
    ctx->tm.stage_label[0] = g;  // one stage over all g chunks
    ctx->tm.stage_max_x[0] = mx;
    ctx->tm.stage_keys_exchanged[0] = sum;
    for (int j = 0; j < g - 1 && j < MSORT_MAX_GPUS / 2; ++j) ctx->tm.stage_pivot[0][j] = 0;
}

// Multiway merge of the g runs sitting back to back in `src` into `dst_final`,
// as a tree of two-run merges (log2 g rounds) ping-ponging through `tmp`.
int merge_tree(msort_ctx* ctx, Rank& R, const Runs& runs, int g, char* src, char* tmp, char* dst_final) {
    const size_t K = key_bytes(ctx->kt);
    uint64_t off[MSORT_MAX_GPUS], len[MSORT_MAX_GPUS];
    int nr = g;
    for (int r = 0; r < g; ++r) {
        off[r] = runs.off[r];
        len[r] = runs.len[r];
    }
    char* in = src;
    char* out = tmp;
    while (nr > 1) {
        const bool last = nr == 2;
        char* o = last ? dst_final : out;
        int m = 0;
        for (int i = 0; i + 1 < nr; i += 2) {
            CUDA_TRY(launch_merge(in + off[i] * K, len[i], in + off[i + 1] * K, len[i + 1], o + off[i] * K, ctx->kt, R.mws,
                                  R.st, &ctx->tm.kernel_launches));
            off[m] = off[i];
            len[m] = len[i] + len[i + 1];
            ++m;
        }
        nr = m;
        in = o;
        out = (o == tmp) ? src : tmp;
    }
    return MSORT_OK;
}

// NEXT-1 fused (exchange mode 2): the first round of the merge tree reads the
// g runs straight from the peers' sorted chunks (B1) over NVLink, so pulled keys
// never make an HBM round trip.  Rounds alternate between d_user and B0 so that
// the last one lands in d_user and no round writes B1, which peers may still be
// reading (the caller orders the next use of B1 after every rank's merges).
int merge_tree_from_peers(msort_ctx* ctx, Rank& R, const Runs& runs, const char* const* run_ptr, int g, char* buf0,
                          char* d_user, bool time_first_round) {
    const size_t K = key_bytes(ctx->kt);
    int levels = 0;
    while ((1 << levels) < g) ++levels;
    uint64_t off[MSORT_MAX_GPUS], len[MSORT_MAX_GPUS];
    for (int r = 0; r < g; ++r) {
        off[r] = runs.off[r];
        len[r] = runs.len[r];
    }
    char* in = nullptr;
    for (int lv = 1, nr = g; lv <= levels; ++lv) {
        char* o = ((levels - lv) % 2 == 0) ? d_user : buf0;
        if (lv == 1 && time_first_round) CUDA_TRY(cudaEventRecord(R.e_xch[0][0], R.st));
        int m = 0;
        for (int i = 0; i + 1 < nr; i += 2) {
            const char* a = lv == 1 ? run_ptr[i] : in + off[i] * K;
            const char* b = lv == 1 ? run_ptr[i + 1] : in + off[i + 1] * K;
            CUDA_TRY(launch_merge(a, len[i], b, len[i + 1], o + off[i] * K, ctx->kt, R.mws, R.st,
                                  &ctx->tm.kernel_launches));
            off[m] = off[i];
            len[m] = len[i] + len[i + 1];
            ++m;
        }
        if (lv == 1 && time_first_round) {
            CUDA_TRY(cudaEventRecord(R.e_xch[0][1], R.st));
            R.xch_rec[0] = true;
        }
        nr = m;
        in = o;
    }
    return MSORT_OK;
}

int alltoall_local(msort_ctx* ctx, uint64_t c) {
    const int g = ctx->g;
    const size_t K = key_bytes(ctx->kt);
    // every rank's sorted chunk (B1) is complete before anyone reads it
    for (int i = 0; i < g; ++i) {
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaEventRecord(ctx->r[i].e_sync[0], ctx->r[i].st));
    }
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        for (int q = 0; q < g; ++q)
            if (q != i) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[0], 0));
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][0], R.st));
    }
    GroupPtrs all{};
    for (int i = 0; i < g; ++i) all.p[i] = ctx->r[i].buf[1];
    Rank& R0 = ctx->r[0];
    CUDA_TRY(cudaSetDevice(R0.dev));
    CUDA_TRY(launch_splitters(all, g, c, ctx->kt, R0.d_pivot, R0.st));
    ctx->tm.kernel_launches += 1;
    const size_t sbytes = size_t(g + 1) * g * sizeof(uint64_t);
    CUDA_TRY(cudaMemcpyAsync(R0.h_pivot, R0.d_pivot, sbytes, cudaMemcpyDeviceToHost, R0.st));
    CUDA_TRY(cudaStreamSynchronize(R0.st));
    std::vector<uint64_t> s(R0.h_pivot, R0.h_pivot + (g + 1) * g);
    record_alltoall_stats(ctx, s.data(), g);
    if (ctx->xmode == 2) {
        // fused: every rank merges its runs straight out of the peers' B1
        for (int j = 0; j < g; ++j) {
            Rank& R = ctx->r[j];
            CUDA_TRY(cudaSetDevice(R.dev));
            const Runs rr = runs_of(s.data(), g, j);
            const char* rp[MSORT_MAX_GPUS];
            for (int r = 0; r < g; ++r) rp[r] = static_cast<const char*>(ctx->r[r].buf[1]) + s[j * g + r] * K;
            MSORT_TRY(merge_tree_from_peers(ctx, R, rr, rp, g, static_cast<char*>(R.buf[0]),
                                            static_cast<char*>(R.user), ctx->timing != 0));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][1], R.st));
            CUDA_TRY(cudaEventRecord(R.e_sync[1], R.st));
        }
        // no rank's B1 is reused (next sort) before every rank finished reading it
        for (int j = 0; j < g; ++j) {
            Rank& R = ctx->r[j];
            CUDA_TRY(cudaSetDevice(R.dev));
            for (int q = 0; q < g; ++q)
                if (q != j) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[1], 0));
            R.cur = -1;
            CUDA_TRY(cudaEventRecord(R.e_end, R.st));
        }
        return MSORT_OK;
    }
    // the single exchange: rank j pulls its run from every chunk into B0
    for (int j = 0; j < g; ++j) {
        Rank& R = ctx->r[j];
        CUDA_TRY(cudaSetDevice(R.dev));
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[0][0], R.st));
        const Runs rr = runs_of(s.data(), g, j);
        for (int r = 0; r < g; ++r)
            if (rr.len[r])
                CUDA_TRY(cudaMemcpyAsync(static_cast<char*>(R.buf[0]) + rr.off[r] * K,
                                         static_cast<const char*>(ctx->r[r].buf[1]) + s[j * g + r] * K, rr.len[r] * K,
                                         cudaMemcpyDefault, R.st));
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[0][1], R.st));
        R.xch_rec[0] = ctx->timing != 0;
        CUDA_TRY(cudaEventRecord(R.e_sync[1], R.st));
    }
    // every pull is done before any B1 is overwritten by a merge round
    for (int j = 0; j < g; ++j) {
        Rank& R = ctx->r[j];
        CUDA_TRY(cudaSetDevice(R.dev));
        for (int q = 0; q < g; ++q)
            if (q != j) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[1], 0));
        MSORT_TRY(merge_tree(ctx, R, runs_of(s.data(), g, j), g, static_cast<char*>(R.buf[0]),
                             static_cast<char*>(R.buf[1]), static_cast<char*>(R.user)));
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][1], R.st));
        R.cur = -1;
        CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    }
    return MSORT_OK;
}

// Small sorts on one GPU (2^20 keys are L2-resident, so the
// sort is launch- and latency-bound).  The sequence of msort_radix_sort -
// workspace zeroing, histogram, scan, all P passes (a constant digit's pass is
// an identity permutation: no host round trip on the trivial flags; default
// ranking without the skew hints) - captured once as a CUDA graph and replayed
// while the caller sorts the same buffer and size again.  The first call with a
// new (buffer, size) runs the normal path and only remembers it.
static constexpr uint64_t kGraphMaxKeys = 1ull << 22;

int capture_small(msort_ctx* ctx, Rank& R, uint64_t c) {
    const int P = num_passes(ctx->kt);
    if (R.small_exec) {
        cudaGraphExecDestroy(R.small_exec);
        R.small_exec = nullptr;
    }
    cudaGraph_t graph = nullptr;
    CUDA_TRY(cudaStreamBeginCapture(R.st, cudaStreamCaptureModeThreadLocal));
    // timing events inside the graph are external records (recorded on every replay)
    auto rec = [&](cudaEvent_t e) { return cudaEventRecordWithFlags(e, R.st, cudaEventRecordExternal); };
    auto body = [&]() -> int {
        RadixWs ws = radix_ws_layout(R.rws, c, ctx->kt);
        ws.epoch = 0;  // every replay zeroes the (small) workspace: status tags repeat
        CUDA_TRY(radix_prologue(R.user, c, ctx->kt, ws, R.st));
        if (ctx->timing) CUDA_TRY(rec(R.e_hist));
        for (int p = 0; p < P; ++p) {
            const void* in = (p % 2 == 0) ? R.user : R.buf[0];
            void* out = (p % 2 == 0) ? R.buf[0] : R.user;
            const int flags = (p == 0 ? 1 : 0) | (p == P - 1 ? 2 : 0) | ((p == 0 || atomic_rank_ok(R.st)) ? 4 : 0);
            if (ctx->timing) CUDA_TRY(rec(R.e_pass[p][0]));
            CUDA_TRY(launch_onesweep(in, out, c, ctx->kt, p, flags, ws, ws.base + p * 256, R.st));
            if (ctx->timing) CUDA_TRY(rec(R.e_pass[p][1]));
        }
        return MSORT_OK;
    };
    const int st = body();
    const cudaError_t ce = cudaStreamEndCapture(R.st, &graph);
    if (st != MSORT_OK) {
        if (graph) cudaGraphDestroy(graph);
        return st;
    }
    CUDA_TRY(ce);
    const cudaError_t ie = cudaGraphInstantiate(&R.small_exec, graph, 0);
    cudaGraphDestroy(graph);
    CUDA_TRY(ie);
    R.small_user = R.user;
    R.small_c = c;
    R.small_timing = ctx->timing;
    return MSORT_OK;
}

// true if the sort ran as a graph replay
int sort_small_graph(msort_ctx* ctx, Rank& R, uint64_t c, bool* done) {
    *done = false;
    const bool same = R.small_user == R.user && R.small_c == c;
    if (!same) {  // remember; capture if it comes again
        if (R.small_exec) cudaGraphExecDestroy(R.small_exec);
        R.small_exec = nullptr;
        R.small_user = R.user;
        R.small_c = c;
        return MSORT_OK;
    }
    if (!R.small_exec || R.small_timing != ctx->timing) MSORT_TRY(capture_small(ctx, R, c));
    CUDA_TRY(cudaEventRecord(R.e_begin, R.st));
    CUDA_TRY(cudaGraphLaunch(R.small_exec, R.st));
    CUDA_TRY(cudaEventRecord(R.e_sorted, R.st));
    CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    ctx->tm.kernel_launches += 2 + num_passes(ctx->kt);
    R.passes_run = num_passes(ctx->kt);
    R.cur = -1;
    *done = true;
    return MSORT_OK;
}

// Alg.2 merge phase with every decision on the GPUs (exchange mode 0): per
// stage an event barrier across the ranks' streams, then on every rank the
// pivots of all groups (Alg.1), this rank's fused exchange+merge resolved from
// them, and the buffer rotation of all ranks - no host round trip until the
// sort ends.  Ranks start from B1 (the radix output, R.cur == 1).
int alg2_device_local(msort_ctx* ctx, uint64_t c) {
    const int g = ctx->g;
    std::vector<int> labels;
    stage_labels(g, labels);
    const int S = int(labels.size());
    BufTable bt{};
    for (int q = 0; q < g; ++q) {
        bt.p[q][0] = ctx->r[q].user;
        bt.p[q][1] = ctx->r[q].buf[0];
        bt.p[q][2] = ctx->r[q].buf[1];
    }
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        CUDA_TRY(launch_stage_init(R.d_stage, g, R.st));
        ctx->tm.kernel_launches += 1;
    }
    const int S_run = stages_to_run(ctx, S);
    ctx->tm.n_stages = S_run;
    for (int s = 0; s < S_run; ++s) {
        const int label = labels[s];
        const bool last = s == S - 1;
        // barrier: every rank's stream waits for every other rank's previous stage
        for (int i = 0; i < g; ++i) {
            CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
            CUDA_TRY(cudaEventRecord(ctx->r[i].e_sync[s], ctx->r[i].st));
        }
        for (int i = 0; i < g; ++i) {
            Rank& R = ctx->r[i];
            CUDA_TRY(cudaSetDevice(R.dev));
            for (int q = 0; q < g; ++q)
                if (q != i) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[s], 0));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][0], R.st));
            CUDA_TRY(launch_stage_pivots(bt, R.d_stage, s, label, g, c, ctx->kt, R.st));
            ctx->tm.kernel_launches += 1;
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[s][0], R.st));
            CUDA_TRY(launch_stage_merge(bt, R.d_stage, R.d_desc, s, label, i, g, c, last, ctx->kt, R.mws, R.st,
                                        &ctx->tm.kernel_launches));
            if (ctx->timing) {
                CUDA_TRY(cudaEventRecord(R.e_xch[s][1], R.st));
                R.xch_rec[s] = true;
                CUDA_TRY(cudaEventRecord(R.e_stage[s][1], R.st));
            }
        }
    }
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        CUDA_TRY(launch_stage_final(bt, R.d_stage, i, c, ctx->kt, R.st, sm_count_of(R.dev)));
        ctx->tm.kernel_launches += 1;
        if (i == 0) CUDA_TRY(cudaMemcpyAsync(R.h_stage, R.d_stage, sizeof(DevStage), cudaMemcpyDeviceToHost, R.st));
        R.cur = -1;
        CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    }
    ctx->stats_on_device = true;
    return MSORT_OK;
}

int sort_device_local(msort_ctx* ctx, uint64_t c) {
    const int g = ctx->g;
    if (g == 1 && c <= kGraphMaxKeys && ctx->small_graph) {
        bool done = false;
        MSORT_TRY(sort_small_graph(ctx, ctx->r[0], c, &done));
        if (done) return MSORT_OK;
    }
    std::vector<int> labels;
    stage_labels(g, labels);
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        CUDA_TRY(cudaEventRecord(R.e_begin, R.st));
        R.cur = -1;
        MSORT_TRY(radix_begin(ctx, R, R.user, c));
    }
    if (ctx->skip_trivial)
        for (int i = 0; i < g; ++i) CUDA_TRY(cudaStreamSynchronize(ctx->r[i].st));
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        if (g == 1) {
            MSORT_TRY(radix_passes(ctx, R, R.user, R.user, R.buf[0], c));
            R.cur = -1;
        } else {
            MSORT_TRY(radix_passes(ctx, R, R.user, R.buf[1], R.buf[0], c));
            R.cur = 1;
        }
        CUDA_TRY(cudaEventRecord(R.e_sorted, R.st));
    }
    if (g > 1 && (ctx->xmode == 2 || ctx->xmode == 3)) return alltoall_local(ctx, c);
    if (g > 1 && ctx->xmode == 0) return alg2_device_local(ctx, c);
    const int S = int(labels.size());
    const int S_run = stages_to_run(ctx, S);
    ctx->tm.n_stages = S_run;
    for (int s = 0; s < S_run; ++s) {
        const int label = labels[s];
        const bool last = s == S - 1;
        // barrier: every rank's stream waits for every other rank's previous stage
        for (int i = 0; i < g; ++i) {
            CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
            CUDA_TRY(cudaEventRecord(ctx->r[i].e_sync[s], ctx->r[i].st));
        }
        for (int i = 0; i < g; ++i) {
            Rank& R = ctx->r[i];
            CUDA_TRY(cudaSetDevice(R.dev));
            for (int q = 0; q < g; ++q)
                if (q != i) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[s], 0));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][0], R.st));
        }
        // S4: all pivots of the stage in one launch on rank 0 (peer reads)
        GroupPtrs all{};
        for (int i = 0; i < g; ++i) all.p[i] = ctx->r[i].ptr(ctx->r[i].cur);
        Rank& R0 = ctx->r[0];
        CUDA_TRY(cudaSetDevice(R0.dev));
        const int ngroups = g / label;
        CUDA_TRY(launch_pivots(all, ngroups, label, c, ctx->kt, R0.d_pivot, R0.st));
        ctx->tm.kernel_launches += 1;
        CUDA_TRY(cudaMemcpyAsync(R0.h_pivot, R0.d_pivot, ngroups * sizeof(uint64_t), cudaMemcpyDeviceToHost, R0.st));
        CUDA_TRY(cudaStreamSynchronize(R0.st));
        uint64_t piv[MSORT_MAX_GPUS / 2] = {};
        for (int j = 0; j < ngroups; ++j) piv[j] = R0.h_pivot[j];
        Exchange ex;
        plan_exchange(g, label, c, piv, ex);
        ctx->tm.stage_label[s] = label;
        for (int j = 0; j < ngroups; ++j) ctx->tm.stage_pivot[s][j] = piv[j];
        uint64_t mx = 0, sum = 0;
        for (int i = 0; i < g; ++i) {
            mx = std::max(mx, ex.x[i]);
            if (ex.side[i] == 0) sum += ex.x[i];
        }
        ctx->tm.stage_max_x[s] = mx;
        ctx->tm.stage_keys_exchanged[s] = sum;
        if (ctx->xmode == 4) {  // S5 as NCCL send/recv, then S6 below
            for (int i = 0; i < g; ++i)
                if (ctx->timing && ex.x[i]) {
                    CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
                    CUDA_TRY(cudaEventRecord(ctx->r[i].e_xch[s][0], ctx->r[i].st));
                }
            MSORT_TRY(nccl_stage_exchange(ctx, ex, c, last));
        }
        // S5+S6 on every rank
        int new_cur[MSORT_MAX_GPUS];
        for (int i = 0; i < g; ++i) {
            Rank& R = ctx->r[i];
            CUDA_TRY(cudaSetDevice(R.dev));
            const void* own = R.ptr(R.cur);
            const void* peer = ex.partner[i] >= 0 ? ctx->r[ex.partner[i]].ptr(ctx->r[ex.partner[i]].cur) : nullptr;
            MSORT_TRY(launch_exchange(ctx, R, s, last, c, ex.x[i], ex.side[i], own, peer, new_cur[i]));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][1], R.st));
        }
        for (int i = 0; i < g; ++i) ctx->r[i].cur = new_cur[i];
    }
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        if (R.cur != -1)
            CUDA_TRY(cudaMemcpyAsync(R.user, R.ptr(R.cur), c * key_bytes(ctx->kt), cudaMemcpyDeviceToDevice, R.st));
        CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    }
    return MSORT_OK;
}

// Stage statistics of a device-resident Alg.2 merge phase from the pivots the
// GPUs computed (h_stage, copied back with the sort's last D2H).
void stage_stats_from_device(msort_ctx* ctx, const DevStage& ds, uint64_t c) {
    std::vector<int> labels;
    stage_labels(ctx->g, labels);
    const int S = stages_to_run(ctx, int(labels.size()));
    ctx->tm.n_stages = S;
    for (int s = 0; s < S; ++s) {
        const int label = labels[s], ngroups = ctx->g / label;
        uint64_t piv[MSORT_MAX_GPUS / 2] = {};
        for (int j = 0; j < ngroups; ++j) piv[j] = ds.piv[s][j];
        Exchange ex;
        plan_exchange(ctx->g, label, c, piv, ex);
        ctx->tm.stage_label[s] = label;
        uint64_t mx = 0, sum = 0;
        for (int j = 0; j < ngroups; ++j) ctx->tm.stage_pivot[s][j] = piv[j];
        for (int q = 0; q < ctx->g; ++q) {
            mx = std::max(mx, ex.x[q]);
            if (ex.side[q] == 0) sum += ex.x[q];
        }
        ctx->tm.stage_max_x[s] = mx;
        ctx->tm.stage_keys_exchanged[s] = sum;
    }
}

// Fill timings after all events completed.
void collect_timings(msort_ctx* ctx, int nranks, const uint64_t* xs_by_stage_rank = nullptr) {
    (void)xs_by_stage_rank;
    msort_timings& t = ctx->tm;
    for (int i = 0; i < nranks; ++i) {
        Rank& R = ctx->r[i];
        cudaSetDevice(R.dev);
        t.sort_ms = std::max(t.sort_ms, double(elapsed(R.e_begin, R.e_sorted)));
        t.merge_ms = std::max(t.merge_ms, double(elapsed(R.e_sorted, R.e_end)));
        if (ctx->timing) {
            t.hist_ms = std::max(t.hist_ms, double(elapsed(R.e_begin, R.e_hist)));
            double ps = 0;
            for (int j = 0; j < R.passes_run; ++j) ps += elapsed(R.e_pass[j][0], R.e_pass[j][1]);
            t.pass_ms_sum = std::max(t.pass_ms_sum, ps);
            for (int s = 0; s < t.n_stages; ++s) {
                t.stage_ms[s] = std::max(t.stage_ms[s], double(elapsed(R.e_stage[s][0], R.e_stage[s][1])));
            }
        }
        t.passes_run = std::max(t.passes_run, R.passes_run);
    }
}

// exchange timings need to know which ranks recorded e_xch in which stage
struct XchLog {
    bool rec[MSORT_MAX_STAGES][MSORT_MAX_GPUS] = {};
};

std::mutex g_cache_mu;
std::map<std::tuple<int, int, int>, msort_ctx*> g_cache;  // (g, first device, kt) -> ctx

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

const char* msort_status_string(int status) {
    switch (status) {
        case MSORT_OK: return "MSORT_OK";
        case MSORT_ERR_INVALID_ARGUMENT: return "MSORT_ERR_INVALID_ARGUMENT";
        case MSORT_ERR_DEVICE: return "MSORT_ERR_DEVICE";
        case MSORT_ERR_OUT_OF_MEMORY: return "MSORT_ERR_OUT_OF_MEMORY";
        case MSORT_ERR_CUDA: return "MSORT_ERR_CUDA";
        case MSORT_ERR_NCCL: return "MSORT_ERR_NCCL";
        case MSORT_ERR_INTERNAL: return "MSORT_ERR_INTERNAL";
        case MSORT_ERR_TIMEOUT: return "MSORT_ERR_TIMEOUT";
        default: return "MSORT_ERR_UNKNOWN";
    }
}

const char* msort_last_error(void) { return g_last_error.c_str(); }

int msort_version(void) { return 100; }

int msort_rank_mode(int device) {
    int prev = 0;
    if (cudaGetDevice(&prev) != cudaSuccess || cudaSetDevice(device) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    const int r = atomic_rank_ok(nullptr) ? 1 : 0;
    cudaSetDevice(prev);
    return r;
}

// --- plan ---------------------------------------------------------------------

int msort_plan_num_stages(int g) {
    if (!valid_g(g) && g != 16) return -1;
    return g - 1;
}

int msort_plan_stage(int g, int s, int* label) {
    if ((!valid_g(g) && g != 16) || !label) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad g or label");
    std::vector<int> labels;
    stage_labels(g, labels);
    if (s < 0 || s >= int(labels.size())) return set_error(MSORT_ERR_INVALID_ARGUMENT, "stage out of range");
    *label = labels[s];
    return MSORT_OK;
}

int msort_plan_exchange(int g, int s, uint64_t c, const uint64_t* pivots, int* partner, uint64_t* x, int* side) {
    int label = 0;
    if (g > MSORT_MAX_GPUS) return set_error(MSORT_ERR_INVALID_ARGUMENT, "g > 8");
    MSORT_TRY(msort_plan_stage(g, s, &label));
    if (!pivots || !partner || !x || !side) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL output");
    Exchange ex;
    plan_exchange(g, label, c, pivots, ex);
    for (int r = 0; r < g; ++r) {
        partner[r] = ex.partner[r];
        x[r] = ex.x[r];
        side[r] = ex.side[r];
    }
    return MSORT_OK;
}

// --- step-level ---------------------------------------------------------------

uint64_t msort_radix_workspace_bytes(uint64_t n, int key_type) {
    if (!valid_kt(key_type)) return 0;
    return radix_ws_bytes(n, key_type);
}

int msort_step_histogram(const void* d_keys, uint64_t n, int key_type, uint32_t* d_hist, void* stream) {
    if (!valid_kt(key_type) || !d_hist || (n && !d_keys)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    if (n >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "n must be < 2^32");
    CUDA_TRY(launch_histogram(d_keys, n, key_type, d_hist, static_cast<cudaStream_t>(stream)));
    return MSORT_OK;
}

int msort_step_radix_pass(const void* d_in, void* d_out, uint64_t n, int key_type, int pass, const uint32_t* d_hist,
                          int flags, void* d_ws, uint64_t ws_bytes, void* stream) {
    if (!valid_kt(key_type) || pass < 0 || pass >= num_passes(key_type) || !d_hist || (n && (!d_in || !d_out)))
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    if (n >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "n must be < 2^32");
    if (d_in == d_out) return set_error(MSORT_ERR_INVALID_ARGUMENT, "a pass is out of place");
    if (ws_bytes < radix_ws_bytes(n, key_type) || !d_ws) return set_error(MSORT_ERR_INVALID_ARGUMENT, "workspace too small");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    RadixWs ws = radix_ws_layout(d_ws, n, key_type);
    CUDA_TRY(cudaMemsetAsync(ws.counters, 0, ws.zero_bytes, st));
    CUDA_TRY(launch_scan(d_hist, ws.base, ws.trivial, n, key_type, st));
    CUDA_TRY(launch_onesweep(d_in, d_out, n, key_type, pass, (flags & 3) | (atomic_rank_ok(st) ? 4 : 0), ws,
                             ws.base + pass * 256, st));
    return MSORT_OK;
}

int msort_radix_sort(void* d_keys, void* d_aux, uint64_t n, int key_type, void* d_ws, uint64_t ws_bytes, void* stream) {
    if (!valid_kt(key_type) || (n && (!d_keys || !d_aux))) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    if (n >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "n must be < 2^32");
    if (n <= 1) return MSORT_OK;
    if (ws_bytes < radix_ws_bytes(n, key_type) || !d_ws) return set_error(MSORT_ERR_INVALID_ARGUMENT, "workspace too small");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    RadixWs ws = radix_ws_layout(d_ws, n, key_type);
    CUDA_TRY(radix_prologue(d_keys, n, key_type, ws, st));
    const int P = num_passes(key_type);
    for (int p = 0; p < P; ++p) {
        const void* in = (p % 2 == 0) ? d_keys : d_aux;
        void* out = (p % 2 == 0) ? d_aux : d_keys;
        const int flags = (p == 0 ? 1 : 0) | (p == P - 1 ? 2 : 0) | ((p == 0 || atomic_rank_ok(st)) ? 4 : 0);
        CUDA_TRY(launch_onesweep(in, out, n, key_type, p, flags, ws, ws.base + p * 256, st));
    }
    return MSORT_OK;
}

int msort_step_pivot(const void* const* d_chunks, int n_chunks, uint64_t c, int key_type, uint64_t* d_pivot,
                     void* stream) {
    if (!valid_kt(key_type) || !d_chunks || !d_pivot || n_chunks < 2 || n_chunks > MSORT_MAX_GPUS || n_chunks % 2)
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    GroupPtrs all{};
    for (int i = 0; i < n_chunks; ++i) all.p[i] = d_chunks[i];
    if (c == 0) {
        CUDA_TRY(cudaMemsetAsync(d_pivot, 0, 8, static_cast<cudaStream_t>(stream)));
        return MSORT_OK;
    }
    CUDA_TRY(launch_pivots(all, 1, n_chunks, c, key_type, d_pivot, static_cast<cudaStream_t>(stream)));
    return MSORT_OK;
}

int msort_step_splitters(const void* const* d_chunks, int n_chunks, uint64_t c, int key_type, uint64_t* d_s,
                         void* stream) {
    if (!valid_kt(key_type) || !d_chunks || !d_s || n_chunks < 2 || n_chunks > MSORT_MAX_GPUS)
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    GroupPtrs all{};
    for (int i = 0; i < n_chunks; ++i) all.p[i] = d_chunks[i];
    CUDA_TRY(launch_splitters(all, n_chunks, c, key_type, d_s, static_cast<cudaStream_t>(stream)));
    return MSORT_OK;
}

uint64_t msort_merge_workspace_bytes(uint64_t total, int key_type) {
    if (!valid_kt(key_type)) return 0;
    return merge_ws_bytes(total, key_type);
}

int msort_step_merge(const void* d_a, uint64_t a_len, const void* d_b, uint64_t b_len, void* d_out, int key_type,
                     void* d_ws, uint64_t ws_bytes, void* stream) {
    if (!valid_kt(key_type) || (a_len && !d_a) || (b_len && !d_b) || (a_len + b_len && !d_out))
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    if (ws_bytes < merge_ws_bytes(a_len + b_len, key_type) || !d_ws)
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "workspace too small");
    CUDA_TRY(launch_merge(d_a, a_len, d_b, b_len, d_out, key_type, d_ws, static_cast<cudaStream_t>(stream), nullptr));
    return MSORT_OK;
}

// --- context ------------------------------------------------------------------

int msort_create(msort_ctx** out, int n_gpus, const int* device_ids, uint64_t max_keys, int key_type) {
    if (!out || !valid_g(n_gpus) || !valid_kt(key_type)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_error(MSORT_ERR_DEVICE, "no CUDA device");
    }
    DeviceGuard guard;
    auto ctx = std::make_unique<msort_ctx>();
    ctx->g = n_gpus;
    ctx->kt = key_type;
    ctx->nlocal = n_gpus;
    ctx->cap = chunk_size(std::max<uint64_t>(max_keys, 4), n_gpus);
    if (ctx->cap >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "keys per GPU must be < 2^32");
    for (int i = 0; i < n_gpus; ++i) {
        const int d = device_ids ? device_ids[i] : i;
        if (d < 0 || d >= ndev) return set_error(MSORT_ERR_DEVICE, "device id out of range / too few GPUs");
        ctx->r[i].dev = d;
    }
    // peer access between distinct devices (P2P reads and copies over NVLink)
    for (int i = 0; i < n_gpus; ++i)
        for (int j = 0; j < n_gpus; ++j) {
            const int a = ctx->r[i].dev, b = ctx->r[j].dev;
            if (a == b) continue;
            int can = 0;
            CUDA_TRY(cudaDeviceCanAccessPeer(&can, a, b));
            if (!can) return set_error(MSORT_ERR_DEVICE, "no peer access between GPUs");
            CUDA_TRY(cudaSetDevice(a));
            cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
            if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
            else if (e != cudaSuccess) return set_error(MSORT_ERR_DEVICE, cudaGetErrorString(e));
        }
    for (int i = 0; i < n_gpus; ++i) {
        int s = alloc_rank(ctx.get(), ctx->r[i], n_gpus > 1, true);
        if (s != MSORT_OK) {
            for (int j = 0; j <= i; ++j) free_rank(ctx->r[j]);
            return s;
        }
    }
    if (n_gpus > 1) {
        int s = peer_bulk_selftest_local(ctx.get());
        if (s == MSORT_OK) s = apply_exchange_mode(ctx.get());
        if (s != MSORT_OK) {
            for (int j = 0; j < n_gpus; ++j) free_rank(ctx->r[j]);
            return s;
        }
    }
    *out = ctx.release();
    return MSORT_OK;
}

int msort_destroy(msort_ctx* ctx) {
    if (!ctx) return MSORT_OK;
    DeviceGuard guard;
    if (ctx->dist) {
        cudaSetDevice(ctx->r[0].dev);
        for (void* p : ctx->opened) cudaIpcCloseMemHandle(p);
        if (ctx->my_flags) cudaFree(ctx->my_flags);
    }
    nccl_destroy(ctx->nccl);
    for (int i = 0; i < ctx->nlocal; ++i) free_rank(ctx->r[i]);
    delete ctx;
    return MSORT_OK;
}

int msort_set_option(msort_ctx* ctx, int option, int64_t value) {
    if (!ctx) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL ctx");
    DeviceGuard guard;
    switch (option) {
        case MSORT_OPT_TIMING: ctx->timing = value ? 1 : 0; return MSORT_OK;
        case MSORT_OPT_SKIP_TRIVIAL: ctx->skip_trivial = value ? 1 : 0; return MSORT_OK;
        case MSORT_OPT_HOST_PIPELINE: ctx->host_pipeline = value ? 1 : 0; return MSORT_OK;
        case MSORT_OPT_SMALL_GRAPH: ctx->small_graph = value ? 1 : 0; return MSORT_OK;
        case MSORT_OPT_STOP_AFTER_STAGE:  // testing: -1 = run every stage
            ctx->stop_after = value < 0 ? -1 : int(std::min<int64_t>(value, MSORT_MAX_STAGES));
            return MSORT_OK;
        case MSORT_OPT_RADIX_EPOCH:  // testing: the next sort runs at epoch value + 1 (mod the tag cycle)
            if (value < 0 || value >= int64_t(kEpochs)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "epoch 0..511");
            for (int i = 0; i < ctx->nlocal; ++i) ctx->r[i].radix_epoch = uint32_t(value);
            return MSORT_OK;
        case MSORT_OPT_EXCHANGE:
            if (value < 0 || value > 4) return set_error(MSORT_ERR_INVALID_ARGUMENT, "exchange mode 0..4");
            if (value == 1 || value == 4)  // a receive buffer per rank
                for (int i = 0; i < ctx->nlocal; ++i)
                    if (!ctx->r[i].buf[2]) {
                        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
                        CUDA_TRY(cudaMalloc(&ctx->r[i].buf[2], std::max<size_t>(ctx->cap * key_bytes(ctx->kt), 256)));
                    }
            if (value == 4 && !ctx->dist && ctx->nccl.comms.empty()) MSORT_TRY(nccl_init_local(ctx));
            ctx->exchange = int(value);
            return apply_exchange_mode(ctx);
        default: return set_error(MSORT_ERR_INVALID_ARGUMENT, "unknown option");
    }
}

int msort_get_timings(const msort_ctx* ctx, msort_timings* out) {
    if (!ctx || !out) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL argument");
    *out = ctx->tm;
    return MSORT_OK;
}

static int finish_local(msort_ctx* ctx) {
    for (int i = 0; i < ctx->g; ++i) {
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaEventSynchronize(ctx->r[i].e_end));
    }
    return MSORT_OK;
}

static void collect_exchange_timings(msort_ctx* ctx) {
    if (!ctx->timing) return;
    // e_xch events are recorded only on ranks that exchanged in that stage
    for (int s = 0; s < ctx->tm.n_stages; ++s) {
        double mx = 0, sw = 0, pv = 0;
        for (int i = 0; i < ctx->nlocal; ++i) {
            Rank& R = ctx->r[i];
            if (!R.xch_rec[s]) continue;
            cudaSetDevice(R.dev);
            mx = std::max(mx, double(elapsed(R.e_xch[s][0], R.e_xch[s][1])));
            pv = std::max(pv, double(elapsed(R.e_stage[s][0], R.e_xch[s][0])));
            if (ctx->xmode == 1 || ctx->xmode == 4)
                sw = std::max(sw, double(elapsed(R.e_xch[s][0], R.e_swp[s])));
        }
        ctx->tm.stage_exchange_ms[s] = mx;
        ctx->tm.stage_pivot_ms[s] = pv;
        // the transfer alone: separate in modes 1 / 4, the same as the exchange when fused (modes 0, 2)
        ctx->tm.stage_swap_ms[s] = (ctx->xmode == 1 || ctx->xmode == 4) ? sw : mx;
    }
}

int msort_sort_device(msort_ctx* ctx, void* const* chunks, uint64_t keys_per_gpu, void* const* streams) {
    if (!ctx || ctx->dist) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL or dist ctx");
    if (keys_per_gpu && !chunks) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL chunks");
    MSORT_TRY(check_c(ctx, keys_per_gpu));
    if (keys_per_gpu == 0 || (ctx->g == 1 && keys_per_gpu <= 1)) return MSORT_OK;
    DeviceGuard guard;
    reset_timings(ctx, keys_per_gpu);
    // re-create per-sort exchange events so stale records never alias
    for (int i = 0; i < ctx->g; ++i) {
        if (!chunks[i]) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL chunk");
        Rank& R = ctx->r[i];
        R.user = chunks[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        for (bool& b : R.xch_rec) b = false;
        // order the sort after the caller's stream, or after the legacy default
        // stream when none is given (the context's streams are non-blocking)
        cudaStream_t us = (streams && streams[i]) ? static_cast<cudaStream_t>(streams[i]) : cudaStreamLegacy;
        CUDA_TRY(cudaEventRecord(R.e_sync[MSORT_MAX_STAGES], us));
        CUDA_TRY(cudaStreamWaitEvent(R.st, R.e_sync[MSORT_MAX_STAGES], 0));
    }
    MSORT_TRY(sort_device_local(ctx, keys_per_gpu));
    for (int i = 0; i < ctx->g; ++i)
        if (streams && streams[i]) {
            CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
            CUDA_TRY(cudaStreamWaitEvent(static_cast<cudaStream_t>(streams[i]), ctx->r[i].e_end, 0));
        }
    MSORT_TRY(finish_local(ctx));
    if (ctx->stats_on_device) stage_stats_from_device(ctx, *ctx->r[0].h_stage, keys_per_gpu);
    collect_timings(ctx, ctx->g);
    collect_exchange_timings(ctx);
    ctx->tm.total_ms = ctx->tm.sort_ms + ctx->tm.merge_ms;
    return MSORT_OK;
}

// End-to-end sort on one GPU with the transfers overlapped (S0/S8 around
// S1-S3; the paper finds the transfers dominate).
// The chunk arrives in kPieces pieces on the copy stream; each piece is radix
// sorted (in place, B0 as scratch) as soon as it has landed, while the next
// one is still in flight.  Pieces 0+1 merge into B0 while pieces 2-3 arrive,
// pieces 2+3 merge after the last one; the final merge of the two runs is cut
// into growing output ranges at merge-path co-ranks, and every slice is copied
// back while the next one merges.  The pieces shrink (3/8, 3/8, 3/16, 1/16 of
// the chunk) so that little sorting and merging is left once the last byte
// has arrived.  Same result as the sequential path (a sort is unique).
static constexpr uint64_t kPipeMinKeys = 1ull << 20;

// S0 + S1-S3 of the pipelined host sort: H2D of `n` keys from `host` into
// `dst_stage` (c keys, tail padded) in kPieces pieces on the copy stream, each
// piece radix sorted in place as soon as it has landed (B0 as scratch), pieces
// 0+1 and 2+3 merged into B0.  Leaves two sorted runs: B0[0, *split) and
// B0[*split, c).  Records e_h2d0/e_h2d1 (copy stream), e_begin/e_sorted/e_merged.
static int load_sort_pieces(msort_ctx* ctx, Rank& R, const char* host, uint64_t n, uint64_t c, char* dst_stage,
                            uint64_t* split, bool pageable = false) {
    const size_t K = key_bytes(ctx->kt);
    char* stage = dst_stage;
    char* b0 = static_cast<char*>(R.buf[0]);
    auto cut = [&](uint64_t num, uint64_t den) { return c * num / den / 1024 * 1024; };
    const uint64_t pb[kPieces + 1] = {0, cut(3, 8), cut(6, 8), cut(15, 16), c};
    // S0: every piece's H2D (and the tail padding, reading Q3) on the copy stream,
    // ordered after the compute stream's earlier work (the staging buffer's last reader)
    CUDA_TRY(cudaEventRecord(R.e_merged, R.st));
    CUDA_TRY(cudaStreamWaitEvent(R.cst, R.e_merged, 0));
    CUDA_TRY(cudaEventRecord(R.e_h2d0, R.cst));
    auto h2d_piece = [&](int i) -> int {
        const uint64_t lo = std::min(pb[i], n), hi = std::min(pb[i + 1], n);
        if (hi > lo) {
            if (pageable)  // (returns once the host threads have staged the whole piece)
                MSORT_TRY(bounce_h2d(R, stage + lo * K, host + lo * K, (hi - lo) * K, R.cst));
            else
                CUDA_TRY(cudaMemcpyAsync(stage + lo * K, host + lo * K, (hi - lo) * K, cudaMemcpyHostToDevice, R.cst));
        }
        if (i == kPieces - 1 && c > n) {
            CUDA_TRY(launch_fill_max(stage + n * K, c - n, ctx->kt, R.cst));
            ctx->tm.kernel_launches += 1;
        }
        CUDA_TRY(cudaEventRecord(R.e_piece[i], R.cst));
        if (i == kPieces - 1) CUDA_TRY(cudaEventRecord(R.e_h2d1, R.cst));
        return MSORT_OK;
    };
    // pinned: every copy queued at once; pageable: the host stages piece i+1 while the GPU sorts piece i
    for (int i = 0; i < (pageable ? 1 : kPieces); ++i) MSORT_TRY(h2d_piece(i));
    // S1-S3 per piece on the compute stream, round-1 merges as soon as possible
    CUDA_TRY(cudaEventRecord(R.e_begin, R.st));
    for (int i = 0; i < kPieces; ++i) {
        const uint64_t len = pb[i + 1] - pb[i];
        char* p = stage + pb[i] * K;
        CUDA_TRY(cudaStreamWaitEvent(R.st, R.e_piece[i], 0));
        MSORT_TRY(radix_begin(ctx, R, p, len));
        if (ctx->skip_trivial) CUDA_TRY(cudaStreamSynchronize(R.st));
        MSORT_TRY(radix_passes(ctx, R, p, p, b0 + pb[i] * K, len));
        if (i == 1 || i == 3) {  // merge pieces i-1 and i into B0 (the radix scratch of later pieces lies past them)
            const uint64_t a0 = pb[i - 1];
            CUDA_TRY(launch_merge(stage + a0 * K, pb[i] - a0, p, len, b0 + a0 * K, ctx->kt, R.mws, R.st,
                                  &ctx->tm.kernel_launches));
        }
        if (i == kPieces - 1) CUDA_TRY(cudaEventRecord(R.e_sorted, R.st));
        if (pageable && i + 1 < kPieces) MSORT_TRY(h2d_piece(i + 1));
    }
    CUDA_TRY(cudaEventRecord(R.e_merged, R.st));
    *split = pb[2];
    return MSORT_OK;
}

static int sort_host_pipelined(msort_ctx* ctx, char* host, uint64_t n, uint64_t c, bool pageable) {
    Rank& R = ctx->r[0];
    const size_t K = key_bytes(ctx->kt);
    CUDA_TRY(cudaSetDevice(R.dev));
    for (bool& b : R.xch_rec) b = false;
    char* stage = static_cast<char*>(R.stage);
    char* b0 = static_cast<char*>(R.buf[0]);
    uint64_t split = 0;
    MSORT_TRY(load_sort_pieces(ctx, R, host, n, c, stage, &split, pageable));
    // S8 overlapped with the final merge: slice co-ranks, then merge + D2H per slice
    const char* A = b0;
    const uint64_t al = split;
    const char* B = b0 + split * K;
    const uint64_t bl = c - split;
    // co-ranks at multiples of c/64; slices end at 1/64, 1/16, 1/4 and all of
    // the chunk: each copy (PCIe) outlasts the next slice's merge (HBM), so the
    // copies run back to back and only the first, small merge is exposed
    const uint64_t step = (c + 63) / 64 / 1024 * 1024 + 1024;
    const int nsteps = int((c + step - 1) / step);
    CUDA_TRY(launch_corank(A, al, B, bl, step, uint64_t(nsteps) + 1, ctx->kt, R.d_pivot, R.st));
    ctx->tm.kernel_launches += 1;
    CUDA_TRY(cudaMemcpyAsync(R.h_pivot, R.d_pivot, size_t(nsteps + 1) * sizeof(uint64_t), cudaMemcpyDeviceToHost, R.st));
    CUDA_TRY(cudaStreamSynchronize(R.st));
    int ends[kSlices], ns = 0;
    for (int e : {1, 4, 16, nsteps})
        if (e <= nsteps && (ns == 0 || e > ends[ns - 1])) ends[ns++] = e;
    auto slice_lo = [&](int s) { return uint64_t(s ? ends[s - 1] : 0) * step; };
    auto slice_hi = [&](int s) { return std::min(c, uint64_t(ends[s]) * step); };
    auto d2h_slice = [&](int s) -> int {
        const uint64_t lo = slice_lo(s), dhi = std::min(slice_hi(s), n);
        CUDA_TRY(cudaStreamWaitEvent(R.cst, R.e_slice[s], 0));
        if (s == 0) CUDA_TRY(cudaEventRecord(R.e_d2h0, R.cst));
        if (dhi > lo) {
            if (pageable)  // (returns once the slice is in host memory; later slices keep merging meanwhile)
                MSORT_TRY(bounce_d2h(R, host + lo * K, stage + lo * K, (dhi - lo) * K, R.cst));
            else
                CUDA_TRY(cudaMemcpyAsync(host + lo * K, stage + lo * K, (dhi - lo) * K, cudaMemcpyDeviceToHost, R.cst));
        }
        return MSORT_OK;
    };
    for (int s = 0; s < ns; ++s) {
        const int j0 = s ? ends[s - 1] : 0, j1 = ends[s];
        const uint64_t lo = slice_lo(s), hi = slice_hi(s);
        const uint64_t a0 = R.h_pivot[j0], a1 = R.h_pivot[j1];
        const uint64_t b0i = lo - a0, b1i = hi - a1;
        CUDA_TRY(launch_merge(A + a0 * K, a1 - a0, B + b0i * K, b1i - b0i, stage + lo * K, ctx->kt, R.mws, R.st,
                              &ctx->tm.kernel_launches));
        CUDA_TRY(cudaEventRecord(R.e_slice[s], R.st));
        if (!pageable) MSORT_TRY(d2h_slice(s));
    }
    if (pageable)
        for (int s = 0; s < ns; ++s) MSORT_TRY(d2h_slice(s));
    CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    CUDA_TRY(cudaEventRecord(R.e_d2h1, R.cst));
    CUDA_TRY(cudaEventSynchronize(R.e_d2h1));
    CUDA_TRY(cudaEventSynchronize(R.e_end));
    collect_timings(ctx, 1);
    // phases overlap here: h2d = all pieces landed, sort = first piece's sort
    // start .. last piece sorted, merge = .. final merge done, d2h = first
    // slice's copy start .. last byte back
    msort_timings& t = ctx->tm;
    t.sort_ms = elapsed(R.e_begin, R.e_sorted);
    t.merge_ms = elapsed(R.e_sorted, R.e_end);
    t.h2d_ms = elapsed(R.e_h2d0, R.e_h2d1);
    t.d2h_ms = elapsed(R.e_d2h0, R.e_d2h1);
    t.total_ms = elapsed(R.e_h2d0, R.e_d2h1);
    t.hist_ms = 0;  // (pass_ms_sum / passes_run: those of the last piece)
    return MSORT_OK;
}

int msort_sort_host(msort_ctx* ctx, void* host_keys, uint64_t n) {
    if (!ctx || ctx->dist) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL or dist ctx");
    if (n && !host_keys) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL keys");
    if (n <= 1) return MSORT_OK;
    const int g = ctx->g;
    const uint64_t c = chunk_size(n, g);
    MSORT_TRY(check_c(ctx, c));
    DeviceGuard guard;
    reset_timings(ctx, c);
    const size_t K = key_bytes(ctx->kt);
    char* host = static_cast<char*>(host_keys);
    // pageable keys: through pinned bounce buffers (one GPU: pipelined like pinned keys, piece by piece)
    const bool pageable = host_is_pageable(host_keys);
    if (g == 1 && ctx->host_pipeline && c >= kPipeMinKeys) return sort_host_pipelined(ctx, host, n, c, pageable);
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        for (bool& b : R.xch_rec) b = false;
        R.user = R.stage;
        const uint64_t lo = std::min<uint64_t>(n, uint64_t(i) * c);
        const uint64_t cnt = std::min<uint64_t>(n - lo, c);
        CUDA_TRY(cudaEventRecord(R.e_h2d0, R.st));
        if (cnt && pageable) MSORT_TRY(bounce_h2d(R, R.stage, host + lo * K, cnt * K, R.st));
        else if (cnt) CUDA_TRY(cudaMemcpyAsync(R.stage, host + lo * K, cnt * K, cudaMemcpyHostToDevice, R.st));
        CUDA_TRY(launch_fill_max(static_cast<char*>(R.stage) + cnt * K, c - cnt, ctx->kt, R.st));
        if (c > cnt) ctx->tm.kernel_launches += 1;
        CUDA_TRY(cudaEventRecord(R.e_h2d1, R.st));
    }
    MSORT_TRY(sort_device_local(ctx, c));
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        const uint64_t lo = std::min<uint64_t>(n, uint64_t(i) * c);
        const uint64_t cnt = std::min<uint64_t>(n - lo, c);
        CUDA_TRY(cudaEventRecord(R.e_d2h0, R.st));
        if (cnt && pageable) MSORT_TRY(bounce_d2h(R, host + lo * K, R.stage, cnt * K, R.st));
        else if (cnt) CUDA_TRY(cudaMemcpyAsync(host + lo * K, R.stage, cnt * K, cudaMemcpyDeviceToHost, R.st));
        CUDA_TRY(cudaEventRecord(R.e_d2h1, R.st));
    }
    for (int i = 0; i < g; ++i) {
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaEventSynchronize(ctx->r[i].e_d2h1));
    }
    if (ctx->stats_on_device) stage_stats_from_device(ctx, *ctx->r[0].h_stage, c);
    collect_timings(ctx, g);
    collect_exchange_timings(ctx);
    for (int i = 0; i < g; ++i) {
        Rank& R = ctx->r[i];
        cudaSetDevice(R.dev);
        ctx->tm.h2d_ms = std::max(ctx->tm.h2d_ms, double(elapsed(R.e_h2d0, R.e_h2d1)));
        ctx->tm.d2h_ms = std::max(ctx->tm.d2h_ms, double(elapsed(R.e_d2h0, R.e_d2h1)));
        ctx->tm.total_ms = std::max(ctx->tm.total_ms, double(elapsed(R.e_h2d0, R.e_d2h1)));
    }
    return MSORT_OK;
}

int msort_sort(void* keys, uint64_t n, int key_type, int n_gpus, void* stream) {
    if (!valid_kt(key_type) || !valid_g(n_gpus)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad key_type or n_gpus");
    if (n <= 1) return MSORT_OK;
    if (!keys) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL keys");
    DeviceGuard guard;
    cudaPointerAttributes attr{};
    cudaError_t ae = cudaPointerGetAttributes(&attr, keys);
    if (ae != cudaSuccess) {
        cudaGetLastError();
        attr.type = cudaMemoryTypeUnregistered;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < n_gpus) {
        cudaGetLastError();
        return set_error(MSORT_ERR_DEVICE, "too few CUDA devices");
    }
    const bool on_device = attr.type == cudaMemoryTypeDevice || attr.type == cudaMemoryTypeManaged;
    const int first_dev = on_device && n_gpus == 1 ? attr.device : 0;
    std::lock_guard<std::mutex> lock(g_cache_mu);
    auto key = std::make_tuple(n_gpus, first_dev, key_type);
    msort_ctx* ctx = g_cache.count(key) ? g_cache[key] : nullptr;
    const uint64_t c = chunk_size(n, n_gpus);
    if (ctx && ctx->cap < c) {
        msort_destroy(ctx);
        ctx = nullptr;
    }
    if (!ctx) {
        std::vector<int> devs(n_gpus);
        for (int i = 0; i < n_gpus; ++i) devs[i] = first_dev + i;
        MSORT_TRY(msort_create(&ctx, n_gpus, devs.data(), n, key_type));
        g_cache[key] = ctx;
    }
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (!on_device) {
        CUDA_TRY(cudaStreamSynchronize(st));
        return msort_sort_host(ctx, keys, n);
    }
    if (n_gpus == 1) {
        void* chunks[1] = {keys};
        void* streams[1] = {stream};
        return msort_sort_device(ctx, chunks, n, stream ? streams : nullptr);
    }
    // device pointer, several GPUs: distribute into the per-GPU staging chunks
    CUDA_TRY(cudaStreamSynchronize(st));
    const size_t K = key_bytes(key_type);
    char* src = static_cast<char*>(keys);
    std::vector<void*> chunks(n_gpus);
    for (int i = 0; i < n_gpus; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        const uint64_t lo = std::min<uint64_t>(n, uint64_t(i) * c);
        const uint64_t cnt = std::min<uint64_t>(n - lo, c);
        if (cnt) CUDA_TRY(cudaMemcpyAsync(R.stage, src + lo * K, cnt * K, cudaMemcpyDefault, R.st));
        CUDA_TRY(launch_fill_max(static_cast<char*>(R.stage) + cnt * K, c - cnt, key_type, R.st));
        chunks[i] = R.stage;
    }
    MSORT_TRY(msort_sort_device(ctx, chunks.data(), c, nullptr));
    for (int i = 0; i < n_gpus; ++i) {
        Rank& R = ctx->r[i];
        CUDA_TRY(cudaSetDevice(R.dev));
        const uint64_t lo = std::min<uint64_t>(n, uint64_t(i) * c);
        const uint64_t cnt = std::min<uint64_t>(n - lo, c);
        if (cnt) CUDA_TRY(cudaMemcpyAsync(src + lo * K, R.stage, cnt * K, cudaMemcpyDefault, R.st));
    }
    for (int i = 0; i < n_gpus; ++i) {
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaStreamSynchronize(ctx->r[i].st));
    }
    return MSORT_OK;
}

// --- dist mode (one process per GPU) -----------------------------------------

struct DistHandle {
    uint32_t magic;
    int32_t rank;
    uint64_t cap;
    cudaIpcMemHandle_t b0, b1, flags;
};
static_assert(sizeof(DistHandle) <= MSORT_DIST_HANDLE_BYTES, "handle bytes");
static const uint32_t kDistMagic = 0x4D534F52u;

int msort_dist_create(msort_ctx** out, int rank, int world, int device, uint64_t max_keys_per_rank, int key_type) {
    if (!out || !valid_g(world) || rank < 0 || rank >= world || !valid_kt(key_type))
        return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_error(MSORT_ERR_DEVICE, "no CUDA device");
    }
    if (device < 0 || device >= ndev) return set_error(MSORT_ERR_DEVICE, "device id out of range");
    DeviceGuard guard;
    auto ctx = std::make_unique<msort_ctx>();
    ctx->g = world;
    ctx->kt = key_type;
    ctx->dist = true;
    ctx->rank = rank;
    ctx->nlocal = 1;
    ctx->cap = (std::max<uint64_t>(max_keys_per_rank, 4) + 3) / 4 * 4;
    if (ctx->cap >= (1ull << 32)) return set_error(MSORT_ERR_INVALID_ARGUMENT, "keys per GPU must be < 2^32");
    ctx->r[0].dev = device;
    int s = alloc_rank(ctx.get(), ctx->r[0], true, true);
    if (s != MSORT_OK) {
        free_rank(ctx->r[0]);
        return s;
    }
    CUDA_TRY(cudaSetDevice(device));
    CUDA_TRY(cudaMalloc(&ctx->my_flags, 256));
    CUDA_TRY(cudaMemset(ctx->my_flags, 0, 256));
    *out = ctx.release();
    return MSORT_OK;
}

int msort_dist_export(msort_ctx* ctx, void* handle_out) {
    if (!ctx || !ctx->dist || !handle_out) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    DeviceGuard guard;
    CUDA_TRY(cudaSetDevice(ctx->r[0].dev));
    DistHandle h{};
    h.magic = kDistMagic;
    h.rank = ctx->rank;
    h.cap = ctx->cap;
    CUDA_TRY(cudaIpcGetMemHandle(&h.b0, ctx->r[0].buf[0]));
    CUDA_TRY(cudaIpcGetMemHandle(&h.b1, ctx->r[0].buf[1]));
    CUDA_TRY(cudaIpcGetMemHandle(&h.flags, ctx->my_flags));
    std::memset(handle_out, 0, MSORT_DIST_HANDLE_BYTES);
    std::memcpy(handle_out, &h, sizeof(h));
    return MSORT_OK;
}

static int dist_barrier(msort_ctx* ctx);

int msort_dist_import(msort_ctx* ctx, const void* all_handles) {
    if (!ctx || !ctx->dist || !all_handles) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    DeviceGuard guard;
    CUDA_TRY(cudaSetDevice(ctx->r[0].dev));
    const char* base = static_cast<const char*>(all_handles);
    for (int q = 0; q < ctx->g; ++q) {
        DistHandle h;
        std::memcpy(&h, base + size_t(q) * MSORT_DIST_HANDLE_BYTES, sizeof(h));
        if (h.magic != kDistMagic || h.rank != q || h.cap != ctx->cap)
            return set_error(MSORT_ERR_INVALID_ARGUMENT, "handle array does not match (rank order / capacity)");
        if (q == ctx->rank) {
            ctx->peer_buf[q][0] = ctx->r[0].buf[0];
            ctx->peer_buf[q][1] = ctx->r[0].buf[1];
            ctx->peer_flags[q] = ctx->my_flags;
            continue;
        }
        void* p = nullptr;
        CUDA_TRY(cudaIpcOpenMemHandle(&p, h.b0, cudaIpcMemLazyEnablePeerAccess));
        ctx->opened.push_back(p);
        ctx->peer_buf[q][0] = p;
        CUDA_TRY(cudaIpcOpenMemHandle(&p, h.b1, cudaIpcMemLazyEnablePeerAccess));
        ctx->opened.push_back(p);
        ctx->peer_buf[q][1] = p;
        CUDA_TRY(cudaIpcOpenMemHandle(&p, h.flags, cudaIpcMemLazyEnablePeerAccess));
        ctx->opened.push_back(p);
        ctx->peer_flags[q] = static_cast<unsigned long long*>(p);
    }
    ctx->imported = true;
    // self-test of bulk copies from every peer's mapping (collective: every rank
    // writes its odd pattern, a device barrier, merges reading each peer, a
    // barrier before anyone's B0 is reused)
    if (ctx->g > 1 && ctx->cap >= 2 * uint64_t(kSelfTestKeys)) {
        Rank& R = ctx->r[0];
        std::vector<uint32_t> even, odd;
        selftest_pattern(even, odd, kSelfTestKeys);
        CUDA_TRY(cudaMemcpy(R.buf[0], odd.data(), kSelfTestKeys * 4, cudaMemcpyHostToDevice));
        MSORT_TRY(dist_barrier(ctx));
        for (int q = 0; q < ctx->g; ++q) {
            if (q == ctx->rank) continue;
            bool ok = false;
            const int st = selftest_merge(ctx, R, ctx->peer_buf[q][0], kSelfTestKeys, &ok);
            if (st != MSORT_OK || !ok) ctx->peer_bulk_ok = false;
        }
        MSORT_TRY(dist_barrier(ctx));
        CUDA_TRY(cudaMemcpyAsync(R.h_err, R.d_err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
        CUDA_TRY(cudaStreamSynchronize(R.st));
        if (*R.h_err) return set_error(MSORT_ERR_TIMEOUT, "device barrier timed out during the peer self-test");
        MSORT_TRY(apply_exchange_mode(ctx));
    }
    return MSORT_OK;
}

static int dist_barrier(msort_ctx* ctx) {
    Rank& R = ctx->r[0];
    BarrierArgs a{};
    for (int q = 0; q < ctx->g; ++q) a.peer_flags[q] = ctx->peer_flags[q];
    a.my_flags = ctx->my_flags;
    a.rank = ctx->rank;
    a.world = ctx->g;
    a.epoch = ++ctx->epoch;
    const char* env = std::getenv("MSORT_BARRIER_TIMEOUT_S");
    const double tmo = env ? std::atof(env) : 60.0;
    a.timeout_ns = (unsigned long long)(tmo * 1e9);
    a.err = R.d_err;
    CUDA_TRY(launch_barrier(a, R.st));
    ctx->tm.kernel_launches += 1;
    return MSORT_OK;
}

// c = chunk keys, valid = real keys in it (the rest is padded here, reading Q3)
static int dist_sort_impl(msort_ctx* ctx, void* d_chunk, uint64_t c, void* stream, bool keep_timings,
                          const char* host, uint64_t valid, bool pageable = false);

int msort_plan_chunk(uint64_t n, int g, int rank, uint64_t* c, uint64_t* offset, uint64_t* valid) {
    if (!valid_g(g) || rank < 0 || rank >= g) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad g or rank");
    const uint64_t cc = chunk_size(n, g);
    const uint64_t lo = std::min<uint64_t>(n, uint64_t(rank) * cc);
    if (c) *c = cc;
    if (offset) *offset = lo;
    if (valid) *valid = std::min<uint64_t>(n - lo, cc);
    return MSORT_OK;
}

// --- interconnect peaks ----------------------------------------------------------

// One timed pattern over the ranks this process drives: `issue(i)` enqueues rank
// i's copies on its streams; every stream first waits for every rank's start
// marker (they start together), the time is the slowest rank's.  Dist mode: a
// device barrier lines the processes up instead.
}  // extern "C"
template <class Issue>
static int time_pattern(msort_ctx* ctx, int reps, Issue issue, double* ms_out) {
    const int nl = ctx->nlocal;
    double tot = 0;
    for (int r = 0; r < reps + 1; ++r) {
        if (ctx->dist) {
            Rank& R = ctx->r[0];
            CUDA_TRY(cudaSetDevice(R.dev));
            MSORT_TRY(dist_barrier(ctx));
        }
        for (int i = 0; i < nl; ++i) {
            CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
            CUDA_TRY(cudaEventRecord(ctx->r[i].e_sync[0], ctx->r[i].st));
        }
        for (int i = 0; i < nl; ++i) {
            Rank& R = ctx->r[i];
            CUDA_TRY(cudaSetDevice(R.dev));
            for (int q = 0; q < nl; ++q)
                if (q != i) CUDA_TRY(cudaStreamWaitEvent(R.st, ctx->r[q].e_sync[0], 0));
            CUDA_TRY(cudaEventRecord(R.e_begin, R.st));
            CUDA_TRY(cudaStreamWaitEvent(R.cst, R.e_begin, 0));
            MSORT_TRY(issue(i));
            CUDA_TRY(cudaEventRecord(R.e_merged, R.cst));
            CUDA_TRY(cudaStreamWaitEvent(R.st, R.e_merged, 0));
            CUDA_TRY(cudaEventRecord(R.e_end, R.st));
        }
        double mx = 0;
        for (int i = 0; i < nl; ++i) {
            Rank& R = ctx->r[i];
            CUDA_TRY(cudaSetDevice(R.dev));
            CUDA_TRY(cudaEventSynchronize(R.e_end));
            mx = std::max(mx, double(elapsed(R.e_begin, R.e_end)));
        }
        if (r > 0) tot += mx;
    }
    if (ctx->dist && ctx->g > 1) {  // peers are done reading our buffers
        CUDA_TRY(cudaSetDevice(ctx->r[0].dev));
        MSORT_TRY(dist_barrier(ctx));
        CUDA_TRY(cudaStreamSynchronize(ctx->r[0].st));
    }
    *ms_out = tot / std::max(1, reps);
    return MSORT_OK;
}
extern "C" {

int msort_measure_links(msort_ctx* ctx, uint64_t bytes, int reps, msort_link_peaks* out) {
    if (!ctx || !out || reps < 1) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    if (ctx->dist && !ctx->imported) return set_error(MSORT_ERR_INVALID_ARGUMENT, "dist ctx not imported");
    DeviceGuard guard;
    const int g = ctx->g, nl = ctx->nlocal;
    bytes = std::min<uint64_t>(bytes, ctx->cap * key_bytes(ctx->kt)) / 4096 * 4096;
    if (bytes == 0) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bytes below one page");
    *out = msort_link_peaks{};
    out->bytes = bytes;
    out->pairs = g / 2;
    for (int i = 0; i < nl; ++i) {
        CUDA_TRY(cudaSetDevice(ctx->r[i].dev));
        CUDA_TRY(cudaDeviceSynchronize());
    }
    // mirrored pairs: rank i pulls from rank g-1-i's B0 into its staging chunk, all pairs at once
    auto src_of = [&](int i) -> const void* {
        const int me = ctx->dist ? ctx->rank : i, p = g - 1 - me;
        return ctx->dist ? ctx->peer_buf[p][0] : ctx->r[p].buf[0];
    };
    if (g > 1) {
        int same = 0;
        if (ctx->dist) {
            same = -1;  // unknown across processes (the caller knows its device map)
        } else {
            for (int i = 0; i < g; ++i) same |= ctx->r[i].dev == ctx->r[g - 1 - i].dev;
        }
        out->same_device = same;
        double ms = 0;
        MSORT_TRY(time_pattern(ctx, reps, [&](int i) -> int {
            CUDA_TRY(cudaMemcpyAsync(ctx->r[i].stage, src_of(i), bytes, cudaMemcpyDefault, ctx->r[i].st));
            return MSORT_OK;
        }, &ms));
        out->p2p_ce_gbs = bytes / (ms * 1e6);
        MSORT_TRY(time_pattern(ctx, reps, [&](int i) -> int {
            CUDA_TRY(launch_copy_sm(ctx->r[i].stage, src_of(i), bytes, ctx->r[i].st, sm_count_of(ctx->r[i].dev)));
            return MSORT_OK;
        }, &ms));
        out->p2p_sm_gbs = bytes / (ms * 1e6);
    }
    // PCIe (§4.2): pinned host buffers per GPU, all GPUs concurrently
    std::vector<void*> hin(nl, nullptr), hout(nl, nullptr);
    int st = MSORT_OK;
    for (int i = 0; i < nl && st == MSORT_OK; ++i) {
        if (cudaMallocHost(&hin[i], bytes) != cudaSuccess || cudaMallocHost(&hout[i], bytes) != cudaSuccess) {
            cudaGetLastError();
            st = set_error(MSORT_ERR_OUT_OF_MEMORY, "pinned host buffers for the PCIe measurement");
        } else {
            std::memset(hin[i], 0x5A, bytes);
        }
    }
    double ms = 0;
    if (st == MSORT_OK)
        st = time_pattern(ctx, reps, [&](int i) -> int {
            CUDA_TRY(cudaMemcpyAsync(ctx->r[i].stage, hin[i], bytes, cudaMemcpyHostToDevice, ctx->r[i].st));
            return MSORT_OK;
        }, &ms);
    if (st == MSORT_OK) out->h2d_gbs = bytes / (ms * 1e6);
    if (st == MSORT_OK)
        st = time_pattern(ctx, reps, [&](int i) -> int {
            CUDA_TRY(cudaMemcpyAsync(hout[i], ctx->r[i].buf[0], bytes, cudaMemcpyDeviceToHost, ctx->r[i].st));
            return MSORT_OK;
        }, &ms);
    if (st == MSORT_OK) out->d2h_gbs = bytes / (ms * 1e6);
    if (st == MSORT_OK)
        st = time_pattern(ctx, reps, [&](int i) -> int {
            CUDA_TRY(cudaMemcpyAsync(ctx->r[i].stage, hin[i], bytes, cudaMemcpyHostToDevice, ctx->r[i].st));
            CUDA_TRY(cudaMemcpyAsync(hout[i], ctx->r[i].buf[0], bytes, cudaMemcpyDeviceToHost, ctx->r[i].cst));
            return MSORT_OK;
        }, &ms);
    if (st == MSORT_OK) out->bidir_gbs = bytes / (ms * 1e6);
    for (int i = 0; i < nl; ++i) {
        cudaSetDevice(ctx->r[i].dev);
        cudaDeviceSynchronize();
        if (hin[i]) cudaFreeHost(hin[i]);
        if (hout[i]) cudaFreeHost(hout[i]);
    }
    return st;
}

int msort_nccl_unique_id(void* out) {
    if (!out) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL out");
    std::string err;
    if (!nccl_unique_id(out, &err)) return set_error(MSORT_ERR_NCCL, err);
    return MSORT_OK;
}

int msort_dist_nccl_init(msort_ctx* ctx, const void* unique_id) {
    if (!ctx || !ctx->dist || !unique_id) return set_error(MSORT_ERR_INVALID_ARGUMENT, "bad argument");
    DeviceGuard guard;
    CUDA_TRY(cudaSetDevice(ctx->r[0].dev));
    nccl_destroy(ctx->nccl);
    std::string err;
    if (!nccl_init_rank(ctx->nccl, ctx->g, unique_id, ctx->rank, &err)) return set_error(MSORT_ERR_NCCL, err);
    return MSORT_OK;
}

int msort_release_cached(void) {
    std::lock_guard<std::mutex> lock(g_cache_mu);
    for (auto& kv : g_cache) msort_destroy(kv.second);
    g_cache.clear();
    return MSORT_OK;
}

int msort_dist_sort(msort_ctx* ctx, void* d_chunk, uint64_t n_total, void* stream) {
    if (!ctx || !ctx->dist) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL or non-dist ctx");
    uint64_t c = 0, valid = 0;
    MSORT_TRY(msort_plan_chunk(n_total, ctx->g, ctx->rank, &c, nullptr, &valid));
    return dist_sort_impl(ctx, d_chunk, c, stream, false, nullptr, valid);
}

int msort_dist_sort_host(msort_ctx* ctx, void* host_keys, uint64_t n_total) {
    if (!ctx || !ctx->dist || !ctx->imported) return set_error(MSORT_ERR_INVALID_ARGUMENT, "dist ctx not imported");
    uint64_t c = 0, valid = 0;
    MSORT_TRY(msort_plan_chunk(n_total, ctx->g, ctx->rank, &c, nullptr, &valid));
    if (valid && !host_keys) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL keys");
    MSORT_TRY(check_c(ctx, c));
    DeviceGuard guard;
    Rank& R = ctx->r[0];
    CUDA_TRY(cudaSetDevice(R.dev));
    reset_timings(ctx, c);
    const size_t K = key_bytes(ctx->kt);
    const bool pageable = valid && host_is_pageable(host_keys);
    if (ctx->host_pipeline && c >= kPipeMinKeys) {
        // pipelined S0 (MSORT_OPT_HOST_PIPELINE): H2D pieces sorted as they land (the pad is filled there);
        // pageable keys: the host stages piece i+1 through the bounce buffers while the GPU sorts piece i
        MSORT_TRY(dist_sort_impl(ctx, R.stage, c, R.st, true, static_cast<const char*>(host_keys), valid, pageable));
    } else {
        CUDA_TRY(cudaEventRecord(R.e_h2d0, R.st));
        if (pageable) MSORT_TRY(bounce_h2d(R, R.stage, static_cast<const char*>(host_keys), valid * K, R.st));
        else if (valid) CUDA_TRY(cudaMemcpyAsync(R.stage, host_keys, valid * K, cudaMemcpyHostToDevice, R.st));
        CUDA_TRY(cudaEventRecord(R.e_h2d1, R.st));
        MSORT_TRY(dist_sort_impl(ctx, R.stage, c, R.st, true, nullptr, valid));
    }
    CUDA_TRY(cudaEventRecord(R.e_d2h0, R.st));
    if (pageable) MSORT_TRY(bounce_d2h(R, static_cast<char*>(host_keys), R.stage, valid * K, R.st));
    else if (valid) CUDA_TRY(cudaMemcpyAsync(host_keys, R.stage, valid * K, cudaMemcpyDeviceToHost, R.st));
    CUDA_TRY(cudaEventRecord(R.e_d2h1, R.st));
    CUDA_TRY(cudaEventSynchronize(R.e_d2h1));
    ctx->tm.h2d_ms = elapsed(R.e_h2d0, R.e_h2d1);
    ctx->tm.d2h_ms = elapsed(R.e_d2h0, R.e_d2h1);
    ctx->tm.total_ms = elapsed(R.e_h2d0, R.e_d2h1);
    return MSORT_OK;
}

static int dist_sort_impl(msort_ctx* ctx, void* d_chunk, uint64_t c, void* stream, bool keep_timings,
                          const char* host, uint64_t valid, bool pageable) {
    if (!ctx || !ctx->dist || !ctx->imported) return set_error(MSORT_ERR_INVALID_ARGUMENT, "dist ctx not imported");
    if (c && !d_chunk) return set_error(MSORT_ERR_INVALID_ARGUMENT, "NULL chunk");
    MSORT_TRY(check_c(ctx, c));
    DeviceGuard guard;
    const int g = ctx->g, me = ctx->rank;
    Rank& R = ctx->r[0];
    CUDA_TRY(cudaSetDevice(R.dev));
    if (!keep_timings) reset_timings(ctx, c);
    for (bool& b : R.xch_rec) b = false;
    cudaStream_t ust = static_cast<cudaStream_t>(stream);
    CUDA_TRY(cudaEventRecord(R.e_sync[MSORT_MAX_STAGES], ust));
    CUDA_TRY(cudaStreamWaitEvent(R.st, R.e_sync[MSORT_MAX_STAGES], 0));
    R.user = d_chunk;
    CUDA_TRY(cudaEventRecord(R.e_begin, R.st));
    if (c == 0) return MSORT_OK;
    // S1-S3 (host != NULL: S0 too, pipelined - the chunk lands from `host` in
    // pieces, each sorted while the next is in flight, then merged)
    int cur[MSORT_MAX_GPUS];
    void* sorted_dst = g == 1 ? d_chunk : R.buf[1];
    if (host) {
        uint64_t split = 0;
        MSORT_TRY(load_sort_pieces(ctx, R, host, valid, c, static_cast<char*>(d_chunk), &split, pageable));
        const char* b0 = static_cast<const char*>(R.buf[0]);
        CUDA_TRY(launch_merge(b0, split, b0 + split * key_bytes(ctx->kt), c - split, sorted_dst, ctx->kt, R.mws, R.st,
                              &ctx->tm.kernel_launches));
    } else {
        if (valid < c) {  // reading Q3: pad with the largest key under T
            CUDA_TRY(launch_fill_max(static_cast<char*>(d_chunk) + valid * key_bytes(ctx->kt), c - valid, ctx->kt, R.st));
            ctx->tm.kernel_launches += 1;
        }
        MSORT_TRY(radix_begin(ctx, R, d_chunk, c));
        if (ctx->skip_trivial) CUDA_TRY(cudaStreamSynchronize(R.st));
        MSORT_TRY(radix_passes(ctx, R, d_chunk, sorted_dst, R.buf[0], c));
    }
    for (int q = 0; q < g; ++q) cur[q] = g == 1 ? -1 : 1;
    CUDA_TRY(cudaEventRecord(R.e_sorted, R.st));
    if (g > 1 && (ctx->xmode == 2 || ctx->xmode == 3)) {
        // NEXT-1: splitters from every peer's sorted chunk, one pull per peer,
        // barrier (peers' B1 no longer read), local merge tree into d_chunk
        const size_t K = key_bytes(ctx->kt);
        MSORT_TRY(dist_barrier(ctx));
        if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][0], R.st));
        GroupPtrs all{};
        for (int q = 0; q < g; ++q) all.p[q] = ctx->peer_buf[q][1];
        CUDA_TRY(launch_splitters(all, g, c, ctx->kt, R.d_pivot, R.st));
        ctx->tm.kernel_launches += 1;
        CUDA_TRY(cudaMemcpyAsync(R.h_pivot, R.d_pivot, size_t(g + 1) * g * sizeof(uint64_t), cudaMemcpyDeviceToHost,
                                 R.st));
        CUDA_TRY(cudaMemcpyAsync(R.h_err, R.d_err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
        CUDA_TRY(cudaStreamSynchronize(R.st));
        if (*R.h_err) return set_error(MSORT_ERR_TIMEOUT, "device barrier timed out (a peer rank did not arrive)");
        std::vector<uint64_t> s(R.h_pivot, R.h_pivot + (g + 1) * g);
        record_alltoall_stats(ctx, s.data(), g);
        const Runs rr = runs_of(s.data(), g, me);
        if (ctx->xmode == 2) {
            // fused: merge straight out of the peers' B1, then one barrier so that
            // no rank reuses its B1 while a peer may still be reading it
            const char* rp[MSORT_MAX_GPUS];
            for (int q = 0; q < g; ++q) rp[q] = static_cast<const char*>(ctx->peer_buf[q][1]) + s[me * g + q] * K;
            MSORT_TRY(merge_tree_from_peers(ctx, R, rr, rp, g, static_cast<char*>(R.buf[0]),
                                            static_cast<char*>(d_chunk), ctx->timing != 0));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][1], R.st));
            MSORT_TRY(dist_barrier(ctx));
        } else {
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[0][0], R.st));
            for (int q = 0; q < g; ++q)
                if (rr.len[q])
                    CUDA_TRY(cudaMemcpyAsync(static_cast<char*>(R.buf[0]) + rr.off[q] * K,
                                             static_cast<const char*>(ctx->peer_buf[q][1]) + s[me * g + q] * K, rr.len[q] * K,
                                             cudaMemcpyDefault, R.st));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[0][1], R.st));
            R.xch_rec[0] = ctx->timing != 0;
            MSORT_TRY(dist_barrier(ctx));  // every rank finished pulling from our B1
            MSORT_TRY(merge_tree(ctx, R, rr, g, static_cast<char*>(R.buf[0]), static_cast<char*>(R.buf[1]),
                                 static_cast<char*>(d_chunk)));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[0][1], R.st));
        }
        CUDA_TRY(cudaEventRecord(R.e_end, R.st));
        CUDA_TRY(cudaMemcpyAsync(R.h_err, R.d_err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
        CUDA_TRY(cudaStreamWaitEvent(ust, R.e_end, 0));
        CUDA_TRY(cudaStreamSynchronize(R.st));
        if (*R.h_err) return set_error(MSORT_ERR_TIMEOUT, "device barrier timed out (a peer rank did not arrive)");
        collect_timings(ctx, 1);
        collect_exchange_timings(ctx);
        ctx->tm.total_ms = ctx->tm.sort_ms + ctx->tm.merge_ms;
        return MSORT_OK;
    }
    std::vector<int> labels;
    stage_labels(g, labels);
    const int S = int(labels.size());
    const int S_run = stages_to_run(ctx, S);
    ctx->tm.n_stages = S_run;
    if (g > 1 && ctx->xmode == 0) {
        // device-resident Alg.2 (see alg2_device_local): a device barrier per
        // stage, pivots / exchange / rotation decided on the GPU, no host round trip
        BufTable bt{};
        for (int q = 0; q < g; ++q) {
            bt.p[q][0] = q == me ? d_chunk : nullptr;  // (peers' user chunks are never read)
            bt.p[q][1] = ctx->peer_buf[q][0];
            bt.p[q][2] = ctx->peer_buf[q][1];
        }
        CUDA_TRY(launch_stage_init(R.d_stage, g, R.st));
        ctx->tm.kernel_launches += 1;
        for (int s = 0; s < S_run; ++s) {
            MSORT_TRY(dist_barrier(ctx));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][0], R.st));
            CUDA_TRY(launch_stage_pivots(bt, R.d_stage, s, labels[s], g, c, ctx->kt, R.st));
            ctx->tm.kernel_launches += 1;
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_xch[s][0], R.st));
            CUDA_TRY(launch_stage_merge(bt, R.d_stage, R.d_desc, s, labels[s], me, g, c, s == S - 1, ctx->kt, R.mws,
                                        R.st, &ctx->tm.kernel_launches));
            if (ctx->timing) {
                CUDA_TRY(cudaEventRecord(R.e_xch[s][1], R.st));
                R.xch_rec[s] = true;
                CUDA_TRY(cudaEventRecord(R.e_stage[s][1], R.st));
            }
        }
        CUDA_TRY(launch_stage_final(bt, R.d_stage, me, c, ctx->kt, R.st, sm_count_of(R.dev)));
        ctx->tm.kernel_launches += 1;
        CUDA_TRY(cudaMemcpyAsync(R.h_stage, R.d_stage, sizeof(DevStage), cudaMemcpyDeviceToHost, R.st));
        ctx->stats_on_device = true;
        for (int q = 0; q < g; ++q) cur[q] = -1;
    } else {
        auto peer_ptr = [&](int q, int which) -> const void* {
            return which < 0 ? (q == me ? d_chunk : nullptr) : ctx->peer_buf[q][which];
        };
        for (int s = 0; s < S_run; ++s) {
            const int label = labels[s];
            const bool last = s == S - 1;
            MSORT_TRY(dist_barrier(ctx));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][0], R.st));
            GroupPtrs all{};
            for (int q = 0; q < g; ++q) all.p[q] = peer_ptr(q, cur[q]);
            const int ngroups = g / label;
            CUDA_TRY(launch_pivots(all, ngroups, label, c, ctx->kt, R.d_pivot, R.st));
            ctx->tm.kernel_launches += 1;
            CUDA_TRY(cudaMemcpyAsync(R.h_pivot, R.d_pivot, ngroups * sizeof(uint64_t), cudaMemcpyDeviceToHost, R.st));
            CUDA_TRY(cudaMemcpyAsync(R.h_err, R.d_err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
            CUDA_TRY(cudaStreamSynchronize(R.st));
            if (*R.h_err) return set_error(MSORT_ERR_TIMEOUT, "device barrier timed out (a peer rank did not arrive)");
            uint64_t piv[MSORT_MAX_GPUS / 2] = {};
            for (int j = 0; j < ngroups; ++j) piv[j] = R.h_pivot[j];
            Exchange ex;
            plan_exchange(g, label, c, piv, ex);
            ctx->tm.stage_label[s] = label;
            uint64_t mx = 0, sum = 0;
            for (int j = 0; j < ngroups; ++j) ctx->tm.stage_pivot[s][j] = piv[j];
            for (int q = 0; q < g; ++q) {
                mx = std::max(mx, ex.x[q]);
                if (ex.side[q] == 0) sum += ex.x[q];
            }
            ctx->tm.stage_max_x[s] = mx;
            ctx->tm.stage_keys_exchanged[s] = sum;
            R.cur = cur[me];
            int mine = cur[me];
            if (ctx->xmode == 4) {
                if (ctx->nccl.comms.empty())
                    return set_error(MSORT_ERR_NCCL, "exchange mode 4 needs msort_dist_nccl_init first");
                if (ctx->timing && ex.x[me]) CUDA_TRY(cudaEventRecord(R.e_xch[s][0], R.st));
                R.user = d_chunk;
                MSORT_TRY(nccl_stage_exchange(ctx, ex, c, last));
            }
            const void* peer = ex.partner[me] >= 0 ? peer_ptr(ex.partner[me], cur[ex.partner[me]]) : nullptr;
            MSORT_TRY(launch_exchange(ctx, R, s, last, c, ex.x[me], ex.side[me], peer_ptr(me, cur[me]), peer, mine));
            if (ctx->timing) CUDA_TRY(cudaEventRecord(R.e_stage[s][1], R.st));
            // replicate every rank's buffer rotation (all ranks see the same pivots)
            for (int q = 0; q < g; ++q)
                if (ex.x[q] != 0) cur[q] = last ? -1 : (cur[q] == 0 ? 1 : 0);
            if (cur[me] != mine) return set_error(MSORT_ERR_INTERNAL, "buffer rotation diverged");
        }
    }
    if (cur[me] != -1)
        CUDA_TRY(cudaMemcpyAsync(d_chunk, ctx->peer_buf[me][cur[me]], c * key_bytes(ctx->kt), cudaMemcpyDeviceToDevice, R.st));
    if (g > 1) MSORT_TRY(dist_barrier(ctx));  // peers finished reading our buffers before the next sort reuses them
    CUDA_TRY(cudaEventRecord(R.e_end, R.st));
    CUDA_TRY(cudaMemcpyAsync(R.h_err, R.d_err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
    CUDA_TRY(cudaStreamWaitEvent(ust, R.e_end, 0));
    CUDA_TRY(cudaStreamSynchronize(R.st));
    if (*R.h_err) return set_error(MSORT_ERR_TIMEOUT, "device barrier timed out (a peer rank did not arrive)");
    if (ctx->stats_on_device) stage_stats_from_device(ctx, *R.h_stage, c);
    collect_timings(ctx, 1);
    collect_exchange_timings(ctx);
    ctx->tm.total_ms = ctx->tm.sort_ms + ctx->tm.merge_ms;
    return MSORT_OK;
}

}  // extern "C"
