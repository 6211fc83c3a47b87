// HET sort for data larger than the GPUs' memory (comparison baseline, SURVEY
// NEXT-4; never the product path).  PAPER.md §5.3 "Sorting Large Data"
// and the 2n-approach (Fig.11):
//   * the keys are cut into chunks of `chunk_keys`; a CHUNK GROUP is one chunk
//     per GPU; groups are sorted one after the other;
//   * every GPU holds two chunk buffers (2n): a chunk is copied in, sorted
//     (libmsort's radix sort, the other buffer as its auxiliary memory, while no
//     copy runs), then copied back WHILE the next chunk is copied into the other
//     buffer (both PCIe directions at once);
//   * the sorted chunks land back in place in host memory; a CPU multiway merge
//     (gnu_parallel::multiway_merge, a loser tree) merges all of
//     them into a separate host buffer (out-of-place).
// Keys order by T (reading Q1).  Built by baseline/het.py with g++
// against the CUDA runtime and libmsort.so (its C ABI only).
#include <cuda_runtime.h>
#include <omp.h>
#include <parallel/algorithm>

#include <chrono>
#include <cstdint>
#include <cstring>
#include <string>
#include <thread>
#include <utility>
#include <vector>

#include "../include/msort.h"

namespace {

template <typename U, bool FLOAT>
struct TLess {
    static U code(U u) {
        if (!FLOAT) return u;
        constexpr int B = sizeof(U) * 8;
        const U sign = U(1) << (B - 1);
        return (u & sign) ? U(~u) : U(u ^ sign);
    }
    bool operator()(U a, U b) const { return code(a) < code(b); }
};

template <typename U, bool FLOAT>
void merge_all(char* host, const std::vector<std::pair<uint64_t, uint64_t>>& runs, char* out, int threads) {
    std::vector<std::pair<U*, U*>> seqs;
    uint64_t total = 0;
    for (auto& r : runs) {
        U* p = reinterpret_cast<U*>(host) + r.first;
        seqs.emplace_back(p, p + r.second);
        total += r.second;
    }
    if (threads > 0) omp_set_num_threads(threads);
    __gnu_parallel::multiway_merge(seqs.begin(), seqs.end(), reinterpret_cast<U*>(out), total, TLess<U, FLOAT>(),
                                   __gnu_parallel::parallel_tag(threads > 0 ? threads : 0));
}

double now_s() {
    return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

struct Gpu {
    int dev = 0;
    void* buf[2] = {nullptr, nullptr};
    void* ws = nullptr;
    uint64_t ws_bytes = 0;
    cudaStream_t st = nullptr, h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev[4] = {};
};

thread_local std::string g_err;

#define OOC_TRY(x)                                                         \
    do {                                                                   \
        cudaError_t e_ = (x);                                              \
        if (e_ != cudaSuccess) {                                           \
            g_err = std::string(#x) + ": " + cudaGetErrorString(e_);       \
            return 4;                                                      \
        }                                                                  \
    } while (0)

// The 2n pipeline of one GPU over its chunks (every g-th chunk, starting at `first`).
int run_gpu(Gpu& G, char* host, uint64_t n, uint64_t ck, int K, int kt, int first, int stride,
            std::vector<std::pair<uint64_t, uint64_t>>* runs) {
    OOC_TRY(cudaSetDevice(G.dev));
    std::vector<uint64_t> mine;
    for (uint64_t j = first; j * ck < n; j += stride) mine.push_back(j);
    if (mine.empty()) return 0;
    auto lo = [&](size_t i) { return mine[i] * ck; };
    auto len = [&](size_t i) { return std::min(ck, n - mine[i] * ck); };
    // chunk 0 in
    OOC_TRY(cudaMemcpyAsync(G.buf[0], host + lo(0) * K, len(0) * K, cudaMemcpyHostToDevice, G.h2d));
    OOC_TRY(cudaEventRecord(G.ev[0], G.h2d));
    for (size_t i = 0; i < mine.size(); ++i) {
        const int x = int(i & 1), y = x ^ 1;  // chunk i sits in buf[x]; buf[y] is the sort's auxiliary memory
        // sort (no copy runs meanwhile: the previous D2H out of buf[y] and this chunk's H2D are done)
        OOC_TRY(cudaStreamWaitEvent(G.st, G.ev[0], 0));
        OOC_TRY(cudaStreamWaitEvent(G.st, G.ev[1], 0));
        const int rc = msort_radix_sort(G.buf[x], G.buf[y], len(i), kt, G.ws, G.ws_bytes, G.st);
        if (rc != MSORT_OK) {
            g_err = std::string("msort_radix_sort: ") + msort_last_error();
            return rc;
        }
        OOC_TRY(cudaEventRecord(G.ev[2], G.st));
        // sorted chunk i back to its place in host memory || chunk i+1 into buf[y]
        OOC_TRY(cudaStreamWaitEvent(G.d2h, G.ev[2], 0));
        OOC_TRY(cudaMemcpyAsync(host + lo(i) * K, G.buf[x], len(i) * K, cudaMemcpyDeviceToHost, G.d2h));
        OOC_TRY(cudaEventRecord(G.ev[1], G.d2h));  // buf[x] free again
        if (i + 1 < mine.size()) {
            OOC_TRY(cudaStreamWaitEvent(G.h2d, G.ev[2], 0));
            OOC_TRY(cudaMemcpyAsync(G.buf[y], host + lo(i + 1) * K, len(i + 1) * K, cudaMemcpyHostToDevice, G.h2d));
            OOC_TRY(cudaEventRecord(G.ev[0], G.h2d));
        }
        runs->emplace_back(lo(i), len(i));
    }
    OOC_TRY(cudaStreamSynchronize(G.d2h));
    OOC_TRY(cudaStreamSynchronize(G.h2d));
    OOC_TRY(cudaStreamSynchronize(G.st));
    return 0;
}

}  // namespace

extern "C" {

typedef struct {
    double gpu_phase_s;    // all chunk groups: H2D, sorts, D2H (2n pipelines of every GPU)
    double merge_s;        // CPU multiway merge of all sorted chunks
    double total_s;
    uint64_t chunks;       // sorted sublists merged
    uint64_t chunk_groups; // ceil(chunks / g)
    int threads;
} het_ooc_stats;

const char* het_ooc_last_error(void) { return g_err.c_str(); }

// Sort n keys at host_keys (pinned for full PCIe rate; its chunks are sorted in
// place) into host_out (n keys, separate: the out-of-place merge) on the GPUs
// devs[0..g) with chunks of chunk_keys (< 2^32) keys and two chunk buffers per
// GPU.  Device memory is allocated and freed inside, outside the timed phases.
int het_ooc_sort(void* host_keys, uint64_t n, int key_type, int g, const int* devs, uint64_t chunk_keys,
                 void* host_out, int threads, het_ooc_stats* stats) {
    if (!host_keys || !host_out || g < 1 || g > 8 || chunk_keys == 0 || chunk_keys >= (1ull << 32) || key_type < 0 ||
        key_type > 3) {
        g_err = "bad argument";
        return 1;
    }
    const int K = (key_type == 1 || key_type == 3) ? 8 : 4;
    const uint64_t ck = std::min<uint64_t>(chunk_keys, std::max<uint64_t>(n, 1));
    std::vector<Gpu> gs(g);
    int rc = 0;
    for (int i = 0; i < g && rc == 0; ++i) {
        Gpu& G = gs[i];
        G.dev = devs ? devs[i] : i;
        if (cudaSetDevice(G.dev) != cudaSuccess || cudaMalloc(&G.buf[0], ck * K) != cudaSuccess ||
            cudaMalloc(&G.buf[1], ck * K) != cudaSuccess) {
            g_err = "device buffers (2 chunks per GPU)";
            rc = 3;
            break;
        }
        G.ws_bytes = msort_radix_workspace_bytes(ck, key_type);
        if (cudaMalloc(&G.ws, G.ws_bytes) != cudaSuccess ||
            cudaStreamCreateWithFlags(&G.st, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&G.h2d, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&G.d2h, cudaStreamNonBlocking) != cudaSuccess) {
            g_err = "workspace / streams";
            rc = 3;
            break;
        }
        for (auto& e : G.ev)
            if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) rc = 4;
    }
    std::vector<std::vector<std::pair<uint64_t, uint64_t>>> runs(g);
    double t0 = now_s(), t1 = t0, t2 = t0;
    if (rc == 0) {
        std::vector<int> rcs(g, 0);
        std::vector<std::string> errs(g);
        std::vector<std::thread> th;
        char* host = static_cast<char*>(host_keys);
        for (int i = 0; i < g; ++i)
            th.emplace_back([&, i]() {
                rcs[i] = run_gpu(gs[i], host, n, ck, K, key_type, i, g, &runs[i]);
                errs[i] = g_err;  // (g_err is per thread: hand it to the caller's thread)
            });
        for (auto& t : th) t.join();
        for (int i = 0; i < g; ++i)
            if (rcs[i] && !rc) {
                rc = rcs[i];
                g_err = errs[i];
            }
        t1 = now_s();
    }
    std::vector<std::pair<uint64_t, uint64_t>> all;
    for (auto& r : runs) all.insert(all.end(), r.begin(), r.end());
    if (rc == 0) {
        char* host = static_cast<char*>(host_keys);
        char* out = static_cast<char*>(host_out);
        switch (key_type) {
            case 0: merge_all<uint32_t, false>(host, all, out, threads); break;
            case 1: merge_all<uint64_t, false>(host, all, out, threads); break;
            case 2: merge_all<uint32_t, true>(host, all, out, threads); break;
            default: merge_all<uint64_t, true>(host, all, out, threads); break;
        }
        t2 = now_s();
    }
    for (auto& G : gs) {
        cudaSetDevice(G.dev);
        for (void* p : {G.buf[0], G.buf[1], G.ws})
            if (p) cudaFree(p);
        for (cudaStream_t s : {G.st, G.h2d, G.d2h})
            if (s) cudaStreamDestroy(s);
        for (auto e : G.ev)
            if (e) cudaEventDestroy(e);
    }
    if (stats) {
        stats->gpu_phase_s = t1 - t0;
        stats->merge_s = t2 - t1;
        stats->total_s = t2 - t0;
        stats->chunks = all.size();
        stats->chunk_groups = (all.size() + g - 1) / g;
        stats->threads = threads > 0 ? threads : omp_get_max_threads();
    }
    return rc;
}

}  // extern "C"
