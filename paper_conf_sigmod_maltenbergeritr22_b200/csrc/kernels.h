// kernels.h - host-side launchers of the libmsort CUDA kernels (internal).
#pragma once

#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace msort {

inline int key_bytes(int kt) { return (kt == 1 || kt == 3) ? 8 : 4; }
inline bool key_is_float(int kt) { return kt == 2 || kt == 3; }
inline int num_passes(int kt) { return key_bytes(kt) * 8 / 8; }

// ----- radix (S1-S3) ------------------------------------------------------
struct RadixWs {
    uint32_t* counters;           // [8] per-pass tile counters
    uint32_t* hist;               // [8][256]
    uint32_t* base;               // [8][256] exclusive digit bases
    uint32_t* trivial;            // [8] 1 if the pass's digit is constant over all keys; [8..16) largest bin;
                                  // [16..24) the 4 most frequent digit values of each pass
    unsigned long long* gagg;     // [passes][groups][256] look-back group aggregates (tiles << 32 | sum)
    unsigned long long* status;   // [tiles][256] decoupled-lookback words (flag << 62 | tag << 32 | count)
    uint64_t tiles;
    uint64_t groups;
    size_t head_bytes;            // bytes of counters..trivial
    size_t gagg_bytes;            // bytes of the group aggregates (zeroed per sort, right after the head)
    size_t zero_bytes;            // head + aggregates + status words for this n
    size_t alloc_bytes = 0;       // whole workspace allocation (zeroed when a new tag cycle starts, epoch 0)
    uint32_t epoch = 0;           // 0..511. 0: zero the workspace; status words carry the tag
                                  // (epoch << 4 | pass + 1), so words of earlier sorts never match
};
uint32_t radix_tile_keys(int kt);
size_t radix_ws_bytes(uint64_t n, int kt);
RadixWs radix_ws_layout(void* ws, uint64_t n, int kt);

// Zero counters/hist/status, histogram all passes of `keys`, scan to bases,
// set trivial flags.  keys are raw (T applied on load).
cudaError_t radix_prologue(const void* keys, uint64_t n, int kt, const RadixWs& ws, cudaStream_t st);
// histogram only into an external [P][256] array (zeroed inside)
// scan_kernel's per-pass outputs (RadixWs::trivial): [0,8) trivial pass, [8,16)
// largest bin, [16,24) the 4 most frequent digit values, [24,32) keys on them
constexpr int kTrivialWords = 32;
cudaError_t launch_histogram(const void* keys, uint64_t n, int kt, uint32_t* hist, cudaStream_t st);
// bases from hist rows (all P)
cudaError_t launch_scan(const uint32_t* hist, uint32_t* base, uint32_t* trivial, uint64_t n, int kt, cudaStream_t st);
// true if this GPU serves same-address shared-memory atomics of one warp
// instruction in lane order (probed once per device; see radix.cu)
// (probed once per device on a private stream; answers false without probing
// while `caller` or this thread is capturing a CUDA graph)
bool atomic_rank_ok(cudaStream_t caller = nullptr);
// one onesweep pass; flags: 1 = encode on load, 2 = decode on store,
// 4 = atomic ranking (always valid for the first pass; used for every pass when
// atomic_rank_ok()), 8 = skewed pass: with atomic ranking, the 4 digit values in
// `hot` (one per byte) are ranked with one atomic per warp row and digit
cudaError_t launch_onesweep(const void* in, void* out, uint64_t n, int kt, int pass, int flags, const RadixWs& ws,
                            const uint32_t* base_row, cudaStream_t st, uint32_t hot = 0);

// ----- merge phase (S4-S6) -------------------------------------------------
struct GroupPtrs {
    const void* p[8];
};
// Alg.1 for n_groups groups of `label` chunks each (group j = chunks [j*label, (j+1)*label)
// of `all`); d_p[j] = pivot of group j.
cudaError_t launch_pivots(const GroupPtrs& all, int n_groups, int label, uint64_t c, int kt, uint64_t* d_p,
                          cudaStream_t st);
// NEXT-1 splitters: d_s[j*g + r] (j = 0..g) = keys of chunk r among the j*c
// smallest of the union of g sorted chunks (all.p[0..g)), ties to lower r.
cudaError_t launch_splitters(const GroupPtrs& all, int g, uint64_t c, int kt, uint64_t* d_s, cudaStream_t st);
size_t merge_ws_bytes(uint64_t total, int kt);
cudaError_t launch_merge(const void* a, uint64_t al, const void* b, uint64_t bl, void* out, int kt, void* ws,
                         cudaStream_t st, int* launches);
// merge-path co-ranks: d_part[j] = a-elements among the first min(j*step, al+bl)
// outputs of merging a and b (a wins ties), j < nparts
cudaError_t launch_corank(const void* a, uint64_t al, const void* b, uint64_t bl, uint64_t step, uint64_t nparts,
                          int kt, uint64_t* d_part, cudaStream_t st);
// ----- device-resident Alg.2 stages (exchange mode 0; merge.cu) -----------
struct BufTable {
    void* p[8][3];  // [rank][0 = the user chunk, 1 = B0, 2 = B1] (peer pointers for other ranks)
};
struct DevStage {   // one replica per rank, in that rank's device memory
    int32_t cur[8];         // chunk buffer (BufTable slot) holding rank q's current keys
    uint64_t piv[8][4];     // pivot of group j in stage s (Alg.1)
};
struct MergeDesc {  // a two-run merge resolved on the device
    const void* a;
    const void* b;
    void* out;
    uint64_t al, bl;
};
cudaError_t launch_stage_init(DevStage* st, int g, cudaStream_t s);
cudaError_t launch_stage_pivots(const BufTable& bt, DevStage* st, int stage, int label, int g, uint64_t c, int kt,
                                cudaStream_t s);
// resolve this rank's pair exchange -> fused exchange+merge -> rotate every rank's buffer
cudaError_t launch_stage_merge(const BufTable& bt, DevStage* st, MergeDesc* desc, int stage, int label, int me, int g,
                               uint64_t c, bool last, int kt, void* mws, cudaStream_t s, int* launches);
// copy rank me's chunk into the user buffer if the last stage left it in B0/B1
cudaError_t launch_stage_final(const BufTable& bt, const DevStage* st, int me, uint64_t c, int kt, cudaStream_t s,
                               int sms);

// SM copy of bytes (multiple of 16, 16-byte aligned; src may be a peer pointer)
cudaError_t launch_copy_sm(void* dst, const void* src, uint64_t bytes, cudaStream_t st, int sms);

// fill count keys with the largest key under T (tail padding, reading Q3)
cudaError_t launch_fill_max(void* p, uint64_t count, int kt, cudaStream_t st);

// ----- cross-process device barrier (dist mode) ----------------------------
struct BarrierArgs {
    unsigned long long* peer_flags[8];  // flags array of every rank (peer-mapped); slot [rank] written by us
    unsigned long long* my_flags;       // our own flags array (slot q written by rank q)
    int rank, world;
    unsigned long long epoch;
    unsigned long long timeout_ns;
    int* err;                            // set to 1 on timeout
};
cudaError_t launch_barrier(const BarrierArgs& a, cudaStream_t st);

}  // namespace msort
