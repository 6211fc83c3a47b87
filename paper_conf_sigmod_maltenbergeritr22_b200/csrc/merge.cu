// merge.cu - merge-phase kernels of the P2P sort.
//
// Paper: §5.2 "P2P-Based Multi-GPU Sort".
//   pivot_kernel   Alg.1 Select_Pivot: the leftmost pivot p of
//                  two concatenated halves A, B of a group (|A| = |B|), read
//                  through peer pointers ("keys of remote GPUs are accessed via
//                  P2P memory reads").  One warp runs a 32-ary
//                  search of the monotone predicate B[i] < A[|A|-1-i] (reading
//                  Q5): 7 rounds of 64 parallel remote loads instead of ~2*32
//                  dependent ones.
//   partition_thread_kernel / merge_pipe_kernel
//                  the local merge of the two sorted runs a GPU holds after a
//                  swap as a merge-path merge.  In
//                  the fused exchange mode run b is the PARTNER's block read over
//                  NVLink inside the merge (the swap and the merge are one
//                  kernel); in swap mode both runs are local.
//   fill_kernel    tail padding with the largest key (reading Q3).
//   barrier_kernel device-side barrier over IPC-mapped flags (dist mode).
// All comparisons are on T(key) (reading Q1), so floats order by totalOrder.
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace msort {

namespace {

// index -> key of the concatenation of equal-size chunks p[first .. first+k)
template <typename U, bool FLOAT>
__device__ __forceinline__ U concat_code(const GroupPtrs& g, int first, uint64_t c, uint64_t i) {
    const uint64_t ch = i / c;
    return encode<U, FLOAT>(reinterpret_cast<const U*>(g.p[first + ch])[i - ch * c]);
}

// First index in [lo, hi) where pred is false (pred monotone true->false), or hi.
// 32-ary search by one warp: every round probes 32 evenly spaced indices.
template <typename Pred>
__device__ __forceinline__ uint64_t warp_first_false(uint64_t lo, uint64_t hi, Pred pred) {
    const int lane = threadIdx.x & 31;
    while (lo < hi) {
        const uint64_t step = (hi - lo + 31) / 32;
        const uint64_t i = lo + uint64_t(lane) * step;
        const bool valid = i < hi;
        const bool f = valid && !pred(i);
        const uint32_t falses = __ballot_sync(0xffffffffu, f);
        if (falses == 0) {
            const int nvalid = __popc(__ballot_sync(0xffffffffu, valid));
            lo = lo + uint64_t(nvalid - 1) * step + 1;
        } else {
            const int fl = __ffs(falses) - 1;
            const uint64_t nhi = lo + uint64_t(fl) * step;
            if (fl > 0) lo = lo + uint64_t(fl - 1) * step + 1;
            hi = nhi;
        }
    }
    return lo;
}

// S4: p = #{i in [0,s) : B[i] < A[s-1-i]} = Alg.1's leftmost pivot.
// `all` lists the current chunk of every GPU in order; block j handles the
// group of chunks [j*label, (j+1)*label): A = its left half, B = its right half.
template <typename U, bool FLOAT>
__global__ void __launch_bounds__(32) pivot_kernel(GroupPtrs all, int label, uint64_t c, uint64_t* p_out) {
    const int half = label / 2;
    const int first = blockIdx.x * label;
    const uint64_t s = uint64_t(half) * c;
    const uint64_t p = warp_first_false(0, s, [&](uint64_t i) {
        const U b = concat_code<U, FLOAT>(all, first + half, c, i);
        const U a = concat_code<U, FLOAT>(all, first, c, s - 1 - i);
        return b < a;
    });
    if (threadIdx.x == 0) p_out[blockIdx.x] = p;
}

// ---------------------------------------------------------------------------
// NEXT-1 ("swapping keys between GPUs only once (all-to-all)"):
// exact multi-sequence splitters.  Block j-1 handles target rank k = j*c over
// the g sorted chunks (peer pointers): a 32-ary search over the key-code
// space finds v = the k-th smallest code (each round, warp r counts
// #{C_r <= candidate} for 32 candidates, one binary search per lane), then the
// keys equal to v are handed to chunks in index order (DESIGN reading Q15).
// Output s[j*g + r] = keys of chunk r among the first k (s[0..g) = 0 and
// s[g*g ..) = c are written by block 0).
// ---------------------------------------------------------------------------
template <typename U, bool FLOAT>
__device__ __forceinline__ uint64_t count_le(const U* p, uint64_t c, U v) {
    uint64_t lo = 0, hi = c;  // first index with code > v
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (encode<U, FLOAT>(p[mid]) <= v) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

template <typename U, bool FLOAT>
__device__ __forceinline__ uint64_t count_lt(const U* p, uint64_t c, U v) {
    uint64_t lo = 0, hi = c;  // first index with code >= v
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (encode<U, FLOAT>(p[mid]) < v) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

template <typename U, bool FLOAT>
__global__ void __launch_bounds__(256) splitter_kernel(GroupPtrs all, int g, uint64_t c, uint64_t* s_out) {
    __shared__ uint64_t cnt[8][32];
    __shared__ U s_lo, s_hi;
    __shared__ uint64_t lt_s[8], le_s[8];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t j = blockIdx.x + 1;
    const uint64_t k = j * c;
    if (blockIdx.x == 0 && threadIdx.x < 8 && int(threadIdx.x) < g) {
        s_out[threadIdx.x] = 0;                       // j = 0
        s_out[uint64_t(g) * g + threadIdx.x] = c;     // j = g
    }
    if (threadIdx.x == 0) {
        s_lo = U(0);
        s_hi = ~U(0);
    }
    __syncthreads();
    // smallest code v with sum_r #{C_r <= v} >= k   (k <= g*c, so v exists)
    for (;;) {
        const U lo = s_lo, hi = s_hi;
        if (lo >= hi) break;
        const U step = (hi - lo) / U(32) + U(1);
        const U span = U(lane) * step;
        const U cand = (span > hi - lo) ? hi : U(lo + span);
        if (warp < g) cnt[warp][lane] = count_le<U, FLOAT>(reinterpret_cast<const U*>(all.p[warp]), c, cand);
        __syncthreads();
        if (warp == 0) {
            uint64_t tot = 0;
            for (int r = 0; r < g; ++r) tot += cnt[r][lane];
            const uint32_t ok = __ballot_sync(0xffffffffu, tot >= k);
            if (lane == 0) {
                // candidates are non-decreasing in lane; lane 31 may be clamped to hi
                const int f = ok ? __ffs(ok) - 1 : 31;
                const U cf = (U(f) * step > hi - lo) ? hi : U(lo + U(f) * step);
                if (!ok) {
                    // every candidate is below the answer (none was clamped to hi)
                    s_lo = U(cf + 1);
                } else if (f == 0) {
                    s_hi = lo;
                } else {
                    const U cp = U(lo + U(f - 1) * step);
                    s_lo = U(cp + 1);
                    s_hi = cf;
                }
            }
        }
        __syncthreads();
    }
    const U v = s_lo;
    if (warp < g && lane == 0) {
        const U* p = reinterpret_cast<const U*>(all.p[warp]);
        lt_s[warp] = count_lt<U, FLOAT>(p, c, v);
        le_s[warp] = count_le<U, FLOAT>(p, c, v);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t lt_tot = 0;
        for (int r = 0; r < g; ++r) lt_tot += lt_s[r];
        uint64_t need = k - lt_tot;
        for (int r = 0; r < g; ++r) {
            const uint64_t eq = le_s[r] - lt_s[r];
            const uint64_t take = eq < need ? eq : need;
            need -= take;
            s_out[j * g + r] = lt_s[r] + take;
        }
    }
}

// Merge-path partition: part[t] = number of a-elements among the first
// min(t*tile, total) outputs (a wins ties), one THREAD per boundary (plain
// binary search): the top levels of all searches hit the same L2 lines, so DRAM
// sees only the last few levels of each search (a warp-wide 32-ary search per
// boundary, round 1, touched 64 sectors per round and was slower).
// dyn != nullptr: the runs and their lengths come from device memory (the
// device-resident Alg.2 stage, resolved on the GPU after the pivot search).
template <typename U, bool FLOAT>
__global__ void __launch_bounds__(256) partition_thread_kernel(const U* __restrict__ a, uint64_t al,
                                                               const U* __restrict__ b, uint64_t bl, uint64_t tile,
                                                               uint64_t nparts, uint64_t* __restrict__ part,
                                                               const MergeDesc* __restrict__ dyn = nullptr) {
    if (dyn) {
        a = static_cast<const U*>(dyn->a);
        b = static_cast<const U*>(dyn->b);
        al = dyn->al;
        bl = dyn->bl;
        const uint64_t np = (al + bl + tile - 1) / tile + 1;
        if (np < nparts) nparts = np;
    }
    const uint64_t w = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (w >= nparts) return;
    const uint64_t total = al + bl;
    const uint64_t k = w * tile < total ? w * tile : total;
    uint64_t lo = k > bl ? k - bl : 0;
    uint64_t hi = k < al ? k : al;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (encode<U, FLOAT>(a[mid]) <= encode<U, FLOAT>(b[k - 1 - mid])) lo = mid + 1;
        else hi = mid;
    }
    part[w] = lo;
}

// ---------------------------------------------------------------------------
// Deeper pipeline (default): STAGES compact smem stages per block, each holding
// one output tile's A range followed by its B range (na + nb = TILE keys, plus
// alignment slack), so 3 blocks x (STAGES-1) tiles of input are in flight per
// SM (Little's law at ~6.5 TB/s x ~1.5 us HBM / NVLink latency needs ~65 KB per
// SM; round 1's two-stage version kept <= 45 KB).  Every range is bulk-copied
// from its 16-byte-aligned start to the 16-byte boundary after its end: the
// over-fetch never leaves the 16-byte units that hold the range's own first and
// last keys, so it cannot cross a page, and no thread-issued tail loads remain
// on the critical path.  A stage is refilled only after the bulk store that
// read it has finished reading (cp.async.bulk.wait_group.read).
// ---------------------------------------------------------------------------
__device__ __forceinline__ void bulk_store_1d(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
                 "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

struct PipeMeta {
    int na, nb;        // keys taken from a / b
    int offA, offB;    // smem slot of key a0 / b0 inside the stage
};

template <typename U, int STAGES_, int IPT32_ = 15>
struct MergePipeCfg {
    static constexpr int kStages = STAGES_;
    static constexpr int kThreads = 256;
    static constexpr int kIpt = sizeof(U) == 4 ? IPT32_ : (IPT32_ - 1) / 2;
    static constexpr int kTile = kThreads * kIpt;
    static constexpr int kV = 16 / int(sizeof(U));
    static constexpr int kStage = (kTile + 4 * kV + kV - 1) / kV * kV;  // keys per stage
    static constexpr size_t kSmem = size_t(kStages) * kStage * sizeof(U);
};

template <typename U, bool FLOAT, int STAGES, int IPT32>
__global__ void __launch_bounds__(256) merge_pipe_kernel(const U* __restrict__ a, const U* __restrict__ b, uint64_t al,
                                                         uint64_t bl, U* __restrict__ out,
                                                         const uint64_t* __restrict__ part, uint32_t tiles,
                                                         const MergeDesc* __restrict__ dyn) {
    using C = MergePipeCfg<U, STAGES, IPT32>;
    constexpr int THREADS = C::kThreads, IPT = C::kIpt, TILE = C::kTile, SK = C::kStage, V = C::kV;
    if (dyn) {  // runs resolved on the device (tiles = the launch's upper bound)
        a = static_cast<const U*>(dyn->a);
        b = static_cast<const U*>(dyn->b);
        out = static_cast<U*>(dyn->out);
        al = dyn->al;
        bl = dyn->bl;
        const uint64_t t = (al + bl + TILE - 1) / TILE;
        if (t < tiles) tiles = uint32_t(t);
    }
    extern __shared__ __align__(128) unsigned char smem_raw[];
    U* stage = reinterpret_cast<U*>(smem_raw);
    __shared__ PipeMeta meta[STAGES];
    __shared__ __align__(8) uint64_t bar[STAGES];
    const int tid = threadIdx.x;
    const uint64_t total = al + bl;

    // thread 0 only; a0/a1 = part[t], part[t+1] (loaded one tile ahead, so the
    // refill never waits on a global load while the other warps wait for it)
    auto issue = [&](uint32_t t, int s, uint64_t a0, uint64_t a1) {
        const uint64_t k0 = uint64_t(t) * TILE;
        const uint64_t k1 = k0 + TILE < total ? k0 + TILE : total;
        const uint64_t b0 = k0 - a0, b1 = k1 - a1;
        PipeMeta& m = meta[s];
        m.na = int(a1 - a0);
        m.nb = int(b1 - b0);
        U* d = stage + size_t(s) * SK;
        uint32_t bytesA = 0, bytesB = 0;
        const void *srcA = nullptr, *srcB = nullptr;
        int offB = 0;
        m.offA = 0;
        if (a1 > a0) {
            const uintptr_t s0 = reinterpret_cast<uintptr_t>(a + a0) & ~uintptr_t(15);
            const uintptr_t e0 = (reinterpret_cast<uintptr_t>(a + a1) + 15) & ~uintptr_t(15);
            srcA = reinterpret_cast<const void*>(s0);
            bytesA = uint32_t(e0 - s0);
            m.offA = int((reinterpret_cast<uintptr_t>(a + a0) - s0) / sizeof(U));
            offB = int(bytesA / sizeof(U));
        }
        m.offB = offB;
        if (b1 > b0) {
            const uintptr_t s0 = reinterpret_cast<uintptr_t>(b + b0) & ~uintptr_t(15);
            const uintptr_t e0 = (reinterpret_cast<uintptr_t>(b + b1) + 15) & ~uintptr_t(15);
            srcB = reinterpret_cast<const void*>(s0);
            bytesB = uint32_t(e0 - s0);
            m.offB = offB + int((reinterpret_cast<uintptr_t>(b + b0) - s0) / sizeof(U));
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])),
                     "r"(bytesA + bytesB)
                     : "memory");
        if (bytesA)
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(d)),
                         "l"(srcA), "r"(bytesA), "r"(smem_u32(&bar[s]))
                         : "memory");
        if (bytesB)
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(d + offB)),
                         "l"(srcB), "r"(bytesB), "r"(smem_u32(&bar[s]))
                         : "memory");
    };
    static_assert(SK >= TILE + 3 * V, "stage holds both ranges with their alignment slack");

    if (tid == 0) {
#pragma unroll
        for (int s = 0; s < STAGES; ++s) mbar_init(&bar[s], 1);
#pragma unroll
        for (int s = 0; s < STAGES - 1; ++s) {
            const uint32_t t = blockIdx.x + uint32_t(s) * gridDim.x;
            if (t < tiles) issue(t, s, part[t], part[t + 1]);
        }
    }
    __syncthreads();
    uint32_t phases = 0;  // bit s: parity of stage s
    int s = 0;
    for (uint32_t t = blockIdx.x, i = 0; t < tiles; t += gridDim.x, ++i) {
        const uint32_t tn = t + uint32_t(STAGES - 1) * gridDim.x;
        uint64_t pa0 = 0, pa1 = 0;
        if (tid == 0 && tn < tiles) {
            pa0 = __ldg(part + tn);
            pa1 = __ldg(part + tn + 1);
        }
        mbar_wait(&bar[s], (phases >> s) & 1u);
        phases ^= 1u << s;
        const PipeMeta m = meta[s];
        U* sbase = stage + size_t(s) * SK;
        const U* xa = sbase + m.offA;
        const U* xb = sbase + m.offB;
        const int na = m.na, nb = m.nb, nt = na + nb;
        const int d0 = min(tid * IPT, nt);
        int lo = max(0, d0 - nb), hi = min(d0, na);
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (encode<U, FLOAT>(xa[mid]) <= encode<U, FLOAT>(xb[d0 - 1 - mid])) lo = mid + 1;
            else hi = mid;
        }
        int ia = lo, ib = d0 - lo;
        U r[IPT];
        // One smem load per output from an address selected by the comparison
        // (A and B share the stage; a read one past the end of a run stays in
        // the stage and is never used).  The path is chosen per WARP: a warp
        // whose lanes cannot exhaust a run within IPT outputs (almost all)
        // skips the bounds predicates; otherwise every lane runs the predicated
        // loop, so no warp executes both paths.
        int pa = m.offA + ia, pb = m.offB + ib;
        U va = sbase[pa], vb = sbase[pb];
        if (__all_sync(0xffffffffu, ia + IPT <= na && ib + IPT <= nb)) {
#pragma unroll
            for (int j = 0; j < IPT; ++j) {
                const bool takeA = encode<U, FLOAT>(va) <= encode<U, FLOAT>(vb);
                r[j] = takeA ? va : vb;
                pa += takeA;
                pb += !takeA;
                const U nx = sbase[takeA ? pa : pb];
                va = takeA ? nx : va;
                vb = takeA ? vb : nx;
            }
        } else {
            const int ea = m.offA + na, eb = m.offB + nb;  // one past the end of each run
#pragma unroll
            for (int j = 0; j < IPT; ++j) {
                const bool takeA = pb >= eb || (pa < ea && encode<U, FLOAT>(va) <= encode<U, FLOAT>(vb));
                r[j] = takeA ? va : vb;
                pa += takeA;
                pb += !takeA;
                const U nx = sbase[takeA ? pa : pb];
                va = takeA ? nx : va;
                vb = takeA ? vb : nx;
            }
        }
        __syncthreads();  // every thread is done reading this stage
        if (d0 + IPT <= nt) {
#pragma unroll
            for (int j = 0; j < IPT; ++j) sbase[d0 + j] = r[j];
        } else {
#pragma unroll
            for (int j = 0; j < IPT; ++j)
                if (d0 + j < nt) sbase[d0 + j] = r[j];
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        U* dst = out + uint64_t(t) * TILE;
        const bool bulk = ((reinterpret_cast<uintptr_t>(dst) & 15) == 0) && ((uint32_t(nt) * sizeof(U)) % 16 == 0);
        if (bulk) {
            if (tid == 0) bulk_store_1d(dst, sbase, uint32_t(nt) * sizeof(U));
        } else {
            for (int j = tid; j < nt; j += THREADS) dst[j] = sbase[j];
            __syncthreads();  // scalar readers done before the stage is refilled
        }
        // refill the stage of the previous tile (its bulk store has had a whole
        // tile of time to drain) with the tile STAGES-1 ahead of this one
        const int sp = s == 0 ? STAGES - 1 : s - 1;
        if (tid == 0 && tn < tiles) {
            asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // all but this tile's store
            issue(tn, sp, pa0, pa1);
        }
        s = s + 1 == STAGES ? 0 : s + 1;
        (void)i;
        (void)V;
    }
    if (tid == 0) bulk_wait_all();
}

// dyn: the runs come from device memory and al + bl is only an upper bound
template <typename U, bool FLOAT, int STAGES, int IPT32>
cudaError_t launch_merge_pipe(const U* a, uint64_t al, const U* b, uint64_t bl, U* out, void* ws, cudaStream_t st,
                              int* launches, const MergeDesc* dyn = nullptr) {
    using C = MergePipeCfg<U, STAGES, IPT32>;
    constexpr uint64_t TILE = C::kTile;
    const uint64_t tiles = (al + bl + TILE - 1) / TILE;
    const uint64_t nparts = tiles + 1;
    uint64_t* part = reinterpret_cast<uint64_t*>(ws);
    partition_thread_kernel<U, FLOAT><<<unsigned((nparts + 255) / 256), 256, 0, st>>>(a, al, b, bl, TILE, nparts, part,
                                                                                       dyn);
    if (launches) *launches += 2;
    auto kern = merge_pipe_kernel<U, FLOAT, STAGES, IPT32>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(C::kSmem));
    if (e != cudaSuccess) return e;
    int per_sm = 0, dev = 0, sms = 0;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, C::kThreads, C::kSmem)) != cudaSuccess)
        return e;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint64_t grid = uint64_t(per_sm > 0 ? per_sm : 1) * (sms > 0 ? sms : 148);
    if (grid > tiles) grid = tiles;
    if (grid == 0) grid = 1;
    kern<<<unsigned(grid), C::kThreads, C::kSmem, st>>>(a, b, al, bl, out, part, uint32_t(tiles), dyn);
    return cudaGetLastError();
}

// measured best (profiles/merge_tuning_r1.md): 3 smem stages, 19 keys/thread (u32), 11 (u64)
template <typename U, bool FLOAT>
cudaError_t launch_merge_t(const void* a, uint64_t al, const void* b, uint64_t bl, void* out, void* ws,
                           cudaStream_t st, int* launches, const MergeDesc* dyn = nullptr) {
    constexpr int IPT32 = sizeof(U) == 4 ? 19 : 23;
    return launch_merge_pipe<U, FLOAT, 3, IPT32>((const U*)a, al, (const U*)b, bl, (U*)out, ws, st, launches, dyn);
}

// ---------------------------------------------------------------------------
// Device-resident Alg.2 stage (exchange mode 0): the pivots, every rank's x_d
// and the chunk-buffer rotation live in device memory (DevStage, one replica
// per rank), so no stage waits for a host round trip.  Per stage and rank:
//   stage_pivot_kernel   Alg.1 for every group of the stage (all ranks compute
//                        all pivots: each replica sees the same values)
//   stage_resolve_kernel this rank's mirrored-pair exchange (reading Q6) as a
//                        MergeDesc: own run + partner run (peer pointer) -> the
//                        other chunk buffer (the user chunk after the last stage)
//   partition + merge    the fused exchange+merge kernels reading MergeDesc
//   stage_rotate_kernel  every rank whose x_d != 0 moved to its other buffer
// and once after the last stage stage_final_kernel copies the chunk into the
// user buffer if the last stage left it elsewhere (x_d = 0).
// ---------------------------------------------------------------------------
__device__ __forceinline__ void pair_of(int me, int label, uint64_t c, uint64_t p, int& partner, uint64_t& x,
                                        int& side) {
    const int lo = me / label * label, mid = lo + label / 2;
    const int d = me < mid ? mid - 1 - me : me - mid;
    partner = me < mid ? mid + d : mid - 1 - d;
    side = me < mid ? 0 : 1;
    const uint64_t dc = uint64_t(d) * c;
    x = p <= dc ? 0 : (p - dc < c ? p - dc : c);
}

__global__ void stage_init_kernel(DevStage* st, int g) {
    const int t = threadIdx.x;
    if (t < 8) st->cur[t] = t < g ? 2 : 0;  // radix output of every rank: B1
    if (t < 32) (&st->piv[0][0])[t] = 0;
}

template <typename U, bool FLOAT>
__global__ void __launch_bounds__(32) stage_pivot_kernel(BufTable bt, DevStage* st, int stage, int label, uint64_t c) {
    GroupPtrs all;
#pragma unroll
    for (int q = 0; q < 8; ++q) all.p[q] = bt.p[q][st->cur[q] & 3];
    const int half = label / 2;
    const int first = blockIdx.x * label;
    const uint64_t s = uint64_t(half) * c;
    const uint64_t p = warp_first_false(0, s, [&](uint64_t i) {
        const U b = concat_code<U, FLOAT>(all, first + half, c, i);
        const U a = concat_code<U, FLOAT>(all, first, c, s - 1 - i);
        return b < a;
    });
    if (threadIdx.x == 0) st->piv[stage][blockIdx.x] = p;
}

__global__ void stage_resolve_kernel(BufTable bt, const DevStage* st, int stage, int label, int me, uint64_t c,
                                     int last, int K, MergeDesc* desc) {
    int partner, side;
    uint64_t x;
    pair_of(me, label, c, st->piv[stage][me / label], partner, x, side);
    MergeDesc m{nullptr, nullptr, nullptr, 0, 0};
    if (x != 0) {
        const char* own = static_cast<const char*>(bt.p[me][st->cur[me]]);
        const char* peer = static_cast<const char*>(bt.p[partner][st->cur[partner]]);
        m.out = last ? bt.p[me][0] : bt.p[me][st->cur[me] == 1 ? 2 : 1];
        if (side == 0) {  // L keeps its first c - x keys, receives R's first x
            m.a = own;
            m.al = c - x;
            m.b = peer;
            m.bl = x;
        } else {          // R receives L's last x keys, keeps its last c - x
            m.a = peer + (c - x) * K;
            m.al = x;
            m.b = own + x * K;
            m.bl = c - x;
        }
    }
    *desc = m;
}

__global__ void stage_rotate_kernel(DevStage* st, int stage, int label, int g, uint64_t c, int last) {
    const int q = threadIdx.x;
    if (q >= g) return;
    int partner, side;
    uint64_t x;
    pair_of(q, label, c, st->piv[stage][q / label], partner, x, side);
    const int cur = st->cur[q];
    __syncwarp();
    if (x != 0) st->cur[q] = last ? 0 : (cur == 1 ? 2 : 1);
}

__global__ void stage_final_kernel(BufTable bt, const DevStage* st, int me, uint64_t bytes) {
    const int cur = st->cur[me];
    if (cur == 0) return;
    const uint4* src = static_cast<const uint4*>(bt.p[me][cur]);
    uint4* dst = static_cast<uint4*>(bt.p[me][0]);
    const uint64_t n16 = bytes / 16;  // (chunk buffers are 16-byte aligned; a ragged tail follows)
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += uint64_t(gridDim.x) * blockDim.x)
        dst[i] = src[i];
    if (blockIdx.x == 0 && threadIdx.x < bytes % 16)
        reinterpret_cast<char*>(dst)[n16 * 16 + threadIdx.x] = reinterpret_cast<const char*>(src)[n16 * 16 + threadIdx.x];
}

template <typename U, bool FLOAT>
__global__ void fill_kernel(U* p, uint64_t count) {
    const U v = decode<U, FLOAT>(~U(0));
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < count; i += uint64_t(gridDim.x) * blockDim.x)
        p[i] = v;
}

__global__ void barrier_kernel(BarrierArgs a) {
    const int q = threadIdx.x;
    if (q < a.world && q != a.rank) {
        // release: everything this GPU wrote before the barrier (earlier
        // kernels in stream order) is visible to peers that acquire the flag
        unsigned long long* dst = a.peer_flags[q] + a.rank;
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(dst), "l"(a.epoch) : "memory");
        const unsigned long long* src = a.my_flags + q;
        const uint64_t t0 = globaltimer_ns();
        while (true) {
            unsigned long long v;
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(src) : "memory");
            if (v >= a.epoch) break;
            if (globaltimer_ns() - t0 > a.timeout_ns) {
                atomicExch(a.err, 1);
                break;
            }
            __nanosleep(256);
        }
    }
    __syncthreads();
}

}  // namespace

cudaError_t launch_pivots(const GroupPtrs& all, int n_groups, int label, uint64_t c, int kt, uint64_t* d_p,
                          cudaStream_t st) {
    switch (kt) {
        case 0: pivot_kernel<uint32_t, false><<<n_groups, 32, 0, st>>>(all, label, c, d_p); break;
        case 1: pivot_kernel<uint64_t, false><<<n_groups, 32, 0, st>>>(all, label, c, d_p); break;
        case 2: pivot_kernel<uint32_t, true><<<n_groups, 32, 0, st>>>(all, label, c, d_p); break;
        case 3: pivot_kernel<uint64_t, true><<<n_groups, 32, 0, st>>>(all, label, c, d_p); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_splitters(const GroupPtrs& all, int g, uint64_t c, int kt, uint64_t* d_s, cudaStream_t st) {
    const unsigned blocks = unsigned(g > 1 ? g - 1 : 1);
    switch (kt) {
        case 0: splitter_kernel<uint32_t, false><<<blocks, 256, 0, st>>>(all, g, c, d_s); break;
        case 1: splitter_kernel<uint64_t, false><<<blocks, 256, 0, st>>>(all, g, c, d_s); break;
        case 2: splitter_kernel<uint32_t, true><<<blocks, 256, 0, st>>>(all, g, c, d_s); break;
        case 3: splitter_kernel<uint64_t, true><<<blocks, 256, 0, st>>>(all, g, c, d_s); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

size_t merge_ws_bytes(uint64_t total, int kt) {
    const uint64_t tile = key_bytes(kt) == 4 ? uint64_t(MergePipeCfg<uint32_t, 3, 19>::kTile)
                                             : uint64_t(MergePipeCfg<uint64_t, 3, 23>::kTile);
    return size_t((total + tile - 1) / tile + 2) * 8 + 256;
}

cudaError_t launch_merge(const void* a, uint64_t al, const void* b, uint64_t bl, void* out, int kt, void* ws,
                         cudaStream_t st, int* launches) {
    if (al + bl == 0) return cudaSuccess;
    switch (kt) {
        case 0: return launch_merge_t<uint32_t, false>(a, al, b, bl, out, ws, st, launches);
        case 1: return launch_merge_t<uint64_t, false>(a, al, b, bl, out, ws, st, launches);
        case 2: return launch_merge_t<uint32_t, true>(a, al, b, bl, out, ws, st, launches);
        case 3: return launch_merge_t<uint64_t, true>(a, al, b, bl, out, ws, st, launches);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_corank(const void* a, uint64_t al, const void* b, uint64_t bl, uint64_t step, uint64_t nparts,
                          int kt, uint64_t* d_part, cudaStream_t st) {
    if (nparts == 0) return cudaSuccess;
    const unsigned blocks = unsigned((nparts + 255) / 256);
    switch (kt) {
        case 0: partition_thread_kernel<uint32_t, false><<<blocks, 256, 0, st>>>((const uint32_t*)a, al, (const uint32_t*)b, bl, step, nparts, d_part); break;
        case 1: partition_thread_kernel<uint64_t, false><<<blocks, 256, 0, st>>>((const uint64_t*)a, al, (const uint64_t*)b, bl, step, nparts, d_part); break;
        case 2: partition_thread_kernel<uint32_t, true><<<blocks, 256, 0, st>>>((const uint32_t*)a, al, (const uint32_t*)b, bl, step, nparts, d_part); break;
        case 3: partition_thread_kernel<uint64_t, true><<<blocks, 256, 0, st>>>((const uint64_t*)a, al, (const uint64_t*)b, bl, step, nparts, d_part); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_fill_max(void* p, uint64_t count, int kt, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    const unsigned blocks = unsigned(count < 256 * 1024 ? (count + 255) / 256 : 1024);
    switch (kt) {
        case 0: fill_kernel<uint32_t, false><<<blocks, 256, 0, st>>>((uint32_t*)p, count); break;
        case 1: fill_kernel<uint64_t, false><<<blocks, 256, 0, st>>>((uint64_t*)p, count); break;
        case 2: fill_kernel<uint32_t, true><<<blocks, 256, 0, st>>>((uint32_t*)p, count); break;
        case 3: fill_kernel<uint64_t, true><<<blocks, 256, 0, st>>>((uint64_t*)p, count); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_stage_init(DevStage* st, int g, cudaStream_t s) {
    stage_init_kernel<<<1, 32, 0, s>>>(st, g);
    return cudaGetLastError();
}

cudaError_t launch_stage_pivots(const BufTable& bt, DevStage* st, int stage, int label, int g, uint64_t c, int kt,
                                cudaStream_t s) {
    const int ngroups = g / label;
    switch (kt) {
        case 0: stage_pivot_kernel<uint32_t, false><<<ngroups, 32, 0, s>>>(bt, st, stage, label, c); break;
        case 1: stage_pivot_kernel<uint64_t, false><<<ngroups, 32, 0, s>>>(bt, st, stage, label, c); break;
        case 2: stage_pivot_kernel<uint32_t, true><<<ngroups, 32, 0, s>>>(bt, st, stage, label, c); break;
        case 3: stage_pivot_kernel<uint64_t, true><<<ngroups, 32, 0, s>>>(bt, st, stage, label, c); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_stage_merge(const BufTable& bt, DevStage* st, MergeDesc* desc, int stage, int label, int me, int g,
                               uint64_t c, bool last, int kt, void* mws, cudaStream_t s, int* launches) {
    const int K = key_bytes(kt);
    stage_resolve_kernel<<<1, 1, 0, s>>>(bt, st, stage, label, me, c, last ? 1 : 0, K, desc);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    // upper bound of the merged length: c (both runs together always hold c keys)
    const void* dummy = bt.p[me][0];
    switch (kt) {
        case 0: e = launch_merge_t<uint32_t, false>(dummy, c, dummy, 0, nullptr, mws, s, launches, desc); break;
        case 1: e = launch_merge_t<uint64_t, false>(dummy, c, dummy, 0, nullptr, mws, s, launches, desc); break;
        case 2: e = launch_merge_t<uint32_t, true>(dummy, c, dummy, 0, nullptr, mws, s, launches, desc); break;
        case 3: e = launch_merge_t<uint64_t, true>(dummy, c, dummy, 0, nullptr, mws, s, launches, desc); break;
        default: return cudaErrorInvalidValue;
    }
    if (e != cudaSuccess) return e;
    stage_rotate_kernel<<<1, 32, 0, s>>>(st, stage, label, g, c, last ? 1 : 0);
    if (launches) *launches += 2;
    return cudaGetLastError();
}

cudaError_t launch_stage_final(const BufTable& bt, const DevStage* st, int me, uint64_t c, int kt, cudaStream_t s,
                               int sms) {
    stage_final_kernel<<<unsigned(sms > 0 ? sms * 4 : 592), 256, 0, s>>>(bt, st, me, c * uint64_t(key_bytes(kt)));
    return cudaGetLastError();
}

__global__ void __launch_bounds__(256) copy16_kernel(uint4* __restrict__ dst, const uint4* __restrict__ src, uint64_t n16) {
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += uint64_t(gridDim.x) * blockDim.x)
        dst[i] = __ldcs(src + i);
}

cudaError_t launch_copy_sm(void* dst, const void* src, uint64_t bytes, cudaStream_t st, int sms) {
    copy16_kernel<<<unsigned(sms > 0 ? sms * 8 : 1184), 256, 0, st>>>(static_cast<uint4*>(dst),
                                                                      static_cast<const uint4*>(src), bytes / 16);
    return cudaGetLastError();
}

cudaError_t launch_barrier(const BarrierArgs& a, cudaStream_t st) {
    barrier_kernel<<<1, 32, 0, st>>>(a);
    return cudaGetLastError();
}

}  // namespace msort
