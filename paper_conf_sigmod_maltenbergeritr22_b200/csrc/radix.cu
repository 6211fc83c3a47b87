// radix.cu - per-GPU LSD radix sort of one key chunk.
//
// Paper: §5.1 "Single-GPU Sorting".  The chunk sort is
// an LSB radix sort whose passes read and write the keys once each, because
// the digit histogram is "calculated once" up front and the prefix sum is
// "decoupled" (Thrust >= 1.11 / onesweep).  This file is a
// from-scratch sm_100a onesweep:
//   hist_kernel      one read of the chunk -> P digit histograms (S2); every
//                    lane owns a private smem column per bin, so the smem
//                    atomics of one warp instruction never collide on a bank
//   scan_kernel      exclusive prefix per pass -> global digit bases (S2)
//   onesweep_kernel  persistent blocks; per tile: block digit counts, stable
//                    warp ranking (lane-ordered smem atomics, or atomicOr /
//                    8-ballot peer masks), decoupled look-back across tiles
//                    (windowed, with per-group aggregates) for the global
//                    digit offset, smem staging, coalesced scatter (S3); the
//                    next tile's keys load during the scatter
// The float codec T (reading Q1) is applied on the first pass's load and T^-1
// on the last pass's store (S1), so no separate codec pass touches HBM.
#include <atomic>
#include <cstdlib>
#include <type_traits>

#include "common.cuh"
#include "kernels.h"

namespace msort {

namespace {

// ---------------------------------------------------------------------------
// S2: digit histograms of T(key) for every pass, one read of the chunk.
// ---------------------------------------------------------------------------
constexpr int kHistThreads = 1024;
constexpr int kHistUnroll = 4;

template <typename U>
struct HistCfg {
    static constexpr int P = sizeof(U);
    static constexpr int REPL = sizeof(U) == 4 ? 32 : 16;  // private columns per bin
    static constexpr size_t kSmem = size_t(P) * 256 * REPL * 4;  // 128 KB
};

template <typename U, bool FLOAT>
__global__ void __launch_bounds__(kHistThreads, 1) hist_kernel(const U* __restrict__ in, uint64_t n,
                                                               uint32_t* __restrict__ hist) {
    constexpr int P = HistCfg<U>::P;
    constexpr int REPL = HistCfg<U>::REPL;
    constexpr int V = 16 / sizeof(U);  // keys per 16-byte vector
    extern __shared__ __align__(16) uint32_t sh[];  // [P][256][REPL]
    {
        uint4* s4 = reinterpret_cast<uint4*>(sh);
        for (int i = threadIdx.x; i < P * 256 * REPL / 4; i += blockDim.x) s4[i] = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();
    const uint32_t col = threadIdx.x % REPL;

    auto count = [&](U k) {
        const U code = encode<U, FLOAT>(k);
#pragma unroll
        for (int p = 0; p < P; ++p) atomicAdd(&sh[((p << 8) + (uint32_t(code >> (8 * p)) & 0xFF)) * REPL + col], 1u);
    };

    const uintptr_t addr = reinterpret_cast<uintptr_t>(in);
    uint64_t head = ((16 - (addr & 15)) & 15) / sizeof(U);
    if (head > n) head = n;
    const uint64_t nvec = (n - head) / V;
    const uint4* vin = reinterpret_cast<const uint4*>(in + head);
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    uint64_t v = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; v + (kHistUnroll - 1) * stride < nvec; v += kHistUnroll * stride) {
        uint4 q[kHistUnroll];
#pragma unroll
        for (int u = 0; u < kHistUnroll; ++u) q[u] = __ldcs(vin + v + u * stride);
#pragma unroll
        for (int u = 0; u < kHistUnroll; ++u) {
            const U* ks = reinterpret_cast<const U*>(&q[u]);
#pragma unroll
            for (int j = 0; j < V; ++j) count(ks[j]);
        }
    }
    for (; v < nvec; v += stride) {
        uint4 q = __ldcs(vin + v);
        const U* ks = reinterpret_cast<const U*>(&q);
#pragma unroll
        for (int j = 0; j < V; ++j) count(ks[j]);
    }
    if (blockIdx.x == 0) {
        const uint64_t tail0 = head + nvec * V;
        for (uint64_t i = threadIdx.x; i < head; i += blockDim.x) count(in[i]);
        for (uint64_t i = tail0 + threadIdx.x; i < n; i += blockDim.x) count(in[i]);
    }
    __syncthreads();
    for (int b = threadIdx.x; b < P * 256; b += blockDim.x) {
        uint32_t s = 0;
#pragma unroll 8
        for (int j = 0; j < REPL; ++j) s += sh[b * REPL + ((j + b) % REPL)];  // rotated: no bank conflicts
        if (s) atomicAdd(&hist[b], s);
    }
}

// ---------------------------------------------------------------------------
// S2: exclusive prefix of each pass's histogram; trivial[p] = one digit value
// holds all n keys (the pass is an identity permutation).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kRadix) scan_kernel(const uint32_t* __restrict__ hist, uint32_t* __restrict__ base,
                                                      uint32_t* __restrict__ trivial, uint64_t n) {
    __shared__ uint32_t wsum[kRadix / 32];
    __shared__ int any_full;
    __shared__ unsigned long long max_bin;  // count << 8 | digit
    const int p = blockIdx.x, d = threadIdx.x, lane = d & 31, warp = d >> 5;
    if (d == 0) {
        any_full = 0;
        max_bin = 0;
    }
    const uint32_t v = hist[p * kRadix + d];
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t pre = 0;
    for (int w = 0; w < warp; ++w) pre += wsum[w];
    base[p * kRadix + d] = pre + x - v;
    if (uint64_t(v) == n) any_full = 1;
    // the 4 most frequent digit values (skewed passes rank them with one atomic
    // per warp row each), largest first
    uint32_t top4 = 0, top_count = 0;
    bool taken = false;
    for (int q = 0; q < 4; ++q) {
        if (!taken) atomicMax(&max_bin, (static_cast<unsigned long long>(v) << 8) | unsigned(d));
        __syncthreads();
        const unsigned long long b = max_bin;
        if (q == 0) top_count = uint32_t(b >> 8);
        top4 |= uint32_t(b & 0xFF) << (8 * q);
        if (uint32_t(b & 0xFF) == uint32_t(d)) taken = true;
        __syncthreads();
        if (d == 0) max_bin = 0;
        __syncthreads();
    }
    if (d == 0 && trivial) {
        trivial[p] = any_full;
        trivial[8 + p] = top_count;  // size of the largest digit bin of the pass (skew)
        trivial[16 + p] = top4;      // the 4 most frequent digit values, one per byte
    }
}

// ---------------------------------------------------------------------------
// S3: onesweep pass.
//
// B200 budget (measured, profiles/): at 80% of HBM a pass must move ~2.2
// keys/cycle/SM, while shared memory serves 1 wavefront (128 B)/cycle/SM and
// the integer ALU pipe 2 warp-instructions/cycle/SM; a random 4-byte smem
// access by 32 lanes costs ~3.5 wavefronts (bank conflicts) and MATCH.ANY
// ~60 ADU cycles.  The ranking therefore mixes two peer-mask methods per item
// (compile-time pattern): an 8-ballot match (ALU only) and an smem atomicOr
// mask (3 smem ops), so both pipes work in parallel.  Per-warp digit counts are
// taken first ("early counts"), the tile aggregate is published before the
// ranking, and the ranking's leader atomicAdd returns the final smem slot.
// ---------------------------------------------------------------------------
constexpr unsigned long long kFlagAgg = 1ull, kFlagIncl = 2ull;

__device__ __forceinline__ unsigned long long pack_status(unsigned long long flag, uint32_t tag, uint32_t count) {
    return (flag << 62) | (uint64_t(tag & 0x3FFFFFFFu) << 32) | count;
}

// Lanes of the warp whose 8-bit digit equals this lane's (8 ballots).
__device__ __forceinline__ uint32_t ballot_match8(uint32_t d) {
    uint32_t peers = 0xffffffffu;
#pragma unroll
    for (int b = 0; b < 8; ++b) {
        asm("{\n\t.reg .pred p;\n\t.reg .b32 t, m;\n\t"
            "and.b32 t, %1, %2;\n\t"
            "setp.ne.u32 p, t, 0;\n\t"
            "vote.sync.ballot.b32 m, p, 0xffffffff;\n\t"
            "@!p not.b32 m, m;\n\t"
            "and.b32 %0, %0, m;\n\t}"
            : "+r"(peers)
            : "r"(d), "r"(1u << b));
    }
    return peers;
}

// THREADS x ITEMS keys per tile; bit i of BALLOT_MASK: item i ranks with the
// ballot match (else smem atomicOr); MINB blocks per SM for __launch_bounds__.
template <int THREADS_, int ITEMS_, uint32_t BALLOT_MASK_, int MINB_, bool PF_, int LB_ = 4, bool ELB_ = false,
          bool CR_ = false, int GROUP_ = 8, bool CE_ = false>
struct OsCfg {
    // prefetch configs: count the next tile's keys right after this tile's scatter
    // (per-warp zeroing, no end-of-tile barrier), so a claimed tile publishes its
    // aggregate sooner
    static constexpr bool kCountEnd = CE_;
    static constexpr uint32_t kGroup = GROUP_;  // look-back group size (tiles); 0 = tile-by-tile walk only
    static constexpr bool kCountRank = CR_;  // atomic-ranked passes: rank = the count atomic's return
    static constexpr bool kEarlyLookback = ELB_;  // look back right after publishing (before the ranking)
    static constexpr bool kPrefetch = PF_;  // load the next tile's keys into registers during the scatter
    static constexpr int kLookback = LB_;  // look-back window (independent status loads per round)
    static constexpr int kThreads = THREADS_;
    static constexpr int kItems = ITEMS_;
    static constexpr uint32_t kBallotMask = BALLOT_MASK_;
    static constexpr int kMinBlocks = MINB_;
    static constexpr int kWarps = THREADS_ / 32;
    static constexpr uint32_t kTile = uint32_t(THREADS_) * ITEMS_;
    static constexpr bool kAnyOr = (BALLOT_MASK_ & ((ITEMS_ >= 32 ? 0u : (1u << ITEMS_)) - 1u)) !=
                                   ((ITEMS_ >= 32 ? 0u : (1u << ITEMS_)) - 1u);
    // (the atomicOr peer masks exist only in the peer-match ranking, STABLE)
    template <typename U, bool STABLE = true>
    static constexpr size_t smem_bytes() {
        return size_t(kTile) * sizeof(U) + size_t(kWarps) * kRadix * 4 * (kAnyOr && STABLE ? 2 : 1);
    }
};

// STABLE = false: "atomic ranking": each key takes its smem slot with ONE
// shared-memory atomicAdd on its warp's digit counter (no peer match).  The
// order in which lanes of one warp instruction that hit the same counter
// receive their values is not specified by PTX; on sm_100 the hardware serves
// them in lane order (measured: tools/probe/atom_order.cu), which makes the
// ranking stable.  atomic_rank_ok() verifies this on the running GPU once per
// device (rank_probe_kernel) before any stable pass uses it; the first LSD pass
// may use it regardless (nothing has ordered the keys yet).
#ifndef MSORT_ABLATE
#define MSORT_ABLATE 0  // timing ablations (tools/ablate_build.py); never set in a real build
#endif
#if MSORT_ABLATE & 8
__device__ unsigned long long g_lb_stats[4];  // tiles, window rounds, polls, status loads
#endif
template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT, class Cfg, bool STABLE = true>
__global__ void __launch_bounds__(Cfg::kThreads, Cfg::kMinBlocks)
    onesweep_kernel(const U* __restrict__ in, U* __restrict__ out, uint32_t n, uint32_t shift,
                    const uint32_t* __restrict__ base, unsigned long long* __restrict__ status,
                    uint32_t* __restrict__ tile_counter, uint32_t tag, unsigned long long* __restrict__ gagg,
                    uint32_t hot, bool hot_on) {
    constexpr int THREADS = Cfg::kThreads;
    constexpr int ITEMS = Cfg::kItems;
    constexpr int WARPS = Cfg::kWarps;
    constexpr uint32_t TILE = Cfg::kTile;
    static_assert(THREADS >= kRadix, "one thread per digit in the look-back");
    static_assert((TILE * sizeof(U)) % 16 == 0, "bulk copies move whole 16-byte units");

    extern __shared__ __align__(128) unsigned char smem_raw[];
    U* s_keys = reinterpret_cast<U*>(smem_raw);                           // digit-ordered staging
    uint32_t(*s_cnt)[kRadix] = reinterpret_cast<uint32_t(*)[kRadix]>(s_keys + TILE);
    uint32_t(*s_match)[kRadix] = s_cnt + WARPS;  // only touched by atomicOr-ranked items
    __shared__ uint32_t s_delta[kRadix];
    __shared__ uint32_t s_wsum[kRadix / 32];
    __shared__ uint32_t s_next;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t ntiles = uint32_t((uint64_t(n) + TILE - 1) / TILE);  // (64-bit: n may be 2^32 - 4)
    const uint32_t lt = lanemask_lt();
    const uint32_t wofs = uint32_t(warp) * 32 * ITEMS + lane;

    // keys of tile t -> registers (warp-striped: warp w owns keys [w*32*ITEMS, (w+1)*32*ITEMS)).
    // Full tiles load raw (encoded by the caller); the partial last tile is
    // encoded here and its out-of-range slots get the largest code: they rank
    // after every real key of digit 255 and are never stored (scatter bound).
    U keys[ITEMS];
    auto load_tile = [&](uint32_t t) {
        const uint64_t tb = uint64_t(t) * TILE;
        const U* src = in + tb + wofs;
        if (tb + TILE <= n) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) keys[i] = __ldcs(src + i * 32);
        } else {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                const bool ok = tb + wofs + uint64_t(i) * 32 < n;
                U k = ok ? src[i * 32] : U(0);
                if (ENC_IN) k = encode<U, FLOAT>(k);
                keys[i] = ok ? k : ~U(0);
            }
        }
    };

    // --- decoupled look-back: exclusive count of digit d over all earlier tiles.
    // Status word per (tile, digit): flag << 62 | tag << 32 | count.  Phase 1
    // walks the predecessors inside this tile's group of kGroup tiles, a window
    // of kLookback status words per round (an unpublished predecessor is then
    // polled alone).  Phase 2 walks whole earlier groups: a group contributes
    // the inclusive count of its last tile if that is published, else its
    // aggregate word (tiles << 32 | sum, complete when tiles == kGroup; every
    // tile adds itself right after counting), so a walk of ~30 tiles takes ~3
    // rounds instead of ~8.  Publishes this tile's inclusive count.
    auto lookback = [&](const int d, const uint32_t tile, const uint32_t my_total) -> uint32_t {
        uint32_t excl = 0;
#if MSORT_ABLATE & 1  // timing ablation: no look-back, uniform-share offsets instead
        excl = uint32_t(uint64_t(tile) * (n >> 8) / ntiles);
        if (false) {
#else
        if (tile > 0) {
#endif
            // high word of a status entry: flag << 30 | tag
            const uint32_t hi_agg = uint32_t(kFlagAgg << 30) | (tag & 0x3FFFFFFFu);
            const uint32_t hi_incl = uint32_t(kFlagIncl << 30) | (tag & 0x3FFFFFFFu);
            constexpr int W = Cfg::kLookback;
            constexpr uint32_t G = Cfg::kGroup;
            const uint32_t first = G ? tile / (G ? G : 1) * G : 0u;  // phase 1 covers tiles [first, tile)
            uint32_t left = tile - first;
            const unsigned long long* p = status + uint64_t(tile - 1) * kRadix + d;
            bool done = false;
            while (left > 0) {
                uint32_t lo[W], hi[W];
#pragma unroll
                for (int k = 0; k < W; ++k) {
                    const unsigned long long w = uint32_t(k) < left ? ld_relaxed_gpu(p - k * kRadix) : 0ull;
                    lo[k] = uint32_t(w);
                    hi[k] = uint32_t(w >> 32);
                }
                bool go = true;
                uint32_t used = 0;
#pragma unroll
                for (int k = 0; k < W; ++k) {
                    go = go && (hi[k] == hi_agg || hi[k] == hi_incl);
                    if (go) {
                        excl += lo[k];
                        ++used;
                        if (hi[k] == hi_incl) {
                            done = true;
                            go = false;
                        }
                    }
                }
#if MSORT_ABLATE & 8
                atomicAdd(&g_lb_stats[1], 1ull);
#endif
                if (done) break;
                left -= used;  // (tile 0 is always inclusive, so G == 0 ends above)
                p -= used * kRadix;
                if (used == 0) {
                    unsigned long long w;
                    do {
                        __nanosleep(32);
#if MSORT_ABLATE & 8
                        atomicAdd(&g_lb_stats[2], 1ull);
#endif
                        w = ld_relaxed_gpu(p);
                    } while (uint32_t(w >> 32) != hi_agg && uint32_t(w >> 32) != hi_incl);
                }
            }
            if (G && !done) {
                uint32_t h = first / (G ? G : 1) - 1;  // newest earlier group not consumed (groups 0..h remain)
                for (;;) {
                    uint32_t val[W];
                    bool ok[W], inc[W];
#pragma unroll
                    for (int k = 0; k < W; ++k) {
                        ok[k] = inc[k] = false;
                        val[k] = 0;
                        if (uint32_t(k) <= h) {
                            const unsigned long long s = ld_relaxed_gpu(status + (uint64_t(h - k + 1) * G - 1) * kRadix + d);
                            const unsigned long long a = ld_relaxed_gpu(gagg + uint64_t(h - k) * kRadix + d);
                            inc[k] = uint32_t(s >> 32) == hi_incl;
                            ok[k] = inc[k] || uint32_t(a >> 32) == G;
                            val[k] = inc[k] ? uint32_t(s) : uint32_t(a);
                        }
                    }
                    bool go = true;
                    uint32_t used = 0;
#pragma unroll
                    for (int k = 0; k < W; ++k) {
                        go = go && ok[k];
                        if (go) {
                            excl += val[k];
                            ++used;
                            if (inc[k]) {
                                done = true;
                                go = false;
                            }
                        }
                    }
#if MSORT_ABLATE & 8
                    atomicAdd(&g_lb_stats[1], 1ull);
#endif
                    if (done || used == h + 1) break;  // (all groups down to 0 consumed)
                    h -= used;
                    if (used == 0) {
#if MSORT_ABLATE & 8
                        atomicAdd(&g_lb_stats[2], 1ull);
#endif
                        __nanosleep(32);
                    }
                }
            }
            st_relaxed_gpu(&status[uint64_t(tile) * kRadix + d], pack_status(kFlagIncl, tag, excl + my_total));
#if MSORT_ABLATE & 8
            atomicAdd(&g_lb_stats[0], 1ull);
#endif
        }
        return excl;
    };

    if (Cfg::kAnyOr && STABLE) {  // (atomic-ranked kernels have no peer-mask array)
        for (int i = tid; i < WARPS * kRadix; i += THREADS) (&s_match[0][0])[i] = 0;
    }
    // per-warp digit counters start at zero; each tile re-zeroes them during its
    // scatter (they are dead after the ranking), so no barrier of its own
    auto zero_counts = [&]() {
        uint4* z = reinterpret_cast<uint4*>(&s_cnt[0][0]);
        for (int i = tid; i < WARPS * kRadix / 4; i += THREADS) z[i] = make_uint4(0, 0, 0, 0);
    };
    zero_counts();
    if (tid == 0) {
        // Tile ids in arrival order: every lower tile is already held by a
        // running block, so the look-back below always makes progress.
        s_next = atomicAdd(tile_counter, 1u);
    }
    __syncthreads();
    uint32_t tile = s_next;
    if (Cfg::kPrefetch && tile < ntiles) load_tile(tile);
    constexpr bool kCountRank = Cfg::kCountRank && !STABLE;
    constexpr bool kCE = Cfg::kCountEnd && Cfg::kPrefetch && !kCountRank;
    auto count_keys = [&]() {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) atomicAdd(&s_cnt[warp][uint32_t(keys[i] >> shift) & 0xFF], 1u);
    };
    bool counted = false;  // kCE: this tile's keys were counted at the end of the previous one

    for (;;) {
        if (tile >= ntiles) break;
        const uint64_t tile_base = uint64_t(tile) * TILE;
        const bool full = tile_base + TILE <= n;
        if (!Cfg::kPrefetch) load_tile(tile);
        if (ENC_IN && full && !counted) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) keys[i] = encode<U, FLOAT>(keys[i]);
        }
        // (s_cnt was zeroed during the previous tile's scatter, or before the loop)

        // --- early counts: per-warp digit histogram (fire-and-forget smem adds).
        // kCountRank (atomic-ranked passes): the count's returned value is the
        // key's stable rank within (warp, digit) - lane order, see STABLE - kept
        // as 16-bit halves, so the ranking below is a plain load, not an atomic.
        uint32_t rk[kCountRank ? (ITEMS + 1) / 2 : 1];
        if (kCE && counted) {
            // counted at the end of the previous tile
        } else if constexpr (kCountRank) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                const uint32_t r = atomicAdd(&s_cnt[warp][uint32_t(keys[i] >> shift) & 0xFF], 1u);
                if (i & 1) rk[i >> 1] |= r << 16;
                else rk[i >> 1] = r;
            }
        } else
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
#if MSORT_ABLATE & 2  // timing ablation only (wrong results): no early counts
            if (keys[i] == U(0x12345)) 
#endif
            atomicAdd(&s_cnt[warp][uint32_t(keys[i] >> shift) & 0xFF], 1u);
        }
        __syncthreads();

        // --- tile totals -> publish aggregate; per-(warp, digit) smem slot bases
        uint32_t my_total = 0, my_start = 0;
        uint32_t excl_early = 0;
        uint32_t col[WARPS];  // this digit's per-warp counts (kept for the slot bases)
        if (tid < kRadix) {
            const int d = tid;
            uint32_t sum = 0;
#pragma unroll
            for (int w = 0; w < WARPS; ++w) {
                col[w] = s_cnt[w][d];
                sum += col[w];
            }
            my_total = sum;
            st_relaxed_gpu(&status[uint64_t(tile) * kRadix + d], pack_status(tile == 0 ? kFlagIncl : kFlagAgg, tag, sum));
            if constexpr (Cfg::kGroup != 0) atomicAdd(&gagg[uint64_t(tile / Cfg::kGroup) * kRadix + d], (1ull << 32) | sum);
            if (Cfg::kEarlyLookback) excl_early = lookback(d, tile, sum);
            uint32_t x = sum;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= o) x += y;
            }
            if (lane == 31) s_wsum[warp] = x;
            my_start = x - sum;  // warp-local exclusive
        }
        __syncthreads();
        if (tid < kRadix) {
            uint32_t pre = 0;
            for (int w = 0; w < (tid >> 5); ++w) pre += s_wsum[w];
            my_start += pre;
            uint32_t run = my_start;
#pragma unroll
            for (int w = 0; w < WARPS; ++w) {
                // (u64 keys leave no registers to spare: reload instead)
                const uint32_t c = sizeof(U) == 4 ? col[w] : s_cnt[w][tid];
                s_cnt[w][tid] = run;
                run += c;
            }
        }
        __syncthreads();

        // --- stable warp ranking straight into the smem slot (tile-local digit order)
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t d = uint32_t(keys[i] >> shift) & 0xFF;
            if constexpr (kCountRank) {
                s_keys[s_cnt[warp][d] + ((rk[i >> 1] >> (16 * (i & 1))) & 0xFFFFu)] = keys[i];
                continue;
            }
            if constexpr (!STABLE) {
                if (hot_on) {
                    // skewed pass: the lanes on one of the 4 most frequent digits
                    // (`hot`, one per byte) reserve their slots with one atomic by
                    // the first lane of their group and rank by lane order (ballot);
                    // every other lane takes one atomic itself - all in ONE atomic
                    // instruction, so no digit value piles up on one address
                    uint32_t mine = 0;
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const uint32_t h = (hot >> (8 * q)) & 0xFFu;
                        const uint32_t m = __ballot_sync(0xffffffffu, d == h);
                        if (d == h) mine = m;
                    }
                    const int first = mine ? __ffs(mine) - 1 : lane;
                    uint32_t got = 0;
                    if (!mine || lane == first) got = atomicAdd(&s_cnt[warp][d], mine ? uint32_t(__popc(mine)) : 1u);
                    got = __shfl_sync(0xffffffffu, got, first);
                    s_keys[got + __popc(mine & lt)] = keys[i];
                    continue;
                }
                s_keys[atomicAdd(&s_cnt[warp][d], 1u)] = keys[i];
                continue;
            }
            uint32_t peers;
            if ((Cfg::kBallotMask >> i) & 1u) {
                peers = ballot_match8(d);
            } else {
                atomicOr(&s_match[warp][d], 1u << lane);
                __syncwarp();
                peers = *reinterpret_cast<volatile uint32_t*>(&s_match[warp][d]);
            }
            const int leader = 31 - __clz(peers);
            uint32_t slot = 0;
            if (lane == leader) slot = atomicAdd(&s_cnt[warp][d], uint32_t(__popc(peers)));
            slot = __shfl_sync(0xffffffffu, slot, leader) + __popc(peers & lt);
            if (!((Cfg::kBallotMask >> i) & 1u)) {
                if (lane == leader) s_match[warp][d] = 0;
                __syncwarp();
            }
            s_keys[slot] = keys[i];
        }

        // --- look-back (deferred until after the ranking unless kEarlyLookback)
        if (tid < kRadix) {
            const int d = tid;
            const uint32_t excl = Cfg::kEarlyLookback ? excl_early : lookback(d, tile, my_total);
            s_delta[d] = base[d] + excl - my_start;
            // Prefetch configs claim the next tile here so that its loads can
            // be issued before (and overlap) this tile's scatter.
            if (Cfg::kPrefetch && tid == 0) s_next = atomicAdd(tile_counter, 1u);
        }
        __syncthreads();
        if (!Cfg::kPrefetch && tid == 0) {
            // Claim the next tile only now: a tile id claimed earlier would sit
            // queued behind this tile while its successors wait for its aggregate.
            s_next = atomicAdd(tile_counter, 1u);
        }
        uint32_t next_tile = 0;
        if (Cfg::kPrefetch) {
            // keys[] is dead until the next iteration: its loads fly during the scatter
            next_tile = s_next;
            if (next_tile < ntiles) load_tile(next_tile);
        }

        // --- scatter: consecutive smem slots of one digit go to consecutive output slots
        if (full) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                const uint32_t j = tid + i * THREADS;
                const U k = s_keys[j];
                uint32_t dst = s_delta[uint32_t(k >> shift) & 0xFF] + j;
                if (MSORT_ABLATE) dst = min(dst, n - 1);
                __stcs(out + dst, DEC_OUT ? decode<U, FLOAT>(k) : k);
            }
        } else {
            const uint32_t valid = uint32_t(n - tile_base);
            for (uint32_t j = tid; j < valid; j += THREADS) {
                const U k = s_keys[j];
                uint32_t dst = s_delta[uint32_t(k >> shift) & 0xFF] + j;
                if (MSORT_ABLATE) dst = min(dst, n - 1);
                out[dst] = DEC_OUT ? decode<U, FLOAT>(k) : k;
            }
        }
        if constexpr (kCE) {
            // s_cnt[warp] is this warp's alone from the look-back barrier until the
            // next count barrier: zero it, count the prefetched keys, and let that
            // barrier order every warp's scatter (s_keys reads) before the next ranking
            uint4* z = reinterpret_cast<uint4*>(&s_cnt[warp][0]);
#pragma unroll
            for (int i = lane; i < kRadix / 4; i += 32) z[i] = make_uint4(0, 0, 0, 0);
            __syncwarp();
            counted = next_tile < ntiles;
            if (counted) {
                if (ENC_IN && uint64_t(next_tile) * TILE + TILE <= n) {
#pragma unroll
                    for (int i = 0; i < ITEMS; ++i) keys[i] = encode<U, FLOAT>(keys[i]);
                }
                count_keys();
            }
            tile = next_tile;
            continue;
        }
        zero_counts();  // for the next tile (ordered before its count atomics by the barrier below)
        __syncthreads();
        tile = Cfg::kPrefetch ? next_tile : s_next;
    }
}
// Tile configurations (selectable with MSORT_OS_CFG for tuning; 0 = default).
// OsCfg<threads, keys/thread, ballot mask, blocks/SM, prefetch, look-back
// window, look-back before ranking, count-rank, look-back group, count at end>; measured on
// B200 in profiles/radix_tuning_r1.md: config 0 is the fastest for both key
// widths; the others stay selectable for tuning.
using Cfg32_0 = OsCfg<256, 28, 0x5555555u, 4, true, 2, false, false, 32, true>;  // 7168-key tiles, 4 blocks of 256,
                                            // prefetch, look-back window 2, groups of 32, next tile counted after
                                            // the scatter (best: +0.7% u32, +1.5% f32, +2% zipf vs config 10)
using Cfg32_1 = OsCfg<256, 28, 0x5555555u, 4, true, 4, false, false, 0>;   // tile-by-tile look-back only
using Cfg32_2 = OsCfg<256, 28, 0x5555555u, 4, true, 4, false, false, 16>;  // look-back groups of 16
using Cfg32_3 = OsCfg<256, 28, 0x5555555u, 4, true, 2, false, false, 64>;  // window 2, look-back groups of 64
using Cfg32_4 = OsCfg<256, 28, 0x5555555u, 4, true, 4, false, false, 32>;  // look-back groups of 32
using Cfg32_5 = OsCfg<256, 28, 0x5555555u, 4, true, 6, false, false, 32>;  // window 6, groups of 32
using Cfg32_6 = OsCfg<256, 28, 0x5555555u, 4, true, 4, false, true>;       // count atomic's return = rank
using Cfg32_7 = OsCfg<256, 28, 0x5555555u, 4, true, 1, false, false, 32>;  // window 1, groups of 32
using Cfg32_8 = OsCfg<256, 24, 0x555555u, 5, true, 2, false, false, 32>;   // 6144-key tiles, 5 blocks/SM (40 warps)
using Cfg32_9 = OsCfg<256, 20, 0x55555u, 6, true, 2, false, false, 32>;    // 5120-key tiles, 6 blocks/SM (48 warps)
using Cfg32_10 = OsCfg<256, 28, 0x5555555u, 4, true, 2, false, false, 32>;  // config 0 with the count at the tile's start (4 barriers)
using Cfg32_11 = OsCfg<256, 28, 0x5555555u, 4, true, 4, false, false, 32, true>;  // config 0 with look-back window 4
using Cfg32_12 = OsCfg<256, 28, 0x5555555u, 4, true, 2, false, false, 16, true>;  // config 0 with look-back groups of 16
using Cfg64_0 = OsCfg<256, 14, 0x1555u, 4, true, 4, false, false, 16>;     // prefetch, groups of 16 (best)
using Cfg64_1 = OsCfg<256, 14, 0x1555u, 4, true, 4, false, false, 0>;      // tile-by-tile look-back only
using Cfg64_2 = OsCfg<256, 14, 0x1555u, 4, true, 4, false, false, 8>;      // groups of 8
using Cfg64_3 = OsCfg<256, 14, 0x1555u, 4, true, 4, false, false, 32>;     // groups of 32
using Cfg64_4 = OsCfg<256, 14, 0x1555u, 4, true, 4, false, false, 16, true>;  // config 0 + next tile counted after the scatter (-3%)

constexpr uint32_t kMinTile32 = 256 * 20;  // smallest u32 tile above (sizes the status array)
constexpr uint32_t kMinTile64 = 256 * 14;  // smallest u64 tile above

int env_cfg() {
    static int v = -1;
    if (v < 0) {
        const char* e = std::getenv("MSORT_OS_CFG");
        v = e ? std::atoi(e) : 0;
        if (v < 0 || v > 12) v = 0;
    }
    return v;
}

__global__ void rank_probe_kernel(uint32_t seed, uint32_t* bad);

std::atomic<int> g_rank_ok[64];  // per device: 0 unknown, 1 lane-ordered, -1 not

bool atomic_rank_ok_impl() {
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) return false;
    int v = g_rank_ok[dev].load();
    if (v != 0) return v > 0;
    const char* e = std::getenv("MSORT_ATOMIC_RANK");
    if (e && e[0] == '0') {
        g_rank_ok[dev] = -1;
        return false;
    }
    uint32_t* bad = nullptr;
    bool ok = false;
    if (cudaMalloc(&bad, 4) == cudaSuccess && cudaMemset(bad, 0, 4) == cudaSuccess) {
        rank_probe_kernel<<<592, 256>>>(0x2545F491u, bad);
        uint32_t hb = 1;
        if (cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost) == cudaSuccess) ok = hb == 0;
    }
    if (bad) cudaFree(bad);
    cudaGetLastError();
    g_rank_ok[dev] = ok ? 1 : -1;
    return ok;
}

int sm_count() {
    int dev = 0, count = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&count, cudaDevAttrMultiProcessorCount, dev);
    return count > 0 ? count : 148;
}

// Self-test of lane-ordered shared-memory atomics (see STABLE above): random
// digit patterns of 1..8 bits, warp-private counters, compare every returned
// value with the match-based stable rank.
__global__ void __launch_bounds__(256) rank_probe_kernel(uint32_t seed, uint32_t* bad) {
    __shared__ uint32_t cnt[8][kRadix];
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 8 * kRadix; i += blockDim.x) (&cnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t lt = lanemask_lt();
    uint32_t h = seed ^ (blockIdx.x * 0x9E3779B9u) ^ (threadIdx.x * 0x85EBCA6Bu);
    for (int r = 0; r < 256; ++r) {
        h ^= h << 13;
        h ^= h >> 17;
        h ^= h << 5;
        const uint32_t d = h & ((2u << (r & 7)) - 1u);  // 1..8 significant bits
        const uint32_t before = cnt[warp][d];
        __syncwarp();
        const uint32_t got = atomicAdd(&cnt[warp][d], 1u);
        const uint32_t want = before + __popc(ballot_match8(d) & lt);
        if (got != want) atomicAdd(bad, 1u);
        __syncwarp();
    }
}

template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT, class Cfg, bool STABLE>
cudaError_t launch_onesweep_c(const void* in, void* out, uint64_t n, int pass, const RadixWs& ws,
                              const uint32_t* base_row, uint32_t tag, cudaStream_t st, uint32_t hot, bool hot_on) {
    const size_t smem = Cfg::template smem_bytes<U, STABLE>();
    auto kern = onesweep_kernel<U, FLOAT, ENC_IN, DEC_OUT, Cfg, STABLE>;
    // per-device attribute: set on every launch (cheap, and correct when one
    // process drives several GPUs)
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, Cfg::kThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
    const uint64_t tiles = (n + Cfg::kTile - 1) / Cfg::kTile;
    uint64_t grid = uint64_t(per_sm) * sm_count();
    if (grid > tiles) grid = tiles;
    kern<<<unsigned(grid), Cfg::kThreads, smem, st>>>(reinterpret_cast<const U*>(in), reinterpret_cast<U*>(out),
                                                     uint32_t(n), uint32_t(8 * pass), base_row, ws.status,
                                                     ws.counters + pass, tag, ws.gagg + size_t(pass) * ws.groups * kRadix,
                                                     hot, hot_on);
    return cudaGetLastError();
}

template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT, bool STABLE>
cudaError_t launch_onesweep_t(const void* in, void* out, uint64_t n, int pass, const RadixWs& ws,
                              const uint32_t* base_row, uint32_t tag, cudaStream_t st, uint32_t hot, bool hot_on) {
    const int c = env_cfg();
    if constexpr (sizeof(U) == 4) {
        switch (c) {
            case 1: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_1, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 2: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_2, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 3: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_3, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 4: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_4, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 5: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_5, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 6: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_6, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 7: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_7, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 8: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_8, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 9: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_9, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 10: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_10, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 11: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_11, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 12: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_12, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            default: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg32_0, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
        }
    } else {
        switch (c) {
            case 1: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_1, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 2: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_2, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 3: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_3, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 4: case 10: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_4, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            case 5: case 6: case 7: case 8: case 9:
                return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_0, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
            default: return launch_onesweep_c<U, FLOAT, ENC_IN, DEC_OUT, Cfg64_0, STABLE>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
        }
    }
}

template <typename U>
cudaError_t launch_onesweep_int(const void* in, void* out, uint64_t n, int pass, int flags, const RadixWs& ws,
                                const uint32_t* base_row, uint32_t tag, cudaStream_t st, uint32_t hot) {
    const bool hot_on = flags & 8;
    if (flags & 4) return launch_onesweep_t<U, false, false, false, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    return launch_onesweep_t<U, false, false, false, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
}

template <typename U>
cudaError_t launch_onesweep_float(const void* in, void* out, uint64_t n, int pass, int flags, const RadixWs& ws,
                                  const uint32_t* base_row, uint32_t tag, cudaStream_t st, uint32_t hot) {
    const bool hot_on = flags & 8;
    const bool enc = flags & 1, dec = flags & 2;
    const bool atom = flags & 4;
    if (enc && dec && atom) return launch_onesweep_t<U, true, true, true, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (dec && !enc && atom) return launch_onesweep_t<U, true, false, true, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (!enc && !dec && atom) return launch_onesweep_t<U, true, false, false, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (enc && dec) return launch_onesweep_t<U, true, true, true, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (enc && (flags & 4)) return launch_onesweep_t<U, true, true, false, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (enc) return launch_onesweep_t<U, true, true, false, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (dec) return launch_onesweep_t<U, true, false, true, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    return launch_onesweep_t<U, true, false, false, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
}

}  // namespace

bool atomic_rank_ok() { return atomic_rank_ok_impl(); }
#if MSORT_ABLATE & 8
}  // namespace msort
extern "C" void msort_debug_lb_stats(unsigned long long* out4, int reset) {
    cudaMemcpyFromSymbol(out4, msort::g_lb_stats, 32);
    if (reset) {
        unsigned long long z[4] = {0, 0, 0, 0};
        cudaMemcpyToSymbol(msort::g_lb_stats, z, 32);
    }
}
namespace msort {
#endif

uint32_t radix_tile_keys(int kt) { return key_bytes(kt) == 4 ? kMinTile32 : kMinTile64; }

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static size_t head_bytes() { return align_up(8 * 4 + 8 * 256 * 4 * 2 + 24 * 4, 256); }

constexpr uint64_t kMinGroup = 8;  // smallest look-back group of the configs above (sizes the allocation)

// look-back group size of the configuration in use (gagg stride; only that much is zeroed per sort)
static uint64_t active_group(int kt) {
    const int c = env_cfg();
    uint32_t gsz;
    if (key_bytes(kt) == 4) {
        constexpr uint32_t G32[13] = {Cfg32_0::kGroup, Cfg32_1::kGroup, Cfg32_2::kGroup, Cfg32_3::kGroup, Cfg32_4::kGroup,
                                      Cfg32_5::kGroup, Cfg32_6::kGroup, Cfg32_7::kGroup, Cfg32_8::kGroup, Cfg32_9::kGroup,
                                      Cfg32_10::kGroup, Cfg32_11::kGroup, Cfg32_12::kGroup};
        gsz = G32[c];
    } else {
        constexpr uint32_t G64[5] = {Cfg64_0::kGroup, Cfg64_1::kGroup, Cfg64_2::kGroup, Cfg64_3::kGroup, Cfg64_4::kGroup};
        gsz = G64[c == 10 ? 4 : (c < 5 ? c : 0)];  // (11, 12: u32 only)
    }
    return gsz ? gsz : kMinGroup;
}

static uint64_t ws_groups(uint64_t tiles) { return tiles / kMinGroup + 1; }

size_t radix_ws_bytes(uint64_t n, int kt) {
    const uint64_t tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    return head_bytes() + align_up(size_t(tiles) * kRadix * 8, 256) +
           size_t(num_passes(kt)) * ws_groups(tiles) * kRadix * 8 + 256;
}

RadixWs radix_ws_layout(void* ws, uint64_t n, int kt) {
    RadixWs w;
    char* p = reinterpret_cast<char*>(ws);
    w.counters = reinterpret_cast<uint32_t*>(p);
    w.hist = w.counters + 8;
    w.base = w.hist + 8 * 256;
    w.trivial = w.base + 8 * 256;
    w.head_bytes = head_bytes();
    w.status = reinterpret_cast<unsigned long long*>(p + w.head_bytes);
    w.tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    w.groups = w.tiles / active_group(kt) + 1;  // <= ws_groups(tiles): the allocation covers any config
    w.gagg = reinterpret_cast<unsigned long long*>(p + w.head_bytes + align_up(size_t(w.tiles) * kRadix * 8, 256));
    w.zero_bytes = w.head_bytes + align_up(size_t(w.tiles) * kRadix * 8, 256) +
                   size_t(num_passes(kt)) * w.groups * kRadix * 8;
    return w;
}

template <typename U, bool FLOAT>
static cudaError_t launch_hist_t(const void* keys, uint64_t n, uint32_t* hist, cudaStream_t st) {
    auto kern = hist_kernel<U, FLOAT>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(HistCfg<U>::kSmem));
    if (e != cudaSuccess) return e;
    const uint64_t vec = n / (16 / sizeof(U)) + 1;
    uint64_t blocks = (vec + uint64_t(kHistThreads) * kHistUnroll - 1) / (uint64_t(kHistThreads) * kHistUnroll);
    const uint64_t cap = uint64_t(sm_count());
    if (blocks > cap) blocks = cap;
    if (blocks == 0) blocks = 1;
    kern<<<unsigned(blocks), kHistThreads, HistCfg<U>::kSmem, st>>>(reinterpret_cast<const U*>(keys), n, hist);
    return cudaGetLastError();
}

cudaError_t launch_histogram(const void* keys, uint64_t n, int kt, uint32_t* hist, cudaStream_t st) {
    const int P = num_passes(kt);
    cudaError_t e = cudaMemsetAsync(hist, 0, size_t(P) * kRadix * 4, st);
    if (e != cudaSuccess || n == 0) return e;
    switch (kt) {
        case 0: return launch_hist_t<uint32_t, false>(keys, n, hist, st);
        case 1: return launch_hist_t<uint64_t, false>(keys, n, hist, st);
        case 2: return launch_hist_t<uint32_t, true>(keys, n, hist, st);
        case 3: return launch_hist_t<uint64_t, true>(keys, n, hist, st);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_scan(const uint32_t* hist, uint32_t* base, uint32_t* trivial, uint64_t n, int kt, cudaStream_t st) {
    scan_kernel<<<num_passes(kt), kRadix, 0, st>>>(hist, base, trivial, n);
    return cudaGetLastError();
}

cudaError_t radix_prologue(const void* keys, uint64_t n, int kt, const RadixWs& ws, cudaStream_t st) {
    cudaError_t e;
    if (ws.epoch == 0) {
        e = cudaMemsetAsync(ws.counters, 0, ws.zero_bytes, st);
    } else {
        // epoch-tagged status words need no zeroing (1.1 GB at 4e9 keys); the
        // per-pass tile counters and the group aggregates (atomic sums) do
        e = cudaMemsetAsync(ws.counters, 0, ws.head_bytes, st);
        if (e == cudaSuccess)
            e = cudaMemsetAsync(ws.gagg, 0, size_t(num_passes(kt)) * ws.groups * kRadix * 8, st);
    }
    if (e != cudaSuccess) return e;
    if ((e = launch_histogram(keys, n, kt, ws.hist, st)) != cudaSuccess) return e;
    return launch_scan(ws.hist, ws.base, ws.trivial, n, kt, st);
}

cudaError_t launch_onesweep(const void* in, void* out, uint64_t n, int kt, int pass, int flags, const RadixWs& ws,
                            const uint32_t* base_row, cudaStream_t st, uint32_t hot) {
    if (n == 0) return cudaSuccess;
    // status words of other passes and of earlier sorts (epochs) are ignored
    const uint32_t tag = ((ws.epoch << 4) + uint32_t(pass) + 1) & 0x3FFFFFFFu;
    switch (kt) {
        case 0: return launch_onesweep_int<uint32_t>(in, out, n, pass, flags, ws, base_row, tag, st, hot);
        case 1: return launch_onesweep_int<uint64_t>(in, out, n, pass, flags, ws, base_row, tag, st, hot);
        case 2: return launch_onesweep_float<uint32_t>(in, out, n, pass, flags, ws, base_row, tag, st, hot);
        case 3: return launch_onesweep_float<uint64_t>(in, out, n, pass, flags, ws, base_row, tag, st, hot);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace msort
