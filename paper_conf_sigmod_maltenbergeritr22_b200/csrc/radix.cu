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
//                    warp ranking (lane-ordered smem atomics, or peer masks
//                    from an 8-ballot match / match.any), decoupled look-back
//                    across tiles (64-bit epoch-tagged status words, per-group
//                    aggregates) for the global digit offset, smem staging, coalesced
//                    scatter (S3); the next tile's keys load during the scatter
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
// Cache operators of the onesweep pass's tile loads and scatter stores (build
// parameters).  ld.global.cg keeps the streamed keys out of L1: no L1 fill in
// the data pipe that binds the pass (session 3: 2e9-key u64 pass 7.71 -> 7.13
// ms, u32 / f32 about 1 % faster than ld.global.cs; profiles/radix_tuning_r2.md)
#ifndef MSORT_TILE_LD
#define MSORT_TILE_LD __ldcg
#endif
#ifndef MSORT_TILE_ST
#define MSORT_TILE_ST __stcs
#endif
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
    uint32_t top4 = 0, top_count = 0, top4_count = 0;
    bool taken = false;
    for (int q = 0; q < 4; ++q) {
        if (!taken) atomicMax(&max_bin, (static_cast<unsigned long long>(v) << 8) | unsigned(d));
        __syncthreads();
        const unsigned long long b = max_bin;
        if (q == 0) top_count = uint32_t(b >> 8);
        top4_count += uint32_t(b >> 8);
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
        trivial[24 + p] = top4_count;  // keys on those 4 values
    }
}

// ---------------------------------------------------------------------------
// S3: onesweep pass.
//
// B200 budget (measured, profiles/): at 80% of HBM a pass must move ~2.2
// keys/cycle/SM, while shared memory serves 1 wavefront (128 B)/cycle/SM and
// the integer ALU pipe 2 warp-instructions/cycle/SM; a random 4-byte smem
// access by 32 lanes costs ~3.5 wavefronts (bank conflicts) and MATCH.ANY
// ~60 ADU cycles.  Per tile: per-warp digit counts first ("early counts"), the
// tile aggregate is published before the ranking, and the ranking's atomic
// returns the key's final smem slot (lane-ordered shared atomics, or a peer
// match that mixes an 8-ballot match (ALU) with match.any (ADU) and, for items
// in neither mask, an smem atomicOr mask).
//
// Decoupled look-back: one 64-bit status word per (tile, digit),
//   flag << 62 | tag << 32 | count       (tag = epoch << 4 | pass + 1)
//   AGG  count = the tile's count of digit d;  INCL  count = inclusive count
//   over all tiles up to this one.  A tile walks its predecessors inside its
//   GROUP of kGroup tiles (kLookback words per round), then whole earlier
//   groups through the last tile's INCL word or the group aggregate
//   gagg[grp][d] = tiles << 32 | sum (complete when tiles == kGroup).
// (Round 2 measured a 32-bit variant with group-relative counts and
// per-group published bases: u32 no faster, u64 7% slower - every tile then
// needs the group base, one more dependent L2 round trip; not adopted,
// profiles/radix_tuning_r2.md.)
// ---------------------------------------------------------------------------
constexpr unsigned long long kFlagAgg = 1ull, kFlagIncl = 2ull;

__device__ __forceinline__ unsigned long long pack_status(unsigned long long flag, uint32_t tag, uint32_t count) {
    return (flag << 62) | (uint64_t(tag & 0x3FFFFFFFu) << 32) | count;
}

// Lanes of the warp whose 8-bit digit equals this lane's (8 ballots).  The
// and / setp / vote.ballot / conditional-not sequence per bit is the standard
// 8-ballot peer-match idiom (CUB's warp_matcher_t::match_any in cub/util_ptx.cuh
// uses the same one).
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

// THREADS x ITEMS keys per tile; bit i of BALLOT_MASK: item i of the peer-match
// ranking uses the ballot match (else smem atomicOr); MINB blocks per SM;
// LB = look-back window (status loads per round); GROUP = look-back group
// (tiles); CE = count the prefetched next tile right after this tile's scatter
// (per-warp counter zeroing, no end-of-tile barrier).
template <int THREADS_, int ITEMS_, uint32_t BALLOT_MASK_, int MINB_, int LB_, int GROUP_, bool CE_>
struct OsCfg {
    static constexpr int kThreads = THREADS_;
    static constexpr int kItems = ITEMS_;
    static constexpr uint32_t kBallotMask = BALLOT_MASK_;
    static constexpr int kMinBlocks = MINB_;
    static constexpr int kLookback = LB_;
    static constexpr uint32_t kGroup = GROUP_;
    static constexpr bool kCountEnd = CE_;
    static constexpr int kWarps = THREADS_ / 32;
    static constexpr uint32_t kTile = uint32_t(THREADS_) * ITEMS_;
    static_assert(GROUP_ >= 2, "look-back groups");
    static constexpr bool kAnyOr = (BALLOT_MASK_ & ((ITEMS_ >= 32 ? 0u : (1u << ITEMS_)) - 1u)) !=
                                   ((ITEMS_ >= 32 ? 0u : (1u << ITEMS_)) - 1u);
    // (the atomicOr peer masks exist only in the peer-match ranking, STABLE)
    template <typename U, bool STABLE = true>
    static constexpr size_t smem_bytes() {
        return size_t(kTile) * sizeof(U) + size_t(kWarps) * kRadix * 4 * (kAnyOr && STABLE ? 2 : 1);
    }
};

// Product tile configurations (profiles/radix_tuning_r1.md; a tuning build
// may override single parameters with -DMSORT_W32=4 etc.):
//   u32/f32: 7168-key tiles, 4 blocks of 256 threads per SM, look-back window 2,
//            groups of 32, next tile counted after the scatter (3 barriers)
//   u64/f64: 7680-key tiles, 2 blocks of 512 threads per SM, window 2, groups
//            of 16, next tile counted after the scatter (session 3: 7.78 ms per
//            2e9-key u64 pass vs 8.35 for 3584-key tiles of 256 threads, window
//            1, four barriers; profiles/radix_tuning_r2.md)
#ifndef MSORT_T32
#define MSORT_T32 256
#endif
#ifndef MSORT_I32
#define MSORT_I32 28
#endif
#ifndef MSORT_B32
#define MSORT_B32 4
#endif
#ifndef MSORT_W32
#define MSORT_W32 2
#endif
#ifndef MSORT_G32
#define MSORT_G32 32
#endif
#ifndef MSORT_W64
#define MSORT_W64 2
#endif
#ifndef MSORT_G64
#define MSORT_G64 16
#endif
#ifndef MSORT_LB_SLEEP_NS
#define MSORT_LB_SLEEP_NS 32  // back-off of a look-back poll on an unpublished predecessor
#endif
#ifndef MSORT_BM32
#define MSORT_BM32 0x7777777u  // peer-match ranking: items by the 8-ballot match (3 of 4); items in neither mask use smem atomicOr masks
#endif
#ifndef MSORT_MM32
#define MSORT_MM32 0x8888888u  // peer-match ranking: the 4th item of every 4 by __match_any_sync (ADU pipe)
#endif
#define MSORT_CFG32 OsCfg<MSORT_T32, MSORT_I32, (MSORT_BM32 | MSORT_MM32), MSORT_B32, MSORT_W32, MSORT_G32, true>
#ifndef MSORT_CE64
#define MSORT_CE64 true
#endif
#ifndef MSORT_T64
#define MSORT_T64 512
#endif
#ifndef MSORT_I64
#define MSORT_I64 15
#endif
#ifndef MSORT_B64
#define MSORT_B64 2
#endif
#ifndef MSORT_BM64
#define MSORT_BM64 0x7777u  // as for 4-byte keys: 3 of 4 items by the ballot match ...
#endif
#ifndef MSORT_MM64
#define MSORT_MM64 0x888u   // ... the 4th by match.any (1e9 u64 with a zipf high word: 33.9 -> 31.0 ms)
#endif
#define MSORT_CFG64 OsCfg<MSORT_T64, MSORT_I64, (MSORT_BM64 | MSORT_MM64), MSORT_B64, MSORT_W64, MSORT_G64, MSORT_CE64>
using Cfg32 = MSORT_CFG32;
using Cfg64 = MSORT_CFG64;
template <typename U>
using CfgOf = std::conditional_t<sizeof(U) == 4, Cfg32, Cfg64>;

// STABLE = false: "atomic ranking": each key takes its smem slot with ONE
// shared-memory atomicAdd on its warp's digit counter (no peer match).  The
// order in which lanes of one warp instruction that hit the same counter
// receive their values is not specified by PTX; on sm_100 the hardware serves
// them in lane order (measured: tools/probe/atom_order.cu), which makes the
// ranking stable.  atomic_rank_ok() verifies this on the running GPU once per
// device (rank_probe_kernel) before any stable pass uses it; the first LSD pass
// may use it regardless (nothing has ordered the keys yet).
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
    constexpr uint32_t G = Cfg::kGroup;
    constexpr int W = Cfg::kLookback;
    static_assert(THREADS >= kRadix, "one thread per digit in the look-back");

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
    // high word of a status entry: flag << 30 | tag
    const uint32_t hi_agg = uint32_t(kFlagAgg << 30) | (tag & 0x3FFFFFFFu);
    const uint32_t hi_incl = uint32_t(kFlagIncl << 30) | (tag & 0x3FFFFFFFu);

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
            for (int i = 0; i < ITEMS; ++i) keys[i] = MSORT_TILE_LD(src + i * 32);
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
    // Phase 1 walks the predecessors inside this tile's group, W status words
    // per round (an unpublished predecessor is then polled alone).  Phase 2
    // walks whole earlier groups: a group contributes the inclusive count of
    // its last tile if that is published, else its aggregate word (complete
    // when tiles == G; every tile adds itself right after counting), so a walk
    // of ~30 tiles takes ~3 rounds instead of ~8.  Publishes this tile's
    // inclusive count.
    auto lookback = [&](const int d, const uint32_t tile, const uint32_t my_total) -> uint32_t {
        uint32_t excl = 0;
        if (tile > 0) {
            const uint32_t first = tile / G * G;  // phase 1 covers tiles [first, tile)
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
                if (done) break;
                left -= used;  // (tile 0 is always inclusive)
                p -= used * kRadix;
                if (used == 0) {
                    unsigned long long w;
                    do {
                        __nanosleep(MSORT_LB_SLEEP_NS);
                        w = ld_relaxed_gpu(p);
                    } while (uint32_t(w >> 32) != hi_agg && uint32_t(w >> 32) != hi_incl);
                }
            }
            if (!done) {
                uint32_t h = first / G - 1;  // newest earlier group not consumed (groups 0..h remain)
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
                    if (done || used == h + 1) break;  // (all groups down to 0 consumed)
                    h -= used;
                    if (used == 0) __nanosleep(MSORT_LB_SLEEP_NS);
                }
            }
            st_relaxed_gpu(&status[uint64_t(tile) * kRadix + d], pack_status(kFlagIncl, tag, excl + my_total));
        }
        return excl;
    };

    if (Cfg::kAnyOr && STABLE) {  // (atomic-ranked kernels have no peer-mask array)
        for (int i = tid; i < WARPS * kRadix; i += THREADS) (&s_match[0][0])[i] = 0;
    }
    // per-warp digit counters start at zero; each tile re-zeroes them during or
    // after its scatter (they are dead after the ranking)
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
    if (tile < ntiles) load_tile(tile);
    constexpr bool kCE = Cfg::kCountEnd;
    auto count_keys = [&]() {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) atomicAdd(&s_cnt[warp][uint32_t(keys[i] >> shift) & 0xFF], 1u);
    };
    bool counted = false;  // kCE: this tile's keys were counted at the end of the previous one

    for (;;) {
        if (tile >= ntiles) break;
        const uint64_t tile_base = uint64_t(tile) * TILE;
        const bool full = tile_base + TILE <= n;
        if (ENC_IN && full && !counted) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) keys[i] = encode<U, FLOAT>(keys[i]);
        }
        // --- early counts: per-warp digit histogram (fire-and-forget smem adds)
        if (!(kCE && counted)) count_keys();
        __syncthreads();

        // --- tile totals -> publish aggregate; per-(warp, digit) smem slot bases
        uint32_t my_total = 0, my_start = 0;
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
            atomicAdd(&gagg[uint64_t(tile / G) * kRadix + d], (1ull << 32) | sum);
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
            constexpr uint32_t kMatch = sizeof(U) == 4 ? MSORT_MM32 : MSORT_MM64;  // items by match.any (ADU pipe)
            if ((kMatch >> i) & 1u) {
                peers = __match_any_sync(0xffffffffu, d);
            } else if ((Cfg::kBallotMask >> i) & 1u) {
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

        // --- look-back (after the ranking: its latency overlaps the other
        // warps' ranking), then claim the next tile so that its loads can be
        // issued before (and overlap) this tile's scatter
        if (tid < kRadix) {
            const int d = tid;
            const uint32_t excl = lookback(d, tile, my_total);
            s_delta[d] = base[d] + excl - my_start;
            if (tid == 0) s_next = atomicAdd(tile_counter, 1u);
        }
        __syncthreads();
        // keys[] is dead until the next iteration: its loads fly during the scatter
        const uint32_t next_tile = s_next;
        if (next_tile < ntiles) load_tile(next_tile);

        // --- scatter: consecutive smem slots of one digit go to consecutive output slots
        if (full) {
#pragma unroll
            for (int i = 0; i < ITEMS; ++i) {
                const uint32_t j = tid + i * THREADS;
                const U k = s_keys[j];
                MSORT_TILE_ST(out + s_delta[uint32_t(k >> shift) & 0xFF] + j, DEC_OUT ? decode<U, FLOAT>(k) : k);
            }
        } else {
            const uint32_t valid = uint32_t(n - tile_base);
            for (uint32_t j = tid; j < valid; j += THREADS) {
                const U k = s_keys[j];
                out[s_delta[uint32_t(k >> shift) & 0xFF] + j] = DEC_OUT ? decode<U, FLOAT>(k) : k;
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
        } else {
            zero_counts();  // for the next tile (ordered before its count atomics by the barrier below)
            __syncthreads();
        }
        tile = next_tile;
    }
}

__global__ void rank_probe_kernel(uint32_t seed, uint32_t* bad);

std::atomic<int> g_rank_ok[64];  // per device: 0 unknown, 1 lane-ordered, -1 not

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

// production-configuration check (below): 0 = equal, 1 = mismatch, -1 = could not run
int production_rank_check(cudaStream_t ps);

// Keys for the production check: many equal pass-1 digits (3 bits of byte 1),
// random low byte, so stability is what decides the order of equal digits.
__global__ void rank_check_keys(uint32_t* k32, uint64_t* k64, uint32_t n, uint32_t seed) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        uint32_t h = (i + 1) * 0x9E3779B9u ^ seed;
        h ^= h >> 16;
        h *= 0x85EBCA6Bu;
        h ^= h >> 13;
        const uint32_t key = (h & 0xFFFF00FFu) | (((h >> 8) & 7u) << 8);
        k32[i] = key;
        k64[i] = (uint64_t(h * 0xC2B2AE35u) << 32) | key;
    }
}

__global__ void count_diff(const uint32_t* a, const uint32_t* b, uint64_t words, uint32_t* bad) {
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < words; i += uint64_t(gridDim.x) * blockDim.x)
        if (a[i] != b[i]) atomicAdd(bad, 1u);
}

// The probe runs once per device on a private stream, outside any capture:
// called while the caller's stream (or this thread) is capturing a CUDA graph
// it answers "no" for this call only (the conservative peer-match ranking) and
// probes later; a failing CUDA call is not cached either, only a measured
// lane-order mismatch is.
bool atomic_rank_ok_impl(cudaStream_t caller) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
        cudaGetLastError();
        return false;
    }
    int v = g_rank_ok[dev].load();
    if (v != 0) return v > 0;
    const char* e = std::getenv("MSORT_ATOMIC_RANK");
    if (e && e[0] == '0') {
        g_rank_ok[dev] = -1;
        return false;
    }
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (caller && cudaStreamIsCapturing(caller, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone) return false;
    if (cudaStreamIsCapturing(cudaStreamLegacy, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) {
        cudaGetLastError();  // (a global-mode capture elsewhere forbids the probe's allocations now)
        return false;
    }
    uint32_t* bad = nullptr;
    cudaStream_t ps = nullptr;
    int verdict = 0;  // 0: could not run (not cached)
    if (cudaStreamCreateWithFlags(&ps, cudaStreamNonBlocking) == cudaSuccess && cudaMalloc(&bad, 4) == cudaSuccess &&
        cudaMemsetAsync(bad, 0, 4, ps) == cudaSuccess) {
        rank_probe_kernel<<<592, 256, 0, ps>>>(0x2545F491u, bad);
        uint32_t hb = 1;
        if (cudaGetLastError() == cudaSuccess && cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, ps) == cudaSuccess &&
            cudaStreamSynchronize(ps) == cudaSuccess)
            verdict = hb == 0 ? 1 : -1;
        // and the production kernels themselves: one stable pass with atomic
        // ranking must equal the same pass with peer-match ranking, byte for byte
        if (verdict == 1) {
            const int pc = production_rank_check(ps);
            verdict = pc == 0 ? 1 : (pc > 0 ? -1 : 0);
        }
    }
    if (bad) cudaFree(bad);
    if (ps) cudaStreamDestroy(ps);
    cudaGetLastError();
    if (verdict != 0) g_rank_ok[dev] = verdict;
    return verdict > 0;
}

template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT, bool STABLE>
cudaError_t launch_onesweep_t(const void* in, void* out, uint64_t n, int pass, const RadixWs& ws,
                              const uint32_t* base_row, uint32_t tag, cudaStream_t st, uint32_t hot, bool hot_on) {
    using Cfg = CfgOf<U>;
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
    const size_t gofs = size_t(pass) * ws.groups * kRadix;
    kern<<<unsigned(grid), Cfg::kThreads, smem, st>>>(reinterpret_cast<const U*>(in), reinterpret_cast<U*>(out),
                                                     uint32_t(n), uint32_t(8 * pass), base_row, ws.status,
                                                     ws.counters + pass, tag, ws.gagg + gofs, hot, hot_on);
    return cudaGetLastError();
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
    if (enc && atom) return launch_onesweep_t<U, true, true, false, false>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (enc) return launch_onesweep_t<U, true, true, false, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    if (dec) return launch_onesweep_t<U, true, false, true, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
    return launch_onesweep_t<U, true, false, false, true>(in, out, n, pass, ws, base_row, tag, st, hot, hot_on);
}

}  // namespace

bool atomic_rank_ok(cudaStream_t caller) { return atomic_rank_ok_impl(caller); }

uint32_t radix_tile_keys(int kt) { return key_bytes(kt) == 4 ? Cfg32::kTile : Cfg64::kTile; }
static uint32_t radix_group(int kt) { return key_bytes(kt) == 4 ? Cfg32::kGroup : Cfg64::kGroup; }

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static size_t head_bytes() { return align_up(8 * 4 + 8 * 256 * 4 * 2 + kTrivialWords * 4, 256); }

// Layout: head (counters, hist, bases, trivial) | group aggregates (zeroed per
// sort) | status words (tagged, zeroed when the epoch wraps)
size_t radix_ws_bytes(uint64_t n, int kt) {
    const uint64_t tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    const uint64_t groups = tiles / radix_group(kt) + 1;
    const size_t garr = align_up(size_t(num_passes(kt)) * groups * kRadix * 8, 256);
    return head_bytes() + garr + align_up(size_t(tiles) * kRadix * 8, 256) + 256;
}

RadixWs radix_ws_layout(void* ws, uint64_t n, int kt) {
    RadixWs w;
    char* p = reinterpret_cast<char*>(ws);
    w.counters = reinterpret_cast<uint32_t*>(p);
    w.hist = w.counters + 8;
    w.base = w.hist + 8 * 256;
    w.trivial = w.base + 8 * 256;
    w.head_bytes = head_bytes();
    w.tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    w.groups = w.tiles / radix_group(kt) + 1;
    const size_t garr = align_up(size_t(num_passes(kt)) * w.groups * kRadix * 8, 256);
    w.gagg = reinterpret_cast<unsigned long long*>(p + w.head_bytes);
    w.status = reinterpret_cast<unsigned long long*>(p + w.head_bytes + garr);
    w.gagg_bytes = garr;
    w.zero_bytes = w.head_bytes + garr + align_up(size_t(w.tiles) * kRadix * 8, 256);
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
        // a new tag cycle: no word of any earlier sort (of any size up to the
        // allocation) may keep a tag that comes round again
        e = cudaMemsetAsync(ws.counters, 0, ws.alloc_bytes > ws.zero_bytes ? ws.alloc_bytes : ws.zero_bytes, st);
    } else {
        // tagged status words need no zeroing; the per-pass
        // tile counters and the group aggregates (atomic sums) do
        e = cudaMemsetAsync(ws.counters, 0, ws.head_bytes + ws.gagg_bytes, st);
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

namespace {

template <typename U>
int production_check_t(cudaStream_t ps, U* keys, U* out_a, U* out_b, void* ws_mem, size_t ws_bytes, uint32_t n,
                       uint32_t* bad) {
    const int kt = sizeof(U) == 4 ? 0 : 1;
    RadixWs ws = radix_ws_layout(ws_mem, n, kt);
    ws.epoch = 0;
    auto ok = [](cudaError_t e) { return e == cudaSuccess; };
    for (int stable = 0; stable < 2; ++stable) {
        if (!ok(cudaMemsetAsync(ws_mem, 0, ws_bytes, ps)) || !ok(radix_prologue(keys, n, kt, ws, ps))) return -1;
        // pass 1 (digit = byte 1): flags 4 = atomic ranking, 0 = peer match
        if (!ok(launch_onesweep(keys, stable ? out_b : out_a, n, kt, 1, stable ? 0 : 4, ws, ws.base + 256, ps)))
            return -1;
    }
    count_diff<<<148, 256, 0, ps>>>(reinterpret_cast<const uint32_t*>(out_a), reinterpret_cast<const uint32_t*>(out_b),
                                    uint64_t(n) * sizeof(U) / 4, bad);
    return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int production_rank_check(cudaStream_t ps) {
    const uint32_t n = 6 * Cfg32::kTile + 1237;  // several tiles and a ragged one (both key widths)
    uint32_t* k32 = nullptr;
    uint64_t* k64 = nullptr;
    void* outs = nullptr;
    void* ws = nullptr;
    uint32_t* bad = nullptr;
    const size_t wsb = std::max(radix_ws_bytes(n, 0), radix_ws_bytes(n, 1));
    int rc = -1;
    if (cudaMalloc(&k32, n * 4ull) == cudaSuccess && cudaMalloc(&k64, n * 8ull) == cudaSuccess &&
        cudaMalloc(&outs, n * 16ull) == cudaSuccess && cudaMalloc(&ws, wsb) == cudaSuccess &&
        cudaMalloc(&bad, 4) == cudaSuccess && cudaMemsetAsync(bad, 0, 4, ps) == cudaSuccess) {
        rank_check_keys<<<148, 256, 0, ps>>>(k32, k64, n, 0x6A09E667u);
        char* o = static_cast<char*>(outs);
        if (production_check_t<uint32_t>(ps, k32, reinterpret_cast<uint32_t*>(o), reinterpret_cast<uint32_t*>(o + n * 4ull),
                                         ws, wsb, n, bad) == 0 &&
            production_check_t<uint64_t>(ps, k64, reinterpret_cast<uint64_t*>(o), reinterpret_cast<uint64_t*>(o + n * 8ull),
                                         ws, wsb, n, bad) == 0) {
            uint32_t hb = 1;
            if (cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, ps) == cudaSuccess && cudaStreamSynchronize(ps) == cudaSuccess)
                rc = hb == 0 ? 0 : 1;
        }
    }
    for (void* p : {static_cast<void*>(k32), static_cast<void*>(k64), outs, ws, static_cast<void*>(bad)})
        if (p) cudaFree(p);
    cudaGetLastError();
    return rc;
}

}  // namespace

}  // namespace msort
