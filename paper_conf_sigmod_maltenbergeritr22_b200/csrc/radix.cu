// radix.cu - per-GPU LSD radix sort of one key chunk.
//
// Paper: §5.1 "Single-GPU Sorting".  The chunk sort is
// an LSB radix sort whose passes read and write the keys once each, because
// the digit histogram is "calculated once" up front and the prefix sum is
// "decoupled" (Thrust >= 1.11 / onesweep).  This file is a
// from-scratch sm_100a onesweep:
//   hist_kernel      one read of the chunk -> P digit histograms (S2)
//   scan_kernel      exclusive prefix per pass -> global digit bases (S2)
//   onesweep_kernel  per tile: warp match-based stable ranking, block digit
//                    counts, decoupled look-back across tiles for the global
//                    digit offset, smem staging, coalesced scatter (S3)
// The float codec T (reading Q1) is applied on the first pass's load and T^-1
// on the last pass's store (S1), so no separate codec pass touches HBM.
#include "common.cuh"
#include "kernels.h"

namespace msort {

namespace {

constexpr int kHistThreads = 512;
constexpr int kHistUnroll = 4;

// ---------------------------------------------------------------------------
// S2: digit histograms of T(key) for every pass, one read of the chunk.
// Two sub-histograms per block (even/odd warps) halve same-bin smem atomic
// collisions; each block flushes its counts with one global atomic per bin.
// ---------------------------------------------------------------------------
template <typename U, bool FLOAT>
__global__ void __launch_bounds__(kHistThreads) hist_kernel(const U* __restrict__ in, uint64_t n,
                                                            uint32_t* __restrict__ hist) {
    constexpr int P = sizeof(U);
    constexpr int V = 16 / sizeof(U);  // keys per 16-byte vector
    __shared__ uint32_t sh[2][P][kRadix];
    for (int i = threadIdx.x; i < 2 * P * kRadix; i += blockDim.x) (&sh[0][0][0])[i] = 0;
    __syncthreads();
    uint32_t(*my)[kRadix] = sh[(threadIdx.x >> 5) & 1];

    auto count = [&](U k) {
        const U code = encode<U, FLOAT>(k);
#pragma unroll
        for (int p = 0; p < P; ++p) atomicAdd(&my[p][uint32_t(code >> (8 * p)) & 0xFF], 1u);
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
    for (int i = threadIdx.x; i < P * kRadix; i += blockDim.x) {
        const uint32_t s = (&sh[0][0][0])[i] + (&sh[1][0][0])[i];
        if (s) atomicAdd(&hist[i], s);
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
    const int p = blockIdx.x, d = threadIdx.x, lane = d & 31, warp = d >> 5;
    if (d == 0) any_full = 0;
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
    __syncthreads();
    if (d == 0 && trivial) trivial[p] = any_full;
}

// ---------------------------------------------------------------------------
// S3: one onesweep pass.
// ---------------------------------------------------------------------------
constexpr unsigned long long kFlagAgg = 1ull, kFlagIncl = 2ull;

__device__ __forceinline__ unsigned long long pack_status(unsigned long long flag, uint32_t tag, uint32_t count) {
    return (flag << 62) | (uint64_t(tag & 0x3FFFFFFFu) << 32) | count;
}

template <typename U>
struct OnesweepCfg;
template <>
struct OnesweepCfg<uint32_t> {
    static constexpr int kThreads = 384;
    static constexpr int kItems = 20;
};
template <>
struct OnesweepCfg<uint64_t> {
    static constexpr int kThreads = 384;
    static constexpr int kItems = 12;
};

template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT>
__global__ void __launch_bounds__(OnesweepCfg<U>::kThreads, 2)
    onesweep_kernel(const U* __restrict__ in, U* __restrict__ out, uint32_t n, uint32_t shift,
                    const uint32_t* __restrict__ base, unsigned long long* __restrict__ status,
                    uint32_t* __restrict__ tile_counter, uint32_t tag) {
    constexpr int THREADS = OnesweepCfg<U>::kThreads;
    constexpr int ITEMS = OnesweepCfg<U>::kItems;
    constexpr int WARPS = THREADS / 32;
    constexpr uint32_t TILE = THREADS * ITEMS;
    static_assert(THREADS >= kRadix, "one thread per digit in the look-back");

    extern __shared__ __align__(16) unsigned char smem_raw[];
    U* s_keys = reinterpret_cast<U*>(smem_raw);
    __shared__ uint32_t s_wcnt[WARPS][kRadix];  // per-warp digit counts, then per-warp exclusive offsets
    __shared__ uint32_t s_total[kRadix];
    __shared__ uint32_t s_dstart[kRadix];
    __shared__ uint32_t s_delta[kRadix];
    __shared__ uint32_t s_wsum[kRadix / 32];
    __shared__ uint32_t s_tile;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // Tile ids in launch-independent arrival order: every lower tile has
    // already started, so the look-back below always makes progress.
    if (tid == 0) s_tile = atomicAdd(tile_counter, 1u);
    for (int i = tid; i < WARPS * kRadix; i += THREADS) (&s_wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t tile_base = uint64_t(tile) * TILE;
    const bool full = tile_base + TILE <= n;

    // --- load (warp-striped: warp w owns keys [w*32*ITEMS, (w+1)*32*ITEMS) of the tile)
    U keys[ITEMS];
    const uint64_t first = tile_base + uint64_t(warp) * 32 * ITEMS + lane;
    const U* src = in + first;
    if (full) {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) keys[i] = __ldcs(src + i * 32);
#pragma unroll
        for (int i = 0; i < ITEMS; ++i)
            if (ENC_IN) keys[i] = encode<U, FLOAT>(keys[i]);
    } else {
        // out-of-range slots get the largest code: they rank after every real
        // key of digit 255 and are never stored (see scatter bound)
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const bool ok = first + uint64_t(i) * 32 < n;
            U k = ok ? src[i * 32] : U(0);
            if (ENC_IN) k = encode<U, FLOAT>(k);
            keys[i] = ok ? k : ~U(0);
        }
    }

    // --- stable warp-level ranking: peers with the same digit via match.any;
    // the lowest peer bumps the warp's digit counter for the whole group.
    uint32_t rk[ITEMS];
    const uint32_t lt = lanemask_lt();
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        const uint32_t d = uint32_t(keys[i] >> shift) & 0xFF;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        const uint32_t below = __popc(peers & lt);
        const int leader = __ffs(peers) - 1;
        uint32_t old = 0;
        if (below == 0) old = atomicAdd(&s_wcnt[warp][d], uint32_t(__popc(peers)));
        old = __shfl_sync(0xffffffffu, old, leader);
        rk[i] = (old + below) | (d << 16);
    }
    __syncthreads();

    // --- block digit totals, per-warp exclusive offsets; publish aggregates
    if (tid < kRadix) {
        const int d = tid;
        uint32_t sum = 0;
#pragma unroll
        for (int w = 0; w < WARPS; ++w) {
            const uint32_t c = s_wcnt[w][d];
            s_wcnt[w][d] = sum;
            sum += c;
        }
        s_total[d] = sum;
        st_relaxed_gpu(&status[uint64_t(tile) * kRadix + d], pack_status(tile == 0 ? kFlagIncl : kFlagAgg, tag, sum));
        // block exclusive scan of totals over digits -> local digit starts
        uint32_t x = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) s_wsum[warp] = x;
        s_dstart[d] = x - sum;  // warp-local exclusive; warp prefix added below
    }
    __syncthreads();
    if (tid < kRadix) {
        uint32_t pre = 0;
        for (int w = 0; w < (tid >> 5); ++w) pre += s_wsum[w];
        s_dstart[tid] += pre;
    }
    __syncthreads();

    // --- stage keys in smem in tile-local digit order
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        const uint32_t d = rk[i] >> 16;
        const uint32_t pos = s_dstart[d] + s_wcnt[warp][d] + (rk[i] & 0xFFFF);
        s_keys[pos] = keys[i];
    }

    // --- decoupled look-back: exclusive count of digit d over all earlier tiles
    if (tid < kRadix) {
        const int d = tid;
        uint32_t excl = 0;
        if (tile > 0) {
            int64_t t = int64_t(tile) - 1;
            while (true) {
                const unsigned long long w = ld_relaxed_gpu(&status[uint64_t(t) * kRadix + d]);
                const unsigned long long flag = w >> 62;
                const uint32_t wtag = uint32_t(w >> 32) & 0x3FFFFFFFu;
                if (flag == 0 || wtag != (tag & 0x3FFFFFFFu)) continue;  // predecessor not published yet
                excl += uint32_t(w);
                if (flag == kFlagIncl) break;
                --t;
            }
            st_relaxed_gpu(&status[uint64_t(tile) * kRadix + d], pack_status(kFlagIncl, tag, excl + s_total[d]));
        }
        s_delta[d] = base[d] + excl - s_dstart[d];
    }
    __syncthreads();

    // --- scatter: consecutive smem slots of one digit go to consecutive output slots
    if (full) {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t j = tid + i * THREADS;
            const U k = s_keys[j];
            const uint32_t dst = s_delta[uint32_t(k >> shift) & 0xFF] + j;
            __stcs(out + dst, DEC_OUT ? decode<U, FLOAT>(k) : k);
        }
    } else {
        const uint32_t valid = uint32_t(n - tile_base);
        for (uint32_t j = tid; j < valid; j += THREADS) {
            const U k = s_keys[j];
            const uint32_t dst = s_delta[uint32_t(k >> shift) & 0xFF] + j;
            out[dst] = DEC_OUT ? decode<U, FLOAT>(k) : k;
        }
    }
}

template <typename U, bool FLOAT, bool ENC_IN, bool DEC_OUT>
cudaError_t launch_onesweep_t(const void* in, void* out, uint64_t n, int pass, const RadixWs& ws,
                              const uint32_t* base_row, uint32_t tag, cudaStream_t st) {
    using Cfg = OnesweepCfg<U>;
    constexpr uint32_t TILE = Cfg::kThreads * Cfg::kItems;
    const size_t smem = size_t(TILE) * sizeof(U);
    auto kern = onesweep_kernel<U, FLOAT, ENC_IN, DEC_OUT>;
    // per-device attribute: set on every launch (cheap, and correct when one
    // process drives several GPUs)
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
    const uint64_t tiles = (n + TILE - 1) / TILE;
    kern<<<unsigned(tiles), Cfg::kThreads, smem, st>>>(reinterpret_cast<const U*>(in), reinterpret_cast<U*>(out),
                                                      uint32_t(n), uint32_t(8 * pass), base_row, ws.status,
                                                      ws.counters + pass, tag);
    return cudaGetLastError();
}

template <typename U, bool FLOAT>
cudaError_t launch_onesweep_f(const void* in, void* out, uint64_t n, int pass, int flags, const RadixWs& ws,
                              const uint32_t* base_row, uint32_t tag, cudaStream_t st) {
    const bool enc = flags & 1, dec = flags & 2;
    if (!FLOAT || (!enc && !dec)) return launch_onesweep_t<U, FLOAT, false, false>(in, out, n, pass, ws, base_row, tag, st);
    if (enc && dec) return launch_onesweep_t<U, FLOAT, true, true>(in, out, n, pass, ws, base_row, tag, st);
    if (enc) return launch_onesweep_t<U, FLOAT, true, false>(in, out, n, pass, ws, base_row, tag, st);
    return launch_onesweep_t<U, FLOAT, false, true>(in, out, n, pass, ws, base_row, tag, st);
}

int sm_count() {
    static int count = 0;
    if (!count) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&count, cudaDevAttrMultiProcessorCount, dev);
        if (count <= 0) count = 148;
    }
    return count;
}

}  // namespace

uint32_t radix_tile_keys(int kt) {
    return key_bytes(kt) == 4 ? OnesweepCfg<uint32_t>::kThreads * OnesweepCfg<uint32_t>::kItems
                              : OnesweepCfg<uint64_t>::kThreads * OnesweepCfg<uint64_t>::kItems;
}

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

size_t radix_ws_bytes(uint64_t n, int kt) {
    const uint64_t tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    const size_t head = align_up(8 * 4 + 8 * 256 * 4 * 2 + 8 * 4, 256);
    return head + align_up(size_t(tiles) * kRadix * 8, 256) + 256;
}

RadixWs radix_ws_layout(void* ws, uint64_t n, int kt) {
    RadixWs w;
    char* p = reinterpret_cast<char*>(ws);
    w.counters = reinterpret_cast<uint32_t*>(p);
    w.hist = w.counters + 8;
    w.base = w.hist + 8 * 256;
    w.trivial = w.base + 8 * 256;
    w.head_bytes = align_up(8 * 4 + 8 * 256 * 4 * 2 + 8 * 4, 256);
    w.status = reinterpret_cast<unsigned long long*>(p + w.head_bytes);
    w.tiles = (n + radix_tile_keys(kt) - 1) / radix_tile_keys(kt);
    return w;
}

cudaError_t launch_histogram(const void* keys, uint64_t n, int kt, uint32_t* hist, cudaStream_t st) {
    const int P = num_passes(kt);
    cudaError_t e = cudaMemsetAsync(hist, 0, size_t(P) * kRadix * 4, st);
    if (e != cudaSuccess || n == 0) return e;
    const uint64_t vec = n / (16 / key_bytes(kt)) + 1;
    uint64_t blocks = (vec + kHistThreads * kHistUnroll - 1) / (kHistThreads * kHistUnroll);
    const uint64_t cap = uint64_t(sm_count()) * 4;
    if (blocks > cap) blocks = cap;
    if (blocks == 0) blocks = 1;
    switch (kt) {
        case 0: hist_kernel<uint32_t, false><<<unsigned(blocks), kHistThreads, 0, st>>>((const uint32_t*)keys, n, hist); break;
        case 1: hist_kernel<uint64_t, false><<<unsigned(blocks), kHistThreads, 0, st>>>((const uint64_t*)keys, n, hist); break;
        case 2: hist_kernel<uint32_t, true><<<unsigned(blocks), kHistThreads, 0, st>>>((const uint32_t*)keys, n, hist); break;
        case 3: hist_kernel<uint64_t, true><<<unsigned(blocks), kHistThreads, 0, st>>>((const uint64_t*)keys, n, hist); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_scan(const uint32_t* hist, uint32_t* base, uint32_t* trivial, uint64_t n, int kt, cudaStream_t st) {
    scan_kernel<<<num_passes(kt), kRadix, 0, st>>>(hist, base, trivial, n);
    return cudaGetLastError();
}

cudaError_t radix_prologue(const void* keys, uint64_t n, int kt, const RadixWs& ws, cudaStream_t st) {
    cudaError_t e = cudaMemsetAsync(ws.counters, 0, ws.head_bytes + size_t(ws.tiles) * kRadix * 8, st);
    if (e != cudaSuccess) return e;
    if ((e = launch_histogram(keys, n, kt, ws.hist, st)) != cudaSuccess) return e;
    return launch_scan(ws.hist, ws.base, ws.trivial, n, kt, st);
}

cudaError_t launch_onesweep(const void* in, void* out, uint64_t n, int kt, int pass, int flags, const RadixWs& ws,
                            const uint32_t* base_row, cudaStream_t st) {
    if (n == 0) return cudaSuccess;
    const uint32_t tag = uint32_t(pass) + 1;  // status words of other passes are ignored
    switch (kt) {
        case 0: return launch_onesweep_f<uint32_t, false>(in, out, n, pass, flags, ws, base_row, tag, st);
        case 1: return launch_onesweep_f<uint64_t, false>(in, out, n, pass, flags, ws, base_row, tag, st);
        case 2: return launch_onesweep_f<uint32_t, true>(in, out, n, pass, flags, ws, base_row, tag, st);
        case 3: return launch_onesweep_f<uint64_t, true>(in, out, n, pass, flags, ws, base_row, tag, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace msort
