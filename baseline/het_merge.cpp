// CPU baselines (comparison only, never the product path):
//   het_multiway_merge  the CPU side of the paper's heterogeneous sort, PAPER.md
//                       §5.3: the g sorted GPU chunks are merged on
//                       the host with a parallel multiway merge
//                       (gnu_parallel::multiway_merge, a loser tree)
//   cpu_parallel_sort   GNU parallel mode's sort on all host cores - one of the
//                       paper's CPU library baselines (§6 "CPU Sort Baseline",
//                       P:2258-2266), reported beside the single-thread oracle
// Keys compare by the T order of DESIGN.md reading Q1 (floats: IEEE totalOrder on bits).
#include <parallel/algorithm>
#include <omp.h>

#include <cstdint>
#include <utility>
#include <vector>

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
int merge(const void* const* runs, const uint64_t* lens, int k, void* out, int threads) {
    using It = U*;  // libstdc++ multiseq_selection wants mutable iterators; inputs are only read
    std::vector<std::pair<It, It>> seqs;
    uint64_t total = 0;
    for (int i = 0; i < k; ++i) {
        U* p = const_cast<U*>(static_cast<const U*>(runs[i]));
        seqs.emplace_back(p, p + lens[i]);
        total += lens[i];
    }
    if (threads > 0) omp_set_num_threads(threads);
    __gnu_parallel::multiway_merge(seqs.begin(), seqs.end(), static_cast<U*>(out), total, TLess<U, FLOAT>(),
                                   __gnu_parallel::parallel_tag(threads > 0 ? threads : 0));
    return 0;
}

}  // namespace

extern "C" int het_multiway_merge(const void* const* runs, const uint64_t* lens, int k, void* out, int key_type,
                                  int threads) {
    switch (key_type) {
        case 0: return merge<uint32_t, false>(runs, lens, k, out, threads);
        case 1: return merge<uint64_t, false>(runs, lens, k, out, threads);
        case 2: return merge<uint32_t, true>(runs, lens, k, out, threads);
        case 3: return merge<uint64_t, true>(runs, lens, k, out, threads);
        default: return 1;
    }
}

template <typename U, bool FLOAT>
int psort(void* keys, uint64_t n, int threads) {
    if (threads > 0) omp_set_num_threads(threads);
    U* p = static_cast<U*>(keys);
    __gnu_parallel::sort(p, p + n, TLess<U, FLOAT>(), __gnu_parallel::default_parallel_tag(threads > 0 ? threads : 0));
    return 0;
}

extern "C" int cpu_parallel_sort(void* keys, uint64_t n, int key_type, int threads) {
    switch (key_type) {
        case 0: return psort<uint32_t, false>(keys, n, threads);
        case 1: return psort<uint64_t, false>(keys, n, threads);
        case 2: return psort<uint32_t, true>(keys, n, threads);
        case 3: return psort<uint64_t, true>(keys, n, threads);
        default: return 1;
    }
}

extern "C" int het_max_threads() { return omp_get_max_threads(); }
