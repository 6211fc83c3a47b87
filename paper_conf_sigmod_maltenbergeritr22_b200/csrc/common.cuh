// common.cuh - shared device helpers of libmsort (CUDA path only).
//
// Key codec T (reading Q1; paper sorts integers/floats/longs/doubles,
// P:3232-3236 §6.3): identity for unsigned integers; for IEEE floats flip all
// bits of negative keys and the sign bit of non-negative ones, so unsigned
// order of T(key) is IEEE totalOrder.  T^-1 restores the exact bits.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace msort {

constexpr int kRadixBits = 8;
constexpr int kRadix = 1 << kRadixBits;

template <typename U>
struct Bits;
template <>
struct Bits<uint32_t> {
    static constexpr int kBits = 32;
    using Signed = int32_t;
};
template <>
struct Bits<uint64_t> {
    static constexpr int kBits = 64;
    using Signed = int64_t;
};

// T: raw bits -> order code.
template <typename U, bool FLOAT>
__device__ __forceinline__ U encode(U u) {
    if constexpr (FLOAT) {
        using S = typename Bits<U>::Signed;
        constexpr U sign = U(1) << (Bits<U>::kBits - 1);
        return u ^ (U(S(u) >> (Bits<U>::kBits - 1)) | sign);
    } else {
        return u;
    }
}

// T^-1: order code -> raw bits.
template <typename U, bool FLOAT>
__device__ __forceinline__ U decode(U c) {
    if constexpr (FLOAT) {
        using S = typename Bits<U>::Signed;
        constexpr U sign = U(1) << (Bits<U>::kBits - 1);
        return c ^ (U(~(S(c) >> (Bits<U>::kBits - 1))) | sign);
    } else {
        return c;
    }
}

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__device__ __forceinline__ unsigned long long ld_relaxed_gpu(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_gpu(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

}  // namespace msort
