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

__device__ __forceinline__ uint32_t ld_relaxed_gpu_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_gpu_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ uint32_t ld_acquire_gpu_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_gpu_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---- TMA bulk copies (cp.async.bulk) + mbarrier, sm_90+ / sm_100a ----------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// arm the barrier with the byte count and start a 1-D bulk copy global -> smem
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

}  // namespace msort
