// Probe: does a shared-memory atomicAdd(addr, 1) executed by several lanes of
// one warp instruction on the same address return values in lane order?
// (ptxas emits ATOMS.POPC.INC for this pattern.)  Checks random digit patterns.
#include <cstdio>
#include <cstdint>
__global__ void probe(const uint32_t* digits, uint32_t* bad, int reps, int bits) {
    __shared__ uint32_t cnt[8][256];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 8 * 256; i += blockDim.x) (&cnt[0][0])[i] = 0;
    __syncthreads();
    uint32_t lt;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
    uint32_t prev[256 / 32];
    for (int r = 0; r < reps; ++r) {
        const uint32_t d = digits[(blockIdx.x * reps + r) * blockDim.x + threadIdx.x] & ((1u << bits) - 1);
        const uint32_t before = cnt[warp][d];  // racy read is fine: only this warp touches its row
        __syncwarp();
        const uint32_t got = atomicAdd(&cnt[warp][d], 1u);
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        const uint32_t want = before + __popc(peers & lt);
        if (got != want) atomicAdd(bad, 1u);
        __syncwarp();
    }
}
int main() {
    const int blocks = 296, threads = 256, reps = 64;
    for (int bits = 1; bits <= 8; bits += (bits < 4 ? 1 : 4)) {
        size_t n = size_t(blocks) * reps * threads;
        uint32_t *d, *bad;
        cudaMalloc(&d, n * 4); cudaMalloc(&bad, 4); cudaMemset(bad, 0, 4);
        uint32_t* h = new uint32_t[n];
        uint64_t s = 88172645463325252ull + bits;
        for (size_t i = 0; i < n; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = uint32_t(s); }
        cudaMemcpy(d, h, n * 4, cudaMemcpyHostToDevice);
        for (int it = 0; it < 20; ++it) probe<<<blocks, threads>>>(d, bad, reps, bits);
        uint32_t hb = 0;
        cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
        printf("bits=%d instructions=%zu mismatches=%u\n", bits, n / 32 * 20, hb);
        cudaFree(d); cudaFree(bad); delete[] h;
    }
    return 0;
}
