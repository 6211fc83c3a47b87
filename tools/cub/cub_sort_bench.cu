// Library context only (never the product path): CUB DeviceRadixSort keys-only
// on B200, to put the hand-written onesweep numbers next to NVIDIA's library.
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
__global__ void fill(uint32_t* k, size_t n, uint64_t seed) {
    for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i < n; i += size_t(gridDim.x) * blockDim.x) {
        uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
        k[i] = uint32_t(z >> 32);
    }
}
int main(int argc, char** argv) {
    size_t n = argc > 1 ? size_t(atof(argv[1])) : 1000000000ull;
    uint32_t *a, *b;
    cudaMalloc(&a, n * 4); cudaMalloc(&b, n * 4);
    void* tmp = nullptr; size_t tb = 0;
    cub::DoubleBuffer<uint32_t> db(a, b);
    cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int64_t)n);
    cudaMalloc(&tmp, tb);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e9, sum = 0; int reps = 5;
    for (int r = 0; r < reps + 2; ++r) {
        fill<<<1184, 256>>>(db.Current(), n, 1);
        cudaEventRecord(e0);
        cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int64_t)n);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (r >= 2) { sum += ms; if (ms < best) best = ms; }
    }
    printf("{\"lib\": \"cub::DeviceRadixSort::SortKeys u32\", \"n\": %zu, \"ms_mean\": %.3f, \"ms_best\": %.3f, \"gkeys_s\": %.2f}\n",
           n, sum / reps, best, n / (sum / reps) / 1e6);
    return 0;
}
