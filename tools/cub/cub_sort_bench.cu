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
// num_items as OffsetT: int (CUB's 32-bit offset path, n < 2^31) or int64_t
template <typename OffsetT>
int run(size_t n, const char* name) {
    uint32_t *a, *b;
    cudaMalloc(&a, n * 4); cudaMalloc(&b, n * 4);
    void* tmp = nullptr; size_t tb = 0;
    cub::DoubleBuffer<uint32_t> db(a, b);
    cub::DeviceRadixSort::SortKeys(tmp, tb, db, (OffsetT)n);
    cudaMalloc(&tmp, tb);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e9, sum = 0; int reps = 5;
    for (int r = 0; r < reps + 2; ++r) {
        fill<<<1184, 256>>>(db.Current(), n, 1);
        cudaEventRecord(e0);
        cub::DeviceRadixSort::SortKeys(tmp, tb, db, (OffsetT)n);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (r >= 2) { sum += ms; if (ms < best) best = ms; }
    }
    printf("{\"lib\": \"cub::DeviceRadixSort::SortKeys u32\", \"offsets\": \"%s\", \"n\": %zu, \"ms_mean\": %.3f, "
           "\"ms_best\": %.3f, \"gkeys_s\": %.2f}\n", name, n, sum / reps, best, n / (sum / reps) / 1e6);
    cudaFree(a); cudaFree(b); cudaFree(tmp);
    return 0;
}

int main(int argc, char** argv) {
    size_t n = argc > 1 ? size_t(atof(argv[1])) : 1000000000ull;
    const bool i64 = argc > 2 && argv[2][0] == 'i' && argv[2][3] == '6';
    if (!i64 && n >= (1ull << 31)) { printf("{\"skip\": \"int offsets need n < 2^31\"}\n"); return 0; }
    return i64 ? run<int64_t>(n, "int64") : run<int>(n, "int");
}
