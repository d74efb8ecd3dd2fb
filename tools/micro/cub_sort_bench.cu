// Reference point only (not product code): CUB radix sort of 268M (u32 key, u32 value) pairs
// on 24-bit keys, to calibrate libtigr's own onesweep CSR build.
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdint>

__global__ void fill(uint32_t* k, uint32_t* v, uint64_t n) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) {
        uint32_t x = (uint32_t)i * 2654435761u; x ^= x >> 13; x *= 0x5bd1e995u; x ^= x >> 15;
        uint32_t r = 0;  // skewed 24-bit key (bit prob 0.24) like R-MAT sources
        for (int b = 0; b < 24; ++b) { x = x * 1664525u + 1013904223u; if ((x >> 16) < 15729) r |= 1u << b; }
        k[i] = r; v[i] = (uint32_t)i;
    }
}

int main() {
    const uint64_t n = 1ull << 28;
    uint32_t *k0, *k1, *v0, *v1;
    cudaMalloc(&k0, n * 4); cudaMalloc(&k1, n * 4); cudaMalloc(&v0, n * 4); cudaMalloc(&v1, n * 4);
    fill<<<(n + 255) / 256, 256>>>(k0, v0, n);
    size_t tmp = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, tmp, k0, k1, v0, v1, (int)n, 0, 24);
    void* t; cudaMalloc(&t, tmp);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int r = 0; r < 4; ++r) {
        cudaEventRecord(e0);
        cub::DeviceRadixSort::SortPairs(t, tmp, k0, k1, v0, v1, (int)n, 0, 24);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        printf("cub SortPairs 2^28 u32/u32 24-bit: %.3f ms (%.1f Gpairs/s)\n", ms, n / (ms * 1e-3) / 1e9);
    }
    printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
}
