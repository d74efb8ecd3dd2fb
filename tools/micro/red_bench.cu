// Microbenchmark: throughput of fire-and-forget global reductions on B200 for different
// target-array sizes and address distributions (uniform / R-MAT-like skew).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

// rmat-ish index: each bit set with prob 0.24 (Graph500 marginal)
__device__ __forceinline__ uint32_t skewed(uint32_t h, uint32_t bits) {
    uint32_t r = 0;
    for (uint32_t b = 0; b < bits; ++b) {
        h = hash32(h + 0x9e3779b9u * (b + 1));
        if ((h & 0xffff) < 15729) r |= 1u << b;  // 0.24 * 65536
    }
    return r;
}

template <int OP>
__global__ void k_red(void* buf, uint32_t mask, uint64_t n_ops, uint32_t mode, uint32_t bits, const uint32_t* idx) {
    uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = tid; i < n_ops; i += stride) {
        uint32_t a;
        if (mode == 0) a = hash32((uint32_t)i * 2654435761u) & mask;
        else a = idx[i];
        if (OP == 0) atomicAdd((double*)buf + a, 1.0);
        else if (OP == 1) atomicAdd((float*)buf + a, 1.0f);
        else if (OP == 2) atomicMin((unsigned*)buf + a, (unsigned)i);
        else if (OP == 3) atomicAdd((unsigned long long*)buf + a, 1ull);
        else if (OP == 4) { double* p = (double*)buf + a; (void)p; asm volatile("" ::: "memory"); }
    }
}

__global__ void k_gen_idx(uint32_t* idx, uint64_t n, uint32_t bits) {
    uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) idx[i] = skewed(hash32((uint32_t)i), bits);
}

int main() {
    const uint64_t n_ops = 1ull << 28;
    void* buf; cudaMalloc(&buf, 1ull << 31);
    cudaMemset(buf, 0, 1ull << 31);
    uint32_t* idx; cudaMalloc(&idx, n_ops * 4);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const char* opn[] = {"f64add", "f32add", "u32min", "u64add", "none"};
    for (int mode = 0; mode < 2; ++mode) {
        for (int lg = 20; lg <= 26; lg += 1) {  // elements
            if (mode == 1) { k_gen_idx<<<(n_ops + 255) / 256, 256>>>(idx, n_ops, lg); cudaDeviceSynchronize(); }
            for (int op = 0; op < 4; ++op) {
                float best = 1e9;
                for (int r = 0; r < 3; ++r) {
                    cudaEventRecord(e0);
                    if (op == 0) k_red<0><<<148 * 8, 256>>>(buf, (1u << lg) - 1, n_ops, mode, lg, idx);
                    if (op == 1) k_red<1><<<148 * 8, 256>>>(buf, (1u << lg) - 1, n_ops, mode, lg, idx);
                    if (op == 2) k_red<2><<<148 * 8, 256>>>(buf, (1u << lg) - 1, n_ops, mode, lg, idx);
                    if (op == 3) k_red<3><<<148 * 8, 256>>>(buf, (1u << lg) - 1, n_ops, mode, lg, idx);
                    cudaEventRecord(e1); cudaEventSynchronize(e1);
                    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
                }
                int esz = (op == 0 || op == 3) ? 8 : 4;
                printf("mode=%s elems=2^%d (%6.1f MB) op=%s  %.3f ms  %.1f G/s\n", mode ? "skew" : "unif", lg,
                       (double)(1ull << lg) * esz / 1e6, opn[op], best, n_ops / (best * 1e-3) / 1e9);
            }
        }
    }
    cudaError_t err = cudaGetLastError();
    printf("err=%s\n", cudaGetErrorString(err));
    return 0;
}
