// gather_ceiling.cu -- measured ceiling of random 4-byte gathers on this GPU (measurement
// infrastructure for bench.py, not part of libtigr).
//
// The frontier relax kernels (frontier_kernel.cuh) read one 4-byte target value per processed
// arc at a data-dependent address; each such read moves a 32-byte sector through L1/L2, so
// their speed is set by the random-gather rate of the memory hierarchy rather than by the HBM
// byte model alone.  This kernel measures that rate: every thread draws uniform indices into an
// array of n 32-bit words with a counter-based hash (no index stream in memory) and sums the
// words it gathers, 8 independent gathers in flight per thread, persistent grid of 148 SMs x
// 8 blocks.  Run on a 64 MB array (L2-resident on B200's 126 MB L2) it is the L2 random-gather
// ceiling the verdict asks for; 2 MB (L1/L2-hot) and 1 GB (HBM) bracket it.
//
//   extern "C" int micro_gather(uint64_t n, uint64_t gathers, int reps, double* ms_best);
// returns 0 and the best-of-reps kernel time in ms for `gathers` random gathers.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint32_t mix(uint64_t x) {  // splitmix64 finaliser
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return (uint32_t)(x ^ (x >> 31));
}

__global__ void __launch_bounds__(256) k_gather(const uint32_t* __restrict__ a, uint64_t n, uint64_t per_thread,
                                                uint32_t* __restrict__ sink) {
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (uint64_t k = 0; k < per_thread; k += 8) {
        uint32_t v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const uint32_t h = mix((t << 24) ^ (k + q));
            v[q] = a[(uint64_t)h * n >> 32];  // uniform in [0, n)
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) acc += v[q];
    }
    if (acc == 0x12345678u) sink[0] = acc;  // keeps the loads alive
}

__global__ void k_fill(uint32_t* a, uint64_t n) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        a[i] = (uint32_t)i;
}

}  // namespace

extern "C" int micro_gather(uint64_t n, uint64_t gathers, int reps, double* ms_best) {
    int dev = 0, sms = 148;
    if (cudaGetDevice(&dev) != cudaSuccess) return -1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t *a = nullptr, *sink = nullptr;
    if (cudaMalloc(&a, n * sizeof(uint32_t)) != cudaSuccess) return -2;
    if (cudaMalloc(&sink, sizeof(uint32_t)) != cudaSuccess) { cudaFree(a); return -2; }
    k_fill<<<sms * 8, 256>>>(a, n);
    const unsigned grid = (unsigned)sms * 8;
    const uint64_t threads = (uint64_t)grid * 256;
    const uint64_t per_thread = ((gathers + threads - 1) / threads + 7) / 8 * 8;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_gather<<<grid, 256>>>(a, n, per_thread, sink);  // warm-up (fills L2)
    double best = 1e30;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(e0);
        k_gather<<<grid, 256>>>(a, n, per_thread, sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        // scale to exactly `gathers` (the grid issues per_thread * threads of them)
        const double scaled = ms * (double)gathers / (double)(per_thread * threads);
        if (scaled < best) best = scaled;
    }
    const cudaError_t err = cudaGetLastError();
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(a);
    cudaFree(sink);
    if (err != cudaSuccess) return -3;
    *ms_best = best;
    return 0;
}

// ---- float64 reductions ---------------------------------------------------------------------
// The PageRank push relax (pr.cu) sends every arc whose accumulator id misses the shared-memory
// hot table to L2 as one fire-and-forget float64 reduction (RED.E.ADD.F64).  This kernel
// measures the rate of such reductions at uniform random addresses of an n-entry float64 array
// (the accumulator's size: L2-resident at scale 24), 8 per thread and step, same grid.
//   extern "C" int micro_red(uint64_t n, uint64_t reds, int reps, double* ms_best);
namespace {
__global__ void __launch_bounds__(256) k_red(double* __restrict__ a, uint64_t n, uint64_t per_thread) {
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (uint64_t k = 0; k < per_thread; k += 8) {
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const uint32_t h = mix((t << 24) ^ (k + q) ^ 0x5bd1e995ull);
            atomicAdd(a + ((uint64_t)h * n >> 32), 1.0);  // result unused: compiles to RED
        }
    }
}
}  // namespace

extern "C" int micro_red(uint64_t n, uint64_t reds, int reps, double* ms_best) {
    int dev = 0, sms = 148;
    if (cudaGetDevice(&dev) != cudaSuccess) return -1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    double* a = nullptr;
    if (cudaMalloc(&a, n * sizeof(double)) != cudaSuccess) return -2;
    cudaMemset(a, 0, n * sizeof(double));
    const unsigned grid = (unsigned)sms * 8;
    const uint64_t threads = (uint64_t)grid * 256;
    const uint64_t per_thread = ((reds + threads - 1) / threads + 7) / 8 * 8;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_red<<<grid, 256>>>(a, n, per_thread);  // warm-up (fills L2)
    double best = 1e30;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(e0);
        k_red<<<grid, 256>>>(a, n, per_thread);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        const double scaled = ms * (double)reds / (double)(per_thread * threads);
        if (scaled < best) best = scaled;
    }
    const cudaError_t err = cudaGetLastError();
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(a);
    if (err != cudaSuccess) return -3;
    *ms_best = best;
    return 0;
}
