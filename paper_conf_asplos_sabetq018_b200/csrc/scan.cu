// scan.cu -- device-wide exclusive prefix sum (reduce / scan-partials / downsweep).
//
// Used for the CSR node array (Fig. 10a "Node" row = exclusive scan of out-degrees,
// L903-925), the padded chunk offsets, and the virtual-node pointers (Fig. 10b edge-pointer
// row "0 3 6 9" = exclusive scan of family sizes ceil(d/K), Def. 2(iii)).
// Three launches; each tile of 4096 items is read coalesced, transposed through shared
// memory so each thread owns 16 consecutive items, and written back coalesced.
#include "internal.cuh"

namespace tigr {
namespace {

constexpr int kScanThreads = 256;
constexpr int kItems = 16;
constexpr int kTile = kScanThreads * kItems;

__device__ __forceinline__ uint64_t scan_value(const uint32_t* in, uint64_t k, int kind, uint32_t div) {
    uint32_t x = in[k];
    if (kind == SCAN_CEIL_DIV) return (uint64_t)(x / div) + (x % div != 0);
    return x;
}

__device__ __forceinline__ uint64_t warp_sum(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// inclusive warp scan
__device__ __forceinline__ uint64_t warp_iscan(uint64_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += t;
    }
    return v;
}

// exclusive block scan of one value per thread; returns exclusive prefix, *total = block sum
template <int NT>
__device__ __forceinline__ uint64_t block_escan(uint64_t v, uint64_t* total) {
    __shared__ uint64_t warp_tot[NT / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint64_t inc = warp_iscan(v);
    if (lane == 31) warp_tot[warp] = inc;
    __syncthreads();
    if (warp == 0) {
        uint64_t t = (lane < NT / 32) ? warp_tot[lane] : 0;
        uint64_t ti = warp_iscan(t);
        if (lane < NT / 32) warp_tot[lane] = ti - t;
        if (lane == NT / 32 - 1) *total = ti;
    }
    __syncthreads();
    uint64_t r = inc - v + warp_tot[warp];
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(kScanThreads) k_reduce(const uint32_t* __restrict__ in, uint64_t count,
                                                         int kind, uint32_t div, uint64_t* partials) {
    const uint64_t base = (uint64_t)blockIdx.x * kTile;
    uint64_t s = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        uint64_t idx = base + (uint64_t)k * kScanThreads + threadIdx.x;
        if (idx < count) s += scan_value(in, idx, kind, div);
    }
    s = warp_sum(s);
    __shared__ uint64_t ws[kScanThreads / 32];
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t t = 0;
        for (int w = 0; w < kScanThreads / 32; ++w) t += ws[w];
        partials[blockIdx.x] = t;
    }
}

// single block: exclusive scan of partials[0..nb) in place, partials[nb] = total
__global__ void __launch_bounds__(1024) k_scan_partials(uint64_t* partials, uint64_t nb) {
    __shared__ uint64_t carry_s;
    __shared__ uint64_t tot_s;
    if (threadIdx.x == 0) carry_s = 0;
    __syncthreads();
    for (uint64_t off = 0; off < nb; off += 1024) {
        uint64_t idx = off + threadIdx.x;
        uint64_t v = idx < nb ? partials[idx] : 0;
        uint64_t ex = block_escan<1024>(v, &tot_s);
        uint64_t carry = carry_s;
        if (idx < nb) partials[idx] = carry + ex;
        __syncthreads();
        if (threadIdx.x == 0) carry_s = carry + tot_s;
        __syncthreads();
    }
    if (threadIdx.x == 0) partials[nb] = carry_s;
}

template <class OutT>
__global__ void __launch_bounds__(kScanThreads) k_downsweep(const uint32_t* __restrict__ in, uint64_t count,
                                                            int kind, uint32_t div,
                                                            const uint64_t* __restrict__ partials,
                                                            uint64_t nb, OutT* __restrict__ out) {
    // padded to avoid 16-way bank conflicts on the per-thread-contiguous reads
    __shared__ uint64_t tile[kTile + kTile / 32];
    __shared__ uint64_t tot_s;
    const uint64_t base = (uint64_t)blockIdx.x * kTile;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        int li = k * kScanThreads + threadIdx.x;
        uint64_t idx = base + li;
        tile[li + li / 32] = idx < count ? scan_value(in, idx, kind, div) : 0;
    }
    __syncthreads();
    uint64_t vals[kItems];
    uint64_t s = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        int li = threadIdx.x * kItems + k;
        vals[k] = tile[li + li / 32];
        s += vals[k];
    }
    uint64_t run = block_escan<kScanThreads>(s, &tot_s) + partials[blockIdx.x];
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        int li = threadIdx.x * kItems + k;
        tile[li + li / 32] = run;
        run += vals[k];
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        int li = k * kScanThreads + threadIdx.x;
        uint64_t idx = base + li;
        if (idx < count) out[idx] = (OutT)tile[li + li / 32];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[count] = (OutT)partials[nb];
}

template <class OutT>
tigr_status scan_impl(const uint32_t* in, uint64_t count, ScanKind kind, uint32_t div, OutT* out,
                      cudaStream_t s, uint64_t* total_host) {
    const uint64_t nb = (count + kTile - 1) / kTile;
    TmpBuf partials;
    TIGR_TRY(partials.alloc(sizeof(uint64_t) * (nb + 1), s));
    if (nb) {
        k_reduce<<<(unsigned)nb, kScanThreads, 0, s>>>(in, count, kind, div, partials.as<uint64_t>());
        TIGR_CKL("scan reduce");
    }
    k_scan_partials<<<1, 1024, 0, s>>>(partials.as<uint64_t>(), nb);
    TIGR_CKL("scan partials");
    k_downsweep<OutT><<<(unsigned)(nb ? nb : 1), kScanThreads, 0, s>>>(in, count, kind, div,
                                                                   partials.as<uint64_t>(), nb, out);
    TIGR_CKL("scan downsweep");
    if (total_host) {
        TIGR_CK(cudaMemcpyAsync(total_host, partials.as<uint64_t>() + nb, sizeof(uint64_t),
                                cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaStreamSynchronize(s));
    }
    return TIGR_OK;
}

}  // namespace

tigr_status exclusive_scan_u64(const uint32_t* in, uint64_t count, ScanKind kind, uint32_t div,
                               uint64_t* out, cudaStream_t s) {
    return scan_impl<uint64_t>(in, count, kind, div, out, s, nullptr);
}

tigr_status exclusive_scan_u32(const uint32_t* in, uint64_t count, ScanKind kind, uint32_t div,
                               uint32_t* out, cudaStream_t s, uint64_t* total_host) {
    return scan_impl<uint32_t>(in, count, kind, div, out, s, total_host);
}

}  // namespace tigr
