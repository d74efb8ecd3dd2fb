// frontier.cu -- the active-node queue build and the dispatch of the frontier relax
// (§8(f) NEXT-3).  The relax kernel itself and its design notes are in
// frontier_kernel.cuh, instantiated per algorithm by frontier_{bfs,sssp,sswp,cc}.cu.
#include <algorithm>

#include "internal.cuh"
#include "relax.cuh"
#include "vgraph.cuh"

namespace tigr {

namespace {
constexpr int kFqThreads = 256;
constexpr int kCompactPer = 8;  // nodes per thread in k_compact
constexpr uint32_t kFull = 0xffffffffu;
}  // namespace

// ------------------------------------------------------------------------------------------
// queue build: nodes stamped for iteration it + delta that own virtual nodes in [lo, hi)
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kFqThreads) k_compact(const uint32_t* __restrict__ stamp,
                                                         const uint4* __restrict__ vinfo, uint32_t n, uint32_t lo,
                                                         uint32_t hi, Ctl* ctl, uint32_t* __restrict__ qv,
                                                         uint32_t* __restrict__ qo, int delta) {
    __shared__ unsigned long long s_warp[kFqThreads / 32];
    __shared__ unsigned long long s_base;
    if (!ctl->cont) return;  // past the fixed point (batched host loop, run.cu); k_init sets cont
    const uint32_t itn = ctl->it + (uint32_t)delta;
    const uint32_t slot = itn & 1u;
    const uint32_t* st = stamp + (uint64_t)slot * n;
    uint32_t* ov = qv + (uint64_t)slot * n;
    uint32_t* oo = qo + (uint64_t)slot * n;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr uint32_t kTileNodes = kFqThreads * kCompactPer;
    for (uint64_t tile0 = (uint64_t)blockIdx.x * kTileNodes; tile0 < n; tile0 += (uint64_t)gridDim.x * kTileNodes) {
        const uint64_t v0 = tile0 + (uint64_t)threadIdx.x * kCompactPer;
        uint32_t m[kCompactPer];
        unsigned long long mine = 0;  // (entries << 32) | vnodes of this thread's nodes
#pragma unroll
        for (int q = 0; q < kCompactPer; ++q) {
            const uint64_t v = v0 + q;
            m[q] = 0;
            if (v < n && __ldg(st + v) == itn) {
                const uint4 info = __ldg(vinfo + v);
                if (info.w && info.z >= lo && info.z < hi) m[q] = info.w;
            }
            if (m[q]) mine += (1ull << 32) | m[q];
        }
        // block exclusive scan of the packed counts (no carry: vnodes < 2^32)
        unsigned long long inc = mine;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long y = __shfl_up_sync(kFull, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) s_warp[wid] = inc;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long run = 0;
            for (int w = 0; w < kFqThreads / 32; ++w) { const unsigned long long t = s_warp[w]; s_warp[w] = run; run += t; }
            s_base = run ? atomicAdd(&ctl->qpack[slot], run) : 0ull;
        }
        __syncthreads();
        unsigned long long pos = s_base + s_warp[wid] + (inc - mine);
        __syncthreads();  // s_warp / s_base reused by the next tile
#pragma unroll
        for (int q = 0; q < kCompactPer; ++q) {
            if (!m[q]) continue;
            const uint32_t e = (uint32_t)(pos >> 32);
            ov[e] = (uint32_t)(v0 + q);
            oo[e] = (uint32_t)pos;
            pos += (1ull << 32) | m[q];
        }
    }
}

// ------------------------------------------------------------------------------------------
// dispatch
// ------------------------------------------------------------------------------------------

FqFn relax_fq_kernel_bfs(int layout, int unit, bool bsp, bool stats);
FqFn relax_fq_kernel_sssp(int layout, int unit, bool bsp, bool stats);
FqFn relax_fq_kernel_sswp(int layout, int unit, bool bsp, bool stats);
FqFn relax_fq_kernel_cc(int layout, int unit, bool bsp, bool stats);

FqFn relax_fq_kernel(int algo, int layout, int unit, bool bsp, bool stats) {
    switch (algo) {
        case TIGR_BFS: return relax_fq_kernel_bfs(layout, unit, bsp, stats);
        case TIGR_SSSP: return relax_fq_kernel_sssp(layout, unit, bsp, stats);
        case TIGR_CC: return relax_fq_kernel_cc(layout, unit, bsp, stats);
        case TIGR_SSWP: return relax_fq_kernel_sswp(layout, unit, bsp, stats);
    }
    return nullptr;
}
unsigned relax_fq_grid(FqFn fn) {
    int per_sm = 0, dev = 0, sms = 148;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kFqThreads, 0);
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return (unsigned)(sms * (per_sm > 0 ? per_sm : 1));
}

int relax_fq_threads() { return kFqThreads; }

tigr_status compact_launch(const tigr_vgraph* vg, Ctl* ctl, int delta, cudaStream_t s) {
    const uint32_t n = vg->g->n;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t tiles = ((uint64_t)n + kFqThreads * kCompactPer - 1) / (kFqThreads * kCompactPer);
    const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(tiles, (uint64_t)sms * 8));
    k_compact<<<grid, kFqThreads, 0, s>>>(vg->ws.stamp.as<uint32_t>(), vg->vinfo.as<uint4>(), n, vg->lo, vg->hi, ctl,
                                          const_cast<uint32_t*>(vg->ws.qv.as<uint32_t>()),
                                          const_cast<uint32_t*>(vg->ws.qo.as<uint32_t>()), delta);
    TIGR_CK(cudaGetLastError());
    return TIGR_OK;
}

}  // namespace tigr
