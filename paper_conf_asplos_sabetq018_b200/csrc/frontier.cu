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
// SSSP / SSWP (bmode 1 / 2) also keep the settled bitmap of k_relax_fq (frontier_kernel.cuh):
//   * bound: the minimum / maximum value over the stamped nodes -- those with arcs in this
//     rank's range on one GPU; every stamped node with replicas (bound_all), since another rank
//     may own their arcs -- into ctl->bound[slot];
//   * settle (delta = 1, i.e. after iteration it): every node whose value is below (SSSP) / at
//     least (SSWP) iteration it's bound is final; its bit is set here, one owner lane per 32-node
//     word (so the relax never issues atomics for it and never re-reads a stale word).
__global__ void __launch_bounds__(kFqThreads) k_compact(const uint32_t* __restrict__ stamp,
                                                         const uint4* __restrict__ vinfo, uint32_t n, uint32_t lo,
                                                         uint32_t hi, Ctl* ctl, uint32_t* __restrict__ qv,
                                                         uint32_t* __restrict__ qo, int delta,
                                                         const uint32_t* __restrict__ val, int bmode, int bound_all,
                                                         uint32_t* __restrict__ settled) {
    __shared__ unsigned long long s_warp[kFqThreads / 32];
    __shared__ unsigned long long s_base;
    if (!ctl->cont) return;  // past the fixed point (batched host loop, run.cu); k_init sets cont
    const uint32_t itn = ctl->it + (uint32_t)delta;
    const uint32_t slot = itn & 1u;
    const uint32_t* st = stamp + (uint64_t)slot * n;
    uint32_t* ov = qv + (uint64_t)slot * n;
    uint32_t* oo = qo + (uint64_t)slot * n;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t bnd = bmode == 2 ? 0u : kInf;
    const bool settle = bmode && settled && delta == 1;
    const uint32_t bcur = settle ? ctl->bound[ctl->it & 1u] : 0u;  // bound of the iteration just run
    constexpr uint32_t kTileNodes = kFqThreads * kCompactPer;
    static_assert(32 % kCompactPer == 0, "a settled word spans whole threads");
    for (uint64_t tile0 = (uint64_t)blockIdx.x * kTileNodes; tile0 < n; tile0 += (uint64_t)gridDim.x * kTileNodes) {
        const uint64_t v0 = tile0 + (uint64_t)threadIdx.x * kCompactPer;
        if (settle) {  // 32 / kCompactPer lanes share one bitmap word
            const uint32_t word = v0 < n ? settled[v0 >> 5] : kFull;
            const int sh = (int)(v0 & 31u);
            uint32_t add = 0;
            if (((word >> sh) & 0xFFu) != 0xFFu) {
#pragma unroll
                for (int q = 0; q < kCompactPer; ++q) {
                    const uint64_t v = v0 + q;
                    if (v < n && !((word >> (sh + q)) & 1u)) {
                        const uint32_t x = val[v];
                        if (bmode == 2 ? x >= bcur : x < bcur) add |= 1u << (sh + q);
                    }
                }
            }
#pragma unroll
            for (int o = 1; o < 32 / kCompactPer; o <<= 1) add |= __shfl_xor_sync(kFull, add, o);
            if ((lane & (32 / kCompactPer - 1)) == 0 && (add & ~word)) settled[v0 >> 5] = word | add;
        }
        uint32_t m[kCompactPer];
        unsigned long long mine = 0;  // (entries << 32) | vnodes of this thread's nodes
#pragma unroll
        for (int q = 0; q < kCompactPer; ++q) {
            const uint64_t v = v0 + q;
            m[q] = 0;
            if (v < n && __ldg(st + v) == itn) {
                const uint4 info = __ldg(vinfo + v);
                if (info.w && info.z >= lo && info.z < hi) m[q] = info.w;
                if (bmode && (m[q] || bound_all)) {
                    const uint32_t x = val[v];
                    bnd = bmode == 2 ? max(bnd, x) : min(bnd, x);
                }
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
    if (bmode) {  // one atomic per warp
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const uint32_t y = __shfl_xor_sync(kFull, bnd, o);
            bnd = bmode == 2 ? max(bnd, y) : min(bnd, y);
        }
        if (lane == 0 && bnd != (bmode == 2 ? 0u : kInf)) {
            if (bmode == 2) atomicMax(&ctl->bound[slot], bnd);
            else atomicMin(&ctl->bound[slot], bnd);
        }
    }
}

// ------------------------------------------------------------------------------------------
// dispatch
// ------------------------------------------------------------------------------------------

FqFn relax_fq_kernel_bfs(int layout, bool bsp, bool stats);
FqFn relax_fq_kernel_sssp(int layout, bool bsp, bool stats);
FqFn relax_fq_kernel_sswp(int layout, bool bsp, bool stats);
FqFn relax_fq_kernel_cc(int layout, bool bsp, bool stats);

FqFn relax_fq_kernel(int algo, int layout, bool bsp, bool stats) {
    switch (algo) {
        case TIGR_BFS: return relax_fq_kernel_bfs(layout, bsp, stats);
        case TIGR_SSSP: return relax_fq_kernel_sssp(layout, bsp, stats);
        case TIGR_CC: return relax_fq_kernel_cc(layout, bsp, stats);
        case TIGR_SSWP: return relax_fq_kernel_sswp(layout, bsp, stats);
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

tigr_status compact_launch(const tigr_vgraph* vg, Ctl* ctl, int delta, cudaStream_t s, int bmode, int bound_all,
                           const uint32_t* settled) {
    const uint32_t n = vg->g->n;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t tiles = ((uint64_t)n + kFqThreads * kCompactPer - 1) / (kFqThreads * kCompactPer);
    const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(tiles, (uint64_t)sms * 8));
    k_compact<<<grid, kFqThreads, 0, s>>>(vg->ws.stamp.as<uint32_t>(), vg->vinfo.as<uint4>(), n, vg->lo, vg->hi, ctl,
                                          const_cast<uint32_t*>(vg->ws.qv.as<uint32_t>()),
                                          const_cast<uint32_t*>(vg->ws.qo.as<uint32_t>()), delta,
                                          vg->ws.val.as<uint32_t>(), bmode, bound_all,
                                          bmode ? const_cast<uint32_t*>(settled) : nullptr);
    TIGR_CK(cudaGetLastError());
    return TIGR_OK;
}

}  // namespace tigr
