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
constexpr int kCompactPer = 8;  // nodes per thread in k_compact (8 or 16)
constexpr uint32_t kFull = 0xffffffffu;
}  // namespace

// ------------------------------------------------------------------------------------------
// queue build: nodes stamped for iteration it + delta that own virtual nodes in [lo, hi)
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kFqThreads) k_compact(const stamp_t* __restrict__ stamp,
                                                         const uint32_t* __restrict__ vptr, uint32_t n, uint32_t lo,
                                                         uint32_t hi, Ctl* ctl, uint32_t* __restrict__ qv,
                                                         uint32_t* __restrict__ qo, int delta) {
    __shared__ unsigned long long s_warp[kFqThreads / 32];
    __shared__ unsigned long long s_base;
    if (!ctl->cont) return;  // past the fixed point (batched host loop, run.cu); k_init sets cont
    const uint32_t itn = ctl->it + (uint32_t)delta;
    const uint32_t slot = itn & 1u;
    const stamp_t* st = stamp + (uint64_t)slot * n;
    const stamp_t sv = stamp_of(itn);
    uint32_t* ov = qv + (uint64_t)slot * n;
    uint32_t* oo = qo + (uint64_t)slot * n;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr uint32_t kTileNodes = kFqThreads * kCompactPer;
    // the thread's stamps: one kCompactPer-byte load when the slot is aligned (n % kCompactPer == 0)
    const bool vec = (n & (kCompactPer - 1u)) == 0;
    for (uint64_t tile0 = (uint64_t)blockIdx.x * kTileNodes; tile0 < n; tile0 += (uint64_t)gridDim.x * kTileNodes) {
        const uint64_t v0 = tile0 + (uint64_t)threadIdx.x * kCompactPer;
        uint32_t act = 0;  // bit q: node v0 + q is stamped for iteration itn
        if (vec && v0 + kCompactPer <= n) {
            uint32_t ww[kCompactPer / 4];
            if constexpr (kCompactPer == 16) {
                const uint4 w = __ldg(reinterpret_cast<const uint4*>(st + v0));
                ww[0] = w.x; ww[1] = w.y; ww[2] = w.z; ww[3] = w.w;
            } else {
                const uint2 w = __ldg(reinterpret_cast<const uint2*>(st + v0));
                ww[0] = w.x; ww[1] = w.y;
            }
#pragma unroll
            for (int q = 0; q < kCompactPer; ++q)
                if (((ww[q >> 2] >> (8 * (q & 3))) & 0xFFu) == sv) act |= 1u << q;
        } else {
#pragma unroll
            for (int q = 0; q < kCompactPer; ++q)
                if (v0 + q < n && __ldg(st + v0 + q) == sv) act |= 1u << q;
        }
        // a tile without a stamped node costs one barrier (most tiles of a sparse iteration)
        if (!__syncthreads_or(act != 0)) continue;
        uint32_t m[kCompactPer];
        unsigned long long mine = 0;  // (entries << 32) | vnodes of this thread's nodes
        // family sizes m_v = vnode_ptr[v + 1] - vnode_ptr[v] (and the first virtual node, for this
        // rank's range): the thread's kCompactPer + 1 offsets in vector loads -- in dense
        // iterations a sweep of the 4-byte offsets instead of one 16-byte vinfo gather per node
        uint32_t vp[kCompactPer + 1];
        if (act) {
            if (v0 + kCompactPer <= n) {  // v0 is a multiple of kCompactPer: aligned
#pragma unroll
                for (int h = 0; h < kCompactPer / 4; ++h) {
                    const uint4 w = __ldg(reinterpret_cast<const uint4*>(vptr + v0) + h);
                    vp[4 * h] = w.x; vp[4 * h + 1] = w.y; vp[4 * h + 2] = w.z; vp[4 * h + 3] = w.w;
                }
                vp[kCompactPer] = __ldg(vptr + v0 + kCompactPer);
            } else {
#pragma unroll
                for (int q = 0; q <= kCompactPer; ++q) vp[q] = v0 + q <= n ? __ldg(vptr + v0 + q) : 0u;
            }
        }
#pragma unroll
        for (int q = 0; q < kCompactPer; ++q) {
            m[q] = 0;
            if ((act >> q) & 1u) {
                const uint32_t f = vp[q], mv = vp[q + 1] - vp[q];
                if (mv && f >= lo && f < hi) m[q] = mv;
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
        // (s_warp / s_base are next written after the next tile's __syncthreads_or)
        unsigned long long pos = s_base + s_warp[wid] + (inc - mine);
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
// packed arcs for SSSP / SSWP: target | (w - wmin) << idbits in one 32-bit slot
// ------------------------------------------------------------------------------------------
__global__ void k_weight_range(const uint4* __restrict__ c4, const uint4* __restrict__ w4, uint64_t nchunks,
                               uint32_t* __restrict__ mm) {
    uint32_t lo = kInf, hi = 0;
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks; k += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 c = __ldg(c4 + k), w = __ldg(w4 + k);
        const uint32_t cc[4] = {c.x, c.y, c.z, c.w}, ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (cc[q] != kPad) { lo = min(lo, ww[q]); hi = max(hi, ww[q]); }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        lo = min(lo, __shfl_xor_sync(kFull, lo, o));
        hi = max(hi, __shfl_xor_sync(kFull, hi, o));
    }
    if ((threadIdx.x & 31) == 0) { atomicMin(mm, lo); atomicMax(mm + 1, hi); }
}

__global__ void k_pack_arcs(const uint4* __restrict__ c4, const uint4* __restrict__ w4, uint64_t nchunks,
                            uint32_t idbits, uint32_t wmin, uint4* __restrict__ out) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks; k += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 c = __ldg(c4 + k), w = __ldg(w4 + k);
        uint32_t cc[4] = {c.x, c.y, c.z, c.w};
        const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) cc[q] = cc[q] == kPad ? kPad : (cc[q] | ((ww[q] - wmin) << idbits));
        out[k] = make_uint4(cc[0], cc[1], cc[2], cc[3]);
    }
}

// once per virtual graph: pack when the ids and the weight range fit one 32-bit slot together
// (idbits: the smallest b with 2^b > n, so the all-ones id field is never a node and marks pads)
tigr_status pack_arcs_prepare(tigr_vgraph* vg, cudaStream_t s) {
    Workspace& ws = vg->ws;
    if (ws.cw_state) return TIGR_OK;
    const tigr_graph* g = vg->g;
    ws.cw_state = 2;  // not packable until shown otherwise
    if (!g->weighted || g->nchunks == 0) return TIGR_OK;
    uint32_t idbits = 1;
    while (idbits < 32 && ((1ull << idbits) - 1) < (uint64_t)g->n) ++idbits;
    TmpBuf mm;
    TIGR_TRY(mm.alloc(2 * sizeof(uint32_t), s));
    const uint32_t init[2] = {kInf, 0u};
    TIGR_CK(cudaMemcpyAsync(mm.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const unsigned grid = (unsigned)std::min<uint64_t>(grid_for(g->nchunks), (uint64_t)sms * 8);
    k_weight_range<<<grid, kFqThreads, 0, s>>>(g->col.as<uint4>(), g->wt.as<uint4>(), g->nchunks, mm.as<uint32_t>());
    TIGR_CKL("pack: weight range");
    uint32_t h[2] = {0, 0};
    TIGR_CK(cudaMemcpyAsync(h, mm.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    if (h[0] > h[1]) return TIGR_OK;  // no arcs
    uint32_t wbits = 0;
    while (wbits < 32 && ((uint64_t)(h[1] - h[0]) >> wbits) != 0) ++wbits;
    if (idbits > 31 || idbits + wbits > 32) return TIGR_OK;
    TIGR_TRY(ws.cw.alloc(sizeof(uint32_t) * kChunk * g->nchunks, s));
    k_pack_arcs<<<grid, kFqThreads, 0, s>>>(g->col.as<uint4>(), g->wt.as<uint4>(), g->nchunks, idbits, h[0],
                                            ws.cw.as<uint4>());
    TIGR_CKL("pack: arcs");
    ws.cw_idbits = idbits;
    ws.cw_wmin = h[0];
    ws.cw_state = 1;
    return TIGR_OK;
}

// ------------------------------------------------------------------------------------------
// dispatch
// ------------------------------------------------------------------------------------------

FqFn relax_fq_kernel_bfs(int layout, int unit, bool bsp, bool stats, bool packed);
FqFn relax_fq_kernel_sssp(int layout, int unit, bool bsp, bool stats, bool packed);
FqFn relax_fq_kernel_sswp(int layout, int unit, bool bsp, bool stats, bool packed);
FqFn relax_fq_kernel_cc(int layout, int unit, bool bsp, bool stats, bool packed);

FqFn relax_fq_kernel(int algo, int layout, int unit, bool bsp, bool stats, bool packed) {
    switch (algo) {
        case TIGR_BFS: return relax_fq_kernel_bfs(layout, unit, bsp, stats, false);
        case TIGR_SSSP: return relax_fq_kernel_sssp(layout, unit, bsp, stats, packed);
        case TIGR_CC: return relax_fq_kernel_cc(layout, unit, bsp, stats, false);
        case TIGR_SSWP: return relax_fq_kernel_sswp(layout, unit, bsp, stats, packed);
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
    // one tile per block up to 64 blocks per SM: a block walking several tiles paid one stamp-load
    // latency per tile in sequence (an empty cfg4 sweep took 15 us for 16.8 MB)
    const uint64_t cap = (uint64_t)sms * (uint64_t)dev_knob("TIGR_COMPACT_BPS", 64);
    const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(tiles, cap));
    k_compact<<<grid, kFqThreads, 0, s>>>(vg->ws.stamp.as<stamp_t>(), vg->vnode_ptr.as<uint32_t>(), n, vg->lo, vg->hi, ctl,
                                          const_cast<uint32_t*>(vg->ws.qv.as<uint32_t>()),
                                          const_cast<uint32_t*>(vg->ws.qo.as<uint32_t>()), delta);
    TIGR_CK(cudaGetLastError());
    return TIGR_OK;
}

}  // namespace tigr
