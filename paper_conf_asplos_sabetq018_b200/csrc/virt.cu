// virt.cu -- the virtual split transformation on the device.
//
//  a2 family size   m_v = ceil(d_v / K), 0 for d_v = 0        (Def. 2(iii); reading R1)
//  a3 scan          vnode_ptr = exclusive scan of m_v          (Fig. 10b edge-pointer row, L929)
//  a4 vnode emit    vn_phys[i] = v for vnode_ptr[v] <= i < vnode_ptr[v+1]
//                                                              (Fig. 10b physicalNodeId row, L931)
//  a5 layout        per-node record vinfo[v] = {chunk base, d_v, vnode_ptr[v], m_v}: with it a
//                   virtual node derives its offset j and stride m_v (Alg. 3 lines 3-4, L1163-1165)
//                   over the span-aligned segment built by csr.cu; the stride unit is a 32-byte
//                   span (8 | K), a 16-byte chunk (4 | K) or one arc.
// The paper builds the virtual node array serially on the CPU (§6.4, Table 7,
// L1471-1474); here it is three kernels plus the scan.
#include "internal.cuh"
#include "vgraph.cuh"

namespace tigr {
namespace {

// vn_phys emit: thread per node for small families, whole warp for large ones (ballot loop)
__global__ void k_emit(const uint32_t* __restrict__ vptr, uint32_t n, uint32_t* __restrict__ vn_phys) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    uint32_t beg = 0, fam = 0;
    if (v < n) { beg = vptr[v]; fam = vptr[v + 1] - beg; }
    const bool big = fam > 16;
    if (!big)
        for (uint32_t k = 0; k < fam; ++k) vn_phys[beg + k] = v;
    uint32_t mask = __ballot_sync(0xffffffffu, big);
    while (mask) {
        const int l = __ffs(mask) - 1;
        mask &= mask - 1;
        const uint32_t b = __shfl_sync(0xffffffffu, beg, l);
        const uint32_t f = __shfl_sync(0xffffffffu, fam, l);
        const uint32_t vv = __shfl_sync(0xffffffffu, v, l);
        for (uint32_t k = lane; k < f; k += 32) vn_phys[b + k] = vv;
    }
}

// also counts the nodes with out-arcs (the byte model's "active physical vertex with d > 0")
__global__ void k_vinfo(const uint32_t* __restrict__ cptr, const uint32_t* __restrict__ deg,
                        const uint32_t* __restrict__ vptr, uint32_t n, uint4* __restrict__ vinfo,
                        unsigned long long* __restrict__ n_out) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    bool out = false;
    if (v < n) {
        const uint32_t b = vptr[v];
        const uint32_t d = deg[v];
        vinfo[v] = make_uint4(2 * cptr[v], d, b, vptr[v + 1] - b);  // .x: first 16-byte chunk
        out = d != 0;
    }
    const int c = __syncthreads_count(out);
    if (threadIdx.x == 0 && c) atomicAdd(n_out, (unsigned long long)c);
}

}  // namespace

tigr_status virtualize_device(const tigr_graph* g, uint32_t K, tigr_layout layout, cudaStream_t s,
                              tigr_vgraph** out) {
    if (K == 0) return fail(TIGR_EINVAL, "virtualize: K must be >= 1 (Def. 1)");
    if (layout != TIGR_LAYOUT_CONSECUTIVE && layout != TIGR_LAYOUT_STRIDED)
        return fail(TIGR_EINVAL, "virtualize: unknown layout");
    tigr_vgraph* vg = new tigr_vgraph();
    auto bail = [&](tigr_status st) { delete vg; return st; };
    vg->g = g;
    vg->K = K;
    vg->layout = layout;
    // The assignment unit: a 32-byte span of 8 arcs when 8 | K, a 16-byte chunk of
    // 4 when 4 | K, else one arc -- the unit must divide K so that no vnode exceeds K edges
    vg->unit = (K == 0xFFFFFFFFu || K % kSpan == 0) ? kSpan : (K % kChunk == 0 ? kChunk : 1u);
    vg->vec = vg->unit > 1;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0, s);
    tigr_status st;
    if ((st = vg->vnode_ptr.alloc(sizeof(uint32_t) * ((size_t)g->n + 1), s))) return bail(st);
    uint64_t nv = 0;
    if ((st = exclusive_scan_u32(g->deg.as<uint32_t>(), g->n, SCAN_CEIL_DIV, K, vg->vnode_ptr.as<uint32_t>(),
                                 s, &nv)))
        return bail(st);
    if (nv >= 0xFFFFFFFFull) return bail(fail(TIGR_ERANGE, "virtualize: more than 2^32-2 virtual nodes"));
    vg->nv = nv;
    vg->lo = 0;
    vg->hi = (uint32_t)nv;
    if ((st = vg->vn_phys.alloc(sizeof(uint32_t) * (nv ? nv : 1), s))) return bail(st);
    if ((st = vg->vinfo.alloc(sizeof(uint4) * (g->n ? g->n : 1), s))) return bail(st);
    k_emit<<<grid_for(g->n), kBlock, 0, s>>>(vg->vnode_ptr.as<uint32_t>(), g->n, vg->vn_phys.as<uint32_t>());
    count_launch();
    TmpBuf cnt;
    if ((st = cnt.alloc(sizeof(unsigned long long), s))) return bail(st);
    cudaMemsetAsync(cnt.p, 0, sizeof(unsigned long long), s);
    k_vinfo<<<grid_for(g->n), kBlock, 0, s>>>(g->cptr.as<uint32_t>(), g->deg.as<uint32_t>(),
                                               vg->vnode_ptr.as<uint32_t>(), g->n, vg->vinfo.as<uint4>(),
                                               cnt.as<unsigned long long>());
    count_launch();
    unsigned long long n_out = 0;
    cudaMemcpyAsync(&n_out, cnt.p, sizeof(n_out), cudaMemcpyDeviceToHost, s);
    cudaEventRecord(e1, s);
    cudaError_t e = cudaEventSynchronize(e1);
    if (e != cudaSuccess) return bail(cuda_fail(e, "virtualize", __FILE__, __LINE__));
    vg->n_out = n_out;
    vg->m_local = g->m;
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    vg->ms_build = ms;
    *out = vg;
    return TIGR_OK;
}

}  // namespace tigr
