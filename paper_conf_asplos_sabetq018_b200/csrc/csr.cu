// csr.cu -- device CSR construction.
//
// CSR = node array (exclusive scan of out-degrees) + edge array grouped by source
// (Fig. 10a; "we reorder the edges during the construction of CSR",
// L1131-1132).  B200 layout: every node's segment starts on a 32-byte boundary and is
// padded to a multiple of 8 slots (pads = 0xFFFFFFFF), so the relax kernels can move
// edges (and, in a separate array, weights) as 256-bit spans or 128-bit chunks; cptr[v] is
// the first span.
// From an arc list the CSR is built by a stable radix sort on the source (sort.cu), so the
// arcs of a source keep their input order: the canonical CSR, element-identical to a stable
// counting sort.
#include <algorithm>

#include "internal.cuh"

namespace tigr {

tigr_status expand_arcs(const tigr_graph* g, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s);

tigr_status rmat_range(uint32_t n, uint64_t e0, uint64_t count, double a, double b, double c,
                       uint64_t seed, uint64_t wseed, uint32_t wmin, uint32_t wmax, uint32_t* src,
                       uint32_t* dst, uint32_t* w, cudaStream_t s);
tigr_status csr_build_sorted(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                             int symmetrize, cudaStream_t s, tigr_graph* g, uint32_t klo, uint32_t khi,
                             const HostArcs* host);

namespace {

constexpr uint32_t kReorderKeyMax = (1u << 24) - 1;  // in-degrees beyond tie (stable: by id)

__global__ void k_pad(const uint32_t* __restrict__ deg, const uint32_t* __restrict__ cptr, uint32_t n,
                      uint32_t* __restrict__ col, uint32_t* __restrict__ wt) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    const uint64_t base = (uint64_t)cptr[v] * kSpan;
    const uint32_t d = deg[v];
    const uint64_t end = (uint64_t)cptr[v + 1] * kSpan;
    for (uint64_t s = base + d; s < end; ++s) {
        col[s] = kPad;
        if (wt) wt[s] = 0;
    }
}

__global__ void k_deg_from_rowptr(const int64_t* __restrict__ rp, uint32_t n, uint64_t m,
                                  uint32_t* __restrict__ deg, uint32_t* bad) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v == 0 && (rp[0] != 0 || rp[n] != (int64_t)m)) *bad = 1;
    if (v >= n) return;
    const int64_t d = rp[v + 1] - rp[v];
    if (d < 0 || d > 0xFFFFFFFFll) { *bad = 1; deg[v] = 0; return; }
    deg[v] = (uint32_t)d;
}

__device__ __forceinline__ uint32_t owner_of(const int64_t* __restrict__ rp, uint32_t n, uint64_t e) {
    uint32_t lo = 0, hi = n;  // last v with rp[v] <= e
    while (hi - lo > 1) {
        const uint32_t mid = lo + (hi - lo) / 2;
        if ((uint64_t)rp[mid] <= e) lo = mid; else hi = mid;
    }
    return lo;
}

// canonical (row_ptr-indexed) arrays <-> padded segments
__global__ void k_csr_to_padded(const int64_t* __restrict__ rp, uint32_t n, uint64_t m,
                                const uint32_t* __restrict__ cin, const uint32_t* __restrict__ win,
                                const uint32_t* __restrict__ cptr, uint32_t* __restrict__ col,
                                uint32_t* __restrict__ wt, uint32_t* bad) {
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m;
         e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t v = owner_of(rp, n, e);
        const uint64_t slot = (uint64_t)cptr[v] * kSpan + (e - rp[v]);
        const uint32_t c = cin[e];
        if (c >= n) *bad = 1;
        col[slot] = c;
        if (wt) wt[slot] = win[e];
    }
}

__global__ void k_padded_to_csr(const int64_t* __restrict__ rp, uint32_t n, uint64_t m,
                                const uint32_t* __restrict__ cptr, const uint32_t* __restrict__ col,
                                const uint32_t* __restrict__ wt, uint32_t* __restrict__ cout,
                                uint32_t* __restrict__ wout) {
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m;
         e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t v = owner_of(rp, n, e);
        const uint64_t slot = (uint64_t)cptr[v] * kSpan + (e - rp[v]);
        if (cout) cout[e] = col[slot];
        if (wout) wout[e] = wt[slot];
    }
}

// canonical arc list (src, dst, w) of a device CSR, arc-parallel (balanced whatever the
// degrees: one hub's 371 K arcs are spread over many blocks).  Block b owns arc positions
// [b*kExpTile, (b+1)*kExpTile); one thread finds the node owning the first position (binary
// search over row_ptr), the block stages the row offsets of the nodes its tile spans in shared
// memory, and each arc finds its source there by a short binary search.  Tiles that span more
// nodes than the stage holds (long runs of zero-degree nodes) search row_ptr in global memory.
constexpr uint32_t kExpTile = 2048;
constexpr uint32_t kExpStage = 2048;

__device__ __forceinline__ uint32_t owner_of(const int64_t* __restrict__ rp, uint32_t lo, uint32_t hi, uint64_t p) {
    // last v in [lo, hi] with rp[v] <= p
    while (lo < hi) {
        const uint32_t mid = lo + (hi - lo + 1) / 2;
        if ((uint64_t)rp[mid] <= p) lo = mid; else hi = mid - 1;
    }
    return lo;
}

__global__ void __launch_bounds__(256) k_expand_arcs(const int64_t* __restrict__ rp, const uint32_t* __restrict__ cptr,
                                                     uint32_t n, uint64_t m, const uint32_t* __restrict__ col,
                                                     const uint32_t* __restrict__ wt, uint32_t* __restrict__ src,
                                                     uint32_t* __restrict__ dst, uint32_t* __restrict__ w) {
    __shared__ int64_t s_rp[kExpStage + 1];
    __shared__ uint32_t s_v[2];
    for (uint64_t t0 = (uint64_t)blockIdx.x * kExpTile; t0 < m; t0 += (uint64_t)gridDim.x * kExpTile) {
        const uint64_t t1 = min(t0 + kExpTile, m);
        if (threadIdx.x == 0) s_v[0] = owner_of(rp, 0, n - 1, t0);
        if (threadIdx.x == 1) s_v[1] = owner_of(rp, 0, n - 1, t1 - 1);
        __syncthreads();
        const uint32_t v0 = s_v[0], v1 = s_v[1];
        const bool staged = v1 - v0 < kExpStage;
        if (staged)
            for (uint32_t i = threadIdx.x; i <= v1 - v0; i += blockDim.x) s_rp[i] = rp[v0 + i];
        __syncthreads();
        for (uint64_t p = t0 + threadIdx.x; p < t1; p += blockDim.x) {
            uint32_t v;
            int64_t beg;
            if (staged) {
                uint32_t lo = 0, hi = v1 - v0;
                while (lo < hi) {
                    const uint32_t mid = lo + (hi - lo + 1) / 2;
                    if ((uint64_t)s_rp[mid] <= p) lo = mid; else hi = mid - 1;
                }
                v = v0 + lo;
                beg = s_rp[lo];
            } else {
                v = owner_of(rp, v0, v1, p);
                beg = rp[v];
            }
            const uint64_t c = (uint64_t)cptr[v] * kSpan + (p - (uint64_t)beg);
            src[p] = v;
            dst[p] = col[c];
            if (w) w[p] = wt[c];
        }
        __syncthreads();  // s_rp / s_v reused by the next tile
    }
}


// ---- UDT (physical uniform-degree-tree transformation, §3.2 Alg. 1) ----
// Node v of out-degree d > K gets t = ceil((d-K)/(K-1)) new split nodes.  Alg. 1's queue is
// the sequence S = (v's neighbours in CSR order, then the new nodes N_0..N_{t-1}); N_k pops
// S[kK, kK+K) and the root v keeps S[tK, d+t).  So every arc's new source follows from its
// S-position alone: N_{p/K} if p < tK else v -- no queue needed on the device.
__global__ void k_udt_count(const uint32_t* __restrict__ deg, uint32_t n, uint32_t K, uint32_t* __restrict__ t) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    const uint32_t d = deg[v];
    t[v] = d > K ? (d - K + (K - 2)) / (K - 1) : 0u;
}

__global__ void k_udt_arcs(const int64_t* __restrict__ rp, const uint32_t* __restrict__ cptr, uint32_t n,
                           uint64_t m, const uint32_t* __restrict__ col, const uint32_t* __restrict__ wt,
                           const uint32_t* __restrict__ tptr, uint32_t K, uint32_t dumb, uint32_t unit,
                           uint32_t* __restrict__ src, uint32_t* __restrict__ dst, uint32_t* __restrict__ w) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    uint64_t beg = 0, cb = 0;
    uint32_t d = 0, tb = 0, t = 0;
    if (v < n) {
        beg = (uint64_t)rp[v]; d = (uint32_t)(rp[v + 1] - rp[v]); cb = (uint64_t)cptr[v] * kSpan;
        tb = tptr[v]; t = tptr[v + 1] - tb;
    }
    auto parent = [&](uint32_t vv, uint64_t p, uint32_t tt, uint32_t tbb) -> uint32_t {
        return p < (uint64_t)tt * K ? n + tbb + (uint32_t)(p / K) : vv;
    };
    const uint32_t work = d + t;
    const bool big = work > 32;
    if (!big) {
        for (uint32_t p = 0; p < d; ++p) {
            src[beg + p] = parent(v, p, t, tb);
            dst[beg + p] = col[cb + p];
            w[beg + p] = wt ? wt[cb + p] : unit;
        }
        for (uint32_t k = 0; k < t; ++k) {
            src[m + tb + k] = parent(v, (uint64_t)d + k, t, tb);
            dst[m + tb + k] = n + tb + k;
            w[m + tb + k] = dumb;
        }
    }
    uint32_t mask = __ballot_sync(0xffffffffu, big);
    while (mask) {
        const int l = __ffs(mask) - 1;
        mask &= mask - 1;
        const uint64_t b = __shfl_sync(0xffffffffu, beg, l), c = __shfl_sync(0xffffffffu, cb, l);
        const uint32_t dd = __shfl_sync(0xffffffffu, d, l), vv = __shfl_sync(0xffffffffu, v, l);
        const uint32_t tt = __shfl_sync(0xffffffffu, t, l), tbb = __shfl_sync(0xffffffffu, tb, l);
        for (uint32_t p = lane; p < dd; p += 32) {
            src[b + p] = parent(vv, p, tt, tbb);
            dst[b + p] = col[c + p];
            w[b + p] = wt ? wt[c + p] : unit;
        }
        for (uint32_t k = lane; k < tt; k += 32) {
            src[m + tbb + k] = parent(vv, (uint64_t)dd + k, tt, tbb);
            dst[m + tbb + k] = n + tbb + k;
            w[m + tbb + k] = dumb;
        }
    }
}

unsigned capped_grid(uint64_t items) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t want = (items + kBlock - 1) / kBlock;
    const uint64_t cap = (uint64_t)sms * 16;
    return (unsigned)(want == 0 ? 1 : (want < cap ? want : cap));
}

// degrees known -> row_ptr, cptr, edge buffers
tigr_status layout_from_degrees(tigr_graph* g, cudaStream_t s) {
    TIGR_TRY(g->row_ptr.alloc(sizeof(int64_t) * ((size_t)g->n + 1), s));
    TIGR_TRY(exclusive_scan_u64(g->deg.as<uint32_t>(), g->n, SCAN_U32, 1,
                                reinterpret_cast<uint64_t*>(g->row_ptr.p), s));
    TIGR_TRY(g->cptr.alloc(sizeof(uint32_t) * ((size_t)g->n + 1), s));
    uint64_t nch = 0;
    TIGR_TRY(exclusive_scan_u32(g->deg.as<uint32_t>(), g->n, SCAN_CEIL_DIV, kSpan, g->cptr.as<uint32_t>(),
                                s, &nch));
    if (nch >= (1ull << 31)) return fail(TIGR_ERANGE, "graph: padded edge spans exceed 2^31");
    nch *= 2;  // 16-byte chunks
    g->nchunks = nch;
    TIGR_TRY(g->col.alloc(sizeof(uint32_t) * kChunk * (nch ? nch : 1), s));
    if (g->weighted) TIGR_TRY(g->wt.alloc(sizeof(uint32_t) * kChunk * (nch ? nch : 1), s));
    return TIGR_OK;
}


// exact in-degrees: one RED.ADD per arc (pads skipped)
__global__ void k_indeg_count(const uint4* __restrict__ c4, uint64_t nchunks, uint32_t* __restrict__ cnt) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks;
         k += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 c = c4[k];
        if (c.x != kPad) atomicAdd(cnt + c.x, 1u);
        if (c.y != kPad) atomicAdd(cnt + c.y, 1u);
        if (c.z != kPad) atomicAdd(cnt + c.z, 1u);
        if (c.w != kPad) atomicAdd(cnt + c.w, 1u);
    }
}

// sort key for decreasing in-degree (ties: increasing id, the sort is stable)
__global__ void k_reorder_key(const uint32_t* __restrict__ cnt, uint32_t n, uint32_t* __restrict__ key,
                              uint32_t* __restrict__ ids) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    const uint32_t c = cnt[v] < kReorderKeyMax ? cnt[v] : kReorderKeyMax;
    key[v] = kReorderKeyMax - c;
    ids[v] = v;
}

__global__ void k_inverse(const uint32_t* __restrict__ order, uint32_t n, uint32_t* __restrict__ cid) {
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c < n) cid[order[c]] = c;
}

__global__ void k_relabel(uint32_t* __restrict__ src, uint32_t* __restrict__ dst, uint64_t m,
                          const uint32_t* __restrict__ cid) {
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
        src[e] = __ldg(cid + src[e]);
        dst[e] = __ldg(cid + dst[e]);
    }
}

}  // namespace

tigr_status expand_arcs(const tigr_graph* g, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s) {
    if (g->m == 0 || g->n == 0) return TIGR_OK;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t tiles = (g->m + kExpTile - 1) / kExpTile;
    const unsigned grid = (unsigned)std::min<uint64_t>(tiles, (uint64_t)sms * 8);
    k_expand_arcs<<<grid, 256, 0, s>>>(g->row_ptr.as<int64_t>(), g->cptr.as<uint32_t>(), g->n, g->m,
                                       g->col.as<uint32_t>(), g->weighted ? g->wt.as<uint32_t>() : nullptr, src, dst,
                                       w);
    TIGR_CKL("expand arcs");
    return TIGR_OK;
}

// src_lo/src_hi: keep only the arcs whose source lies in [src_lo, src_hi) (multi-GPU partitioned
// builds); the in-degree sketch and the id validation still cover every arc
// host (nullable): src / dst / w are device buffers still to be filled from these host arrays
// (the build copies them in chunks, overlapped with its arc-list scan)
tigr_status graph_from_coo_part_device(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                       const uint32_t* w, int symmetrize, uint32_t src_lo, uint32_t src_hi,
                                       cudaStream_t s, tigr_graph** out, const HostArcs* host) {
    const uint64_t arcs = symmetrize ? 2 * m : m;
    if (arcs >= (1ull << 32) * 3) return fail(TIGR_ERANGE, "graph: too many arcs");
    tigr_graph* g = new tigr_graph();
    g->n = n;
    g->m = arcs;
    g->weighted = w != nullptr;
    g->symmetric = symmetrize != 0;
    tigr_status st = csr_build_sorted(n, m, src, dst, w, symmetrize, s, g, src_lo, src_hi, host);
    g->part_lo = src_lo;
    g->part_hi = src_hi < n ? src_hi : n;
    // pad slots are written by the placement itself (sort.cu k_place)
    if (st != TIGR_OK) { delete g; return st; }
    *out = g;
    return TIGR_OK;
}

tigr_status graph_from_coo_device(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                  const uint32_t* w, int symmetrize, cudaStream_t s, tigr_graph** out) {
    return graph_from_coo_part_device(n, m, src, dst, w, symmetrize, 0, 0xFFFFFFFFu, s, out, nullptr);
}

tigr_status graph_from_csr_device(uint32_t n, uint64_t m, const int64_t* rp, const uint32_t* col,
                                  const uint32_t* w, int symmetric_hint, cudaStream_t s, tigr_graph** out) {
    tigr_graph* g = new tigr_graph();
    g->n = n;
    g->m = m;
    g->weighted = w != nullptr;
    g->symmetric = symmetric_hint != 0;
    auto bail = [&](tigr_status st) { delete g; return st; };
    tigr_status st;
    TmpBuf bad;
    if ((st = bad.alloc(sizeof(uint32_t), s))) return bail(st);
    cudaMemsetAsync(bad.p, 0, sizeof(uint32_t), s);
    if ((st = g->deg.alloc(sizeof(uint32_t) * n, s))) return bail(st);
    k_deg_from_rowptr<<<grid_for(n), kBlock, 0, s>>>(rp, n, m, g->deg.as<uint32_t>(), bad.as<uint32_t>());
    count_launch();
    uint32_t hbad = 0;
    cudaMemcpyAsync(&hbad, bad.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
    cudaError_t e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return bail(cuda_fail(e, "from_csr validate", __FILE__, __LINE__));
    if (hbad) return bail(fail(TIGR_EINVAL, "graph_from_csr: row_ptr not monotone / row_ptr[0] != 0 / row_ptr[n] != m"));
    if ((st = layout_from_degrees(g, s))) return bail(st);
    if (m) {
        k_csr_to_padded<<<capped_grid(m), kBlock, 0, s>>>(rp, n, m, col, w, g->cptr.as<uint32_t>(),
                                                          g->col.as<uint32_t>(), g->wt.as<uint32_t>(),
                                                          bad.as<uint32_t>());
        count_launch();
    }
    k_pad<<<grid_for(n), kBlock, 0, s>>>(g->deg.as<uint32_t>(), g->cptr.as<uint32_t>(), n,
                                          g->col.as<uint32_t>(), g->wt.as<uint32_t>());
    count_launch();
    cudaMemcpyAsync(&hbad, bad.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return bail(cuda_fail(e, "from_csr kernels", __FILE__, __LINE__));
    if (hbad) return bail(fail(TIGR_EINVAL, "graph_from_csr: col id >= n"));
    *out = g;
    return TIGR_OK;
}

tigr_status graph_export_csr_device(const tigr_graph* g, int64_t* rp, uint32_t* col, uint32_t* w,
                                    cudaStream_t s) {
    if (rp)
        TIGR_CK(cudaMemcpyAsync(rp, g->row_ptr.p, sizeof(int64_t) * ((size_t)g->n + 1),
                                cudaMemcpyDeviceToDevice, s));
    if ((col || (w && g->weighted)) && g->m) {
        k_padded_to_csr<<<capped_grid(g->m), kBlock, 0, s>>>(
            g->row_ptr.as<int64_t>(), g->n, g->m, g->cptr.as<uint32_t>(), g->col.as<uint32_t>(),
            g->wt.as<uint32_t>(), col, g->weighted ? w : nullptr);
        TIGR_CKL("export csr");
    }
    return TIGR_OK;
}

// in-CSR of g: arcs reversed, grouped by target, stable in g's (canonical) arc order; carries
// g's out-degrees (src_deg) for pull-based PageRank
tigr_status graph_transpose_device(const tigr_graph* g, cudaStream_t s, tigr_graph** out) {
    const uint64_t m = g->m;
    TmpBuf src, dst, w;
    TIGR_TRY(src.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    TIGR_TRY(dst.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    if (g->weighted) TIGR_TRY(w.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    TIGR_TRY(expand_arcs(g, src.as<uint32_t>(), dst.as<uint32_t>(), g->weighted ? w.as<uint32_t>() : nullptr, s));
    tigr_graph* t = nullptr;
    TIGR_TRY(graph_from_coo_device(g->n, m, dst.as<uint32_t>(), src.as<uint32_t>(),
                                   g->weighted ? w.as<uint32_t>() : nullptr, 0, s, &t));
    t->symmetric = g->symmetric;
    t->transposed = !g->transposed;
    t->part_lo = g->part_lo;
    t->part_hi = g->part_hi;
    tigr_status st = t->src_deg.alloc(sizeof(uint32_t) * (g->n ? g->n : 1), s);
    if (st == TIGR_OK && g->n) {
        cudaError_t e = cudaMemcpyAsync(t->src_deg.p, g->deg.p, sizeof(uint32_t) * g->n, cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) st = cuda_fail(e, "transpose src_deg", __FILE__, __LINE__);
    }
    if (st != TIGR_OK) { delete t; return st; }
    *out = t;
    return TIGR_OK;
}

// Node relabelling by decreasing in-degree (tigr_graph_reorder).  The arcs are expanded,
// both endpoints mapped through cid, and rebuilt by the stable CSR builder, so node c's
// segment is node order[c]'s segment in its canonical order with relabelled targets.
tigr_status sort_pairs_u32(const uint32_t* keys, const uint32_t* vals, uint64_t count, uint32_t key_limit,
                           cudaStream_t s, TmpBuf& keys_out, TmpBuf& vals_out);

tigr_status graph_reorder_device(const tigr_graph* g, cudaStream_t s, tigr_graph** out) {
    if (g->transposed || g->reordered || g->part_lo != 0 || g->part_hi < g->n)
        return fail(TIGR_EUNSUPPORTED, "reorder: needs a full, forward, not yet reordered graph");
    const uint32_t n = g->n;
    const uint64_t m = g->m;
    TmpBuf cnt, key, ids;
    TIGR_TRY(cnt.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(key.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(ids.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_CK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * (n ? n : 1), s));
    if (g->nchunks) {
        k_indeg_count<<<capped_grid(g->nchunks), kBlock, 0, s>>>(g->col.as<uint4>(), g->nchunks, cnt.as<uint32_t>());
        TIGR_CKL("reorder indeg");
    }
    k_reorder_key<<<grid_for(n), kBlock, 0, s>>>(cnt.as<uint32_t>(), n, key.as<uint32_t>(), ids.as<uint32_t>());
    TIGR_CKL("reorder key");
    TmpBuf skeys, order;
    TIGR_TRY(sort_pairs_u32(key.as<uint32_t>(), ids.as<uint32_t>(), n, kReorderKeyMax + 1, s, skeys, order));
    TmpBuf cid;
    TIGR_TRY(cid.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    k_inverse<<<grid_for(n), kBlock, 0, s>>>(order.as<uint32_t>(), n, cid.as<uint32_t>());
    TIGR_CKL("reorder inverse");
    TmpBuf src, dst, w;
    TIGR_TRY(src.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    TIGR_TRY(dst.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    if (g->weighted) TIGR_TRY(w.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    TIGR_TRY(expand_arcs(g, src.as<uint32_t>(), dst.as<uint32_t>(), g->weighted ? w.as<uint32_t>() : nullptr, s));
    if (m) {
        k_relabel<<<capped_grid(m), kBlock, 0, s>>>(src.as<uint32_t>(), dst.as<uint32_t>(), m, cid.as<uint32_t>());
        TIGR_CKL("reorder relabel");
    }
    tigr_graph* t = nullptr;
    TIGR_TRY(graph_from_coo_device(n, m, src.as<uint32_t>(), dst.as<uint32_t>(),
                                   g->weighted ? w.as<uint32_t>() : nullptr, 0, s, &t));
    t->symmetric = g->symmetric;
    t->reordered = true;
    tigr_status st = t->perm_cid.alloc(sizeof(uint32_t) * (n ? n : 1), s);
    if (st == TIGR_OK) st = t->perm_order.alloc(sizeof(uint32_t) * (n ? n : 1), s);
    if (st == TIGR_OK && n) {
        cudaError_t e = cudaMemcpyAsync(t->perm_cid.p, cid.p, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(t->perm_order.p, order.p, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) st = cuda_fail(e, "reorder perm", __FILE__, __LINE__);
    }
    if (st != TIGR_OK) { delete t; return st; }
    *out = t;
    return TIGR_OK;
}

tigr_status graph_udt_device(const tigr_graph* g, uint32_t K, uint32_t dumb, uint32_t unit, cudaStream_t s,
                             tigr_graph** out) {
    if (K < 2) return fail(TIGR_EINVAL, "udt: K must be >= 2 (Alg. 1 does not terminate for K = 1)");
    const uint32_t n = g->n;
    TmpBuf t, tptr;
    TIGR_TRY(t.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(tptr.alloc(sizeof(uint32_t) * ((size_t)n + 1), s));
    k_udt_count<<<grid_for(n), kBlock, 0, s>>>(g->deg.as<uint32_t>(), n, K, t.as<uint32_t>());
    TIGR_CKL("udt count");
    uint64_t T = 0;
    TIGR_TRY(exclusive_scan_u32(t.as<uint32_t>(), n, SCAN_U32, 1, tptr.as<uint32_t>(), s, &T));
    if ((uint64_t)n + T > 0xFFFFFFFEull) return fail(TIGR_ERANGE, "udt: too many split nodes");
    const uint64_t M = g->m + T;
    TmpBuf src, dst, w;
    TIGR_TRY(src.alloc(sizeof(uint32_t) * (M ? M : 1), s));
    TIGR_TRY(dst.alloc(sizeof(uint32_t) * (M ? M : 1), s));
    TIGR_TRY(w.alloc(sizeof(uint32_t) * (M ? M : 1), s));
    k_udt_arcs<<<grid_for(n), kBlock, 0, s>>>(g->row_ptr.as<int64_t>(), g->cptr.as<uint32_t>(), n, g->m,
                                              g->col.as<uint32_t>(), g->weighted ? g->wt.as<uint32_t>() : nullptr,
                                              tptr.as<uint32_t>(), K, dumb, unit, src.as<uint32_t>(),
                                              dst.as<uint32_t>(), w.as<uint32_t>());
    TIGR_CKL("udt arcs");
    return graph_from_coo_device((uint32_t)(n + T), M, src.as<uint32_t>(), dst.as<uint32_t>(), w.as<uint32_t>(), 0, s,
                                 out);
}

tigr_status graph_rmat_device(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed,
                              uint64_t wseed, uint32_t wmin, uint32_t wmax, int weighted, int symmetrize,
                              cudaStream_t s, tigr_graph** out) {
    TmpBuf src, dst, w;
    const size_t bytes = sizeof(uint32_t) * (m ? m : 1);
    TIGR_TRY(src.alloc(bytes, s));
    TIGR_TRY(dst.alloc(bytes, s));
    if (weighted) TIGR_TRY(w.alloc(bytes, s));
    TIGR_TRY(rmat_range(n, 0, m, a, b, c, seed, wseed, wmin, wmax, src.as<uint32_t>(), dst.as<uint32_t>(),
                        weighted ? w.as<uint32_t>() : nullptr, s));
    return graph_from_coo_device(n, m, src.as<uint32_t>(), dst.as<uint32_t>(),
                                 weighted ? w.as<uint32_t>() : nullptr, symmetrize, s, out);
}

}  // namespace tigr
