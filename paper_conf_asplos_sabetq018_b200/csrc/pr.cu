// pr.cu -- PageRank push with an in-degree-ordered accumulator (PR).
//
// The push relax adds contrib[u] = x[u]/d_u into acc[v] for every arc u->v with a float64
// reduction (fn. 7 L1078; Thm. 3).  At scale 24 the accumulator is 134 MB, which
// does not fit the 126 MB L2, and power-law in-degrees make the reductions collide on a few
// sectors.  Measured on B200 (tools/micro/red_bench.cu): spread REDs run at ~190 G/s on an
// L2-resident array, ~61 G/s once the array exceeds L2, ~70 G/s under R-MAT skew.
//
// So, once per graph, destinations get a dense "accumulator id" cid in order of decreasing
// (sampled) in-degree, vertices without in-arcs last:
//   * every arc's reduction lands in the first n_in entries (59 MB at scale 24: L2-resident);
//   * the S hottest destinations (cid < S) are accumulated in shared memory by each persistent
//     block and flushed once per block -- no hashing, the test is cid < S;
// and the PR-only arc array col_pr = cid[col] is built next to the CSR.  The sources, the
// virtual split and its strided layout are untouched: thread i still owns virtual node i and
// its <= K arcs, and reads contrib[v] of its physical node v.  Apply reads acc[cid[v]].
// Same sums as the plain push, associated differently (PR parity is 1e-6).
#include <algorithm>

#include "devutil.cuh"
#include "internal.cuh"
#include "relax.cuh"
#include "vgraph.cuh"

namespace tigr {

tigr_status sort_pairs_u32(const uint32_t* keys, const uint32_t* vals, uint64_t count, uint32_t key_limit,
                           cudaStream_t s, TmpBuf& keys_out, TmpBuf& vals_out);
__global__ void k_hot_sample(const uint4* __restrict__ c4, uint64_t nchunks, uint32_t* __restrict__ cnt);

namespace {


__global__ void k_indeg_flag(const uint4* __restrict__ c4, uint64_t nchunks, uint32_t* __restrict__ flag) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks;
         k += (uint64_t)gridDim.x * blockDim.x) {
        // test before setting: hot targets would otherwise serialise millions of stores on one
        // L2 sector; a (possibly stale) read of 1 skips the store, a stale 0 only repeats it
        const uint4 c = ldg_chunk(c4 + k);
        const uint32_t t4[4] = {c.x, c.y, c.z, c.w};
        uint32_t f[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) f[q] = t4[q] != kPad ? flag[t4[q] >> 5] & (1u << (t4[q] & 31)) : 1u;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (!f[q]) atomicOr(flag + (t4[q] >> 5), 1u << (t4[q] & 31));
    }
}

// sort key: vertices with in-arcs first, by decreasing floor(log2(sampled count)); ties by id
__global__ void k_pr_key(const uint32_t* __restrict__ flag, const uint32_t* __restrict__ cnt, uint32_t n,
                         uint32_t* __restrict__ key, uint32_t* __restrict__ ids, uint32_t* __restrict__ n_in) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    bool in = false;
    if (v < n) {
        in = (flag[v >> 5] >> (v & 31)) & 1u;
        const uint32_t c = cnt[v];
        const uint32_t b = c ? 32u - __clz(c) : 0u;  // 0..32
        key[v] = in ? 32u - b : 33u;                 // 0..33
        ids[v] = v;
    }
    // one atomic per block (a per-warp atomic serialised ~0.5 M adds on one address: 0.36 ms)
    const int c = __syncthreads_count(in);
    if (threadIdx.x == 0 && c) atomicAdd(n_in, (uint32_t)c);
}

__global__ void k_cid_scatter(const uint32_t* __restrict__ order, uint32_t n, uint32_t* __restrict__ cid) {
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c < n) cid[order[c]] = c;
}

__global__ void k_build_col_pr(const uint4* __restrict__ c4, uint64_t nchunks, const uint32_t* __restrict__ cid,
                               uint4* __restrict__ out) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks;
         k += (uint64_t)gridDim.x * blockDim.x) {
        uint4 c = ldg_chunk(c4 + k);
        c.x = c.x == kPad ? kPad : __ldg(cid + c.x);
        c.y = c.y == kPad ? kPad : __ldg(cid + c.y);
        c.z = c.z == kPad ? kPad : __ldg(cid + c.z);
        c.w = c.w == kPad ? kPad : __ldg(cid + c.w);
        out[k] = c;
    }
}

// Fused apply (PrFuse): the relax of iteration t+1 computes each source's contribution from
// the previous iteration's accumulator itself -- x = (1-d)/n + d*acc_t[cid[v]], contrib =
// x/deg_v, the apply's exact arithmetic (no FMA) -- so the separate apply pass disappears;
// x is materialised once, after the last iteration.  mode 0: read contrib[v] (unfused);
// 1: first iteration, x = x0; 2: from acc_prev.
template <int LAYOUT, int U, int B, int T, int SLOTS, int MINB>
__global__ void __launch_bounds__(T, MINB) k_relax_pr_cid(RelaxArgs a, const uint32_t* __restrict__ col_pr,
                                                                   uint32_t tiles, PrFuse fz) {
    extern __shared__ __align__(16) double s_acc[];  // SLOTS entries (dynamic: 64 KB)
    const int t = threadIdx.x;
    for (int i = t; i < SLOTS; i += T) s_acc[i] = 0.0;
    __syncthreads();
    const uint64_t pol = policy_evict_last();
    const uint4* c4 = reinterpret_cast<const uint4*>(col_pr);
    // probe: 0 in every shipped run; development builds (TIGR_PR_EXP) use 1 / 2 / 3 to time the
    // kernel without its hot-slot adds / without its global reductions / with plain stores (wrong
    // sums, measurement only).  The run-time test stays in shipped builds on purpose: with it ptxas
    // lays the push out so that the 1024-thread kernel runs 1.139 ms per cfg4 launch, against 1.174
    // for the best branch-free push (768 threads) and 1.182 for the branch-free 1024-thread push
    // (tools/dev/pr_relax_ab.py, three alternating runs on one box).
    const int probe = fz.probe;
    auto push = [&](uint32_t c, double x) {
        if (c < (uint32_t)SLOTS) { if (probe != 1) atomicAdd(&s_acc[c], x); }
        else if (probe == 3) a.acc[c] = x;
        else if (probe != 2) red_add_f64(a.acc + c, x, pol);
    };
    for (uint32_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
        const uint64_t base = (uint64_t)a.lo + (uint64_t)tile * (B * T) + t;
        uint32_t v[B];
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint64_t i = base + (uint64_t)r * T;
            v[r] = i < a.hi ? __ldg(a.vn_phys + i) : kPad;
        }
        uint4 info[B];
        double x[B];
        uint32_t cv[B];
#pragma unroll
        for (int r = 0; r < B; ++r) {
            info[r] = make_uint4(0, 0, 0, 1);
            x[r] = 0.0;
            cv[r] = 0xFFFFFFFFu;
            if (v[r] != kPad) {
                info[r] = __ldg(a.vinfo + v[r]);
                if (fz.mode == 0) x[r] = __ldg(a.contrib + v[r]);
                else if (fz.mode == 2) cv[r] = __ldg(fz.cid + v[r]);
            }
        }
        if (fz.mode != 0) {
#pragma unroll
            for (int r = 0; r < B; ++r) {
                if (v[r] == kPad) continue;
                double xv = fz.x0;
                if (fz.mode == 2) {
                    const double s = cv[r] < fz.n_in ? __ldg(fz.prev + cv[r]) : 0.0;
                    xv = __dadd_rn(fz.base, __dmul_rn(fz.damping, s));  // = k_pr_apply_cid's x
                }
                x[r] = __ddiv_rn(xv, (double)info[r].y);                 // = its contrib (deg > 0 here)
            }
        }
        uint4 c0[B], c1[B];
        uint32_t kn[B], kend[B], step[B];
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint64_t i = base + (uint64_t)r * T;
            uint32_t k;
            if (v[r] == kPad) { k = 0; step[r] = 1; kend[r] = 0; }
            else unit_range<U, LAYOUT>(info[r].y, (uint32_t)(i - info[r].z), info[r].w, a.K, k, step[r], kend[r]);
            kn[r] = load8<U>(c4, info[r].x, k, step[r], kend[r], c0[r], c1[r], make_uint4(kPad, kPad, kPad, kPad));
        }
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t nb[8] = {c0[r].x, c0[r].y, c0[r].z, c0[r].w, c1[r].x, c1[r].y, c1[r].z, c1[r].w};
#pragma unroll
            for (int q = 0; q < 8; ++q)
                if (nb[q] != kPad) push(nb[q], x[r]);
        }
#pragma unroll
        for (int r = 0; r < B; ++r) {  // units beyond the first 8 slots (K > 8 or no split)
            for (uint32_t k = kn[r]; k < kend[r];) {
                uint4 c, d;
                k = load8<U>(c4, info[r].x, k, step[r], kend[r], c, d, make_uint4(kPad, kPad, kPad, kPad));
                const uint32_t nb[8] = {c.x, c.y, c.z, c.w, d.x, d.y, d.z, d.w};
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    if (nb[q] != kPad) push(nb[q], x[r]);
            }
        }
    }
    __syncthreads();
    for (int i = t; i < SLOTS; i += T)
        if (s_acc[i] != 0.0) red_add_f64(a.acc + i, s_acc[i], pol);
}

// x = (1-d)/n + d*(acc[cid[v]] + dsum/n); contrib = x/deg; next dangling mass -> dsum_next
__global__ void k_pr_apply_cid(uint32_t n, const uint32_t* __restrict__ deg, const uint32_t* __restrict__ cid,
                               uint32_t n_in, double base, double damping, int dangling, double* __restrict__ x,
                               double* __restrict__ contrib, const double* __restrict__ acc,
                               const double* dsum_cur, double* dsum_next) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    double dang = 0.0;
    if (v < n) {
        const uint32_t c = cid[v];
        double s = c < n_in ? acc[c] : 0.0;
        if (dangling) s = __dadd_rn(s, __ddiv_rn(*dsum_cur, (double)n));
        const double r = __dadd_rn(base, __dmul_rn(damping, s));  // no FMA: matches the oracle
        const uint32_t d = deg[v];
        x[v] = r;
        contrib[v] = d ? __ddiv_rn(r, (double)d) : 0.0;
        if (!d) dang = r;
    }
    if (dangling) {
        __shared__ double part[kBlock / 32];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) dang += __shfl_xor_sync(0xffffffffu, dang, o);
        if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = dang;
        __syncthreads();
        if (threadIdx.x == 0) {
            double tt = 0.0;
            for (int w = 0; w < kBlock / 32; ++w) tt += part[w];
            if (tt != 0.0) atomicAdd(dsum_next, tt);
        }
    }
}

unsigned grid_cap(uint64_t items, int per_sm) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t want = (items + kBlock - 1) / kBlock;
    const uint64_t cap = (uint64_t)sms * per_sm;
    return (unsigned)(want == 0 ? 1 : (want < cap ? want : cap));
}

}  // namespace

// once per vgraph: cid order, n_in, col_pr (workspace), all on the device
tigr_status pr_cid_prepare(tigr_vgraph* vg, cudaStream_t s) {
    Workspace& ws = vg->ws;
    if (ws.cid_ready) return TIGR_OK;
    const tigr_graph* g = vg->g;
    const uint32_t n = g->n;
    TIGR_TRY(ws.cid.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(ws.col_pr.alloc(sizeof(uint32_t) * kChunk * (g->nchunks ? g->nchunks : 1), s));
    TmpBuf flag_t, cnt_t, key, ids, nin;
    TIGR_TRY(key.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(ids.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(nin.alloc(sizeof(uint32_t), s));
    TIGR_CK(cudaMemsetAsync(nin.p, 0, sizeof(uint32_t), s));
    const uint4* c4 = g->col.as<uint4>();
    const uint32_t* flag = g->in_flag.as<uint32_t>();
    const uint32_t* cnt = g->in_sample.as<uint32_t>();
    if (!g->has_in_sketch) {  // graph built from a CSR: sketch the in-degrees from the arc array
        const size_t fw = ((size_t)n + 31) / 32 + 1;  // bitmap words
        TIGR_TRY(flag_t.alloc(sizeof(uint32_t) * fw, s));
        TIGR_TRY(cnt_t.alloc(sizeof(uint32_t) * (n ? n : 1), s));
        TIGR_CK(cudaMemsetAsync(flag_t.p, 0, sizeof(uint32_t) * fw, s));
        TIGR_CK(cudaMemsetAsync(cnt_t.p, 0, sizeof(uint32_t) * n, s));
        if (g->nchunks) {
            k_indeg_flag<<<grid_cap(g->nchunks, 16), kBlock, 0, s>>>(c4, g->nchunks, flag_t.as<uint32_t>());
            TIGR_CKL("pr indeg flag");
            k_hot_sample<<<grid_cap(g->nchunks / 16 + 1, 16), kBlock, 0, s>>>(c4, g->nchunks, cnt_t.as<uint32_t>());
            TIGR_CKL("pr sample");
        }
        flag = flag_t.as<uint32_t>();
        cnt = cnt_t.as<uint32_t>();
    }
    trace(s, "pr cid: sketch");
    k_pr_key<<<grid_for(n), kBlock, 0, s>>>(flag, cnt, n, key.as<uint32_t>(),
                                             ids.as<uint32_t>(), nin.as<uint32_t>());
    TIGR_CKL("pr key");
    TmpBuf skeys, order;
    TIGR_TRY(sort_pairs_u32(key.as<uint32_t>(), ids.as<uint32_t>(), n, 34, s, skeys, order));
    k_cid_scatter<<<grid_for(n), kBlock, 0, s>>>(order.as<uint32_t>(), n, ws.cid.as<uint32_t>());
    TIGR_CKL("pr cid");
    trace(s, "pr cid: key+sort+scatter");
    if (g->nchunks) {
        k_build_col_pr<<<grid_cap(g->nchunks, 16), kBlock, 0, s>>>(c4, g->nchunks, ws.cid.as<uint32_t>(),
                                                                    ws.col_pr.as<uint4>());
        TIGR_CKL("pr col_pr");
    }
    trace(s, "pr cid: col_pr");
    uint32_t h = 0;
    TIGR_CK(cudaMemcpyAsync(&h, nin.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    ws.n_in = h;
    ws.cid_ready = true;
    return TIGR_OK;
}

// pull PageRank (NEXT-1) source order: out-degree buckets, largest first; no out-arcs last
__global__ void k_pull_key(const uint32_t* __restrict__ deg, uint32_t n, uint32_t* __restrict__ key,
                           uint32_t* __restrict__ ids) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v < n) {
        const uint32_t d = deg[v];
        key[v] = d ? 32u - (32u - __clz(d)) : 33u;  // 0..33
        ids[v] = v;
    }
}

// Pull PageRank gathers contrib[u] for every in-arc u -> v.  In vertex order that is a random
// 8-byte read from a 134 MB array at scale 24 (larger than L2).  Once per graph the sources get
// an "out id" in order of decreasing out-degree (nodes without out-arcs last, never read): the
// gathered entries then fill the first n_out slots (59 MB, L2-resident) with the most-read
// ones first.  The in-arcs are rewritten to out ids (col_pr) and contrib is kept in out-id
// order by init/apply.  Same terms; only the atomic combine of split families varies in order,
// as before (cfg4: 1.131 -> 1.057 ms per relax; the random gathers stay L2-sector bound).
tigr_status pr_pull_prepare(tigr_vgraph* vg, cudaStream_t s) {
    Workspace& ws = vg->ws;
    if (ws.cid_ready) return TIGR_OK;
    const tigr_graph* g = vg->g;
    const uint32_t n = g->n;
    TIGR_TRY(ws.cid.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(ws.col_pr.alloc(sizeof(uint32_t) * kChunk * (g->nchunks ? g->nchunks : 1), s));
    TmpBuf key, ids, skeys, order;
    TIGR_TRY(key.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_TRY(ids.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    k_pull_key<<<grid_for(n), kBlock, 0, s>>>(g->src_deg.as<uint32_t>(), n, key.as<uint32_t>(), ids.as<uint32_t>());
    TIGR_CKL("pull key");
    TIGR_TRY(sort_pairs_u32(key.as<uint32_t>(), ids.as<uint32_t>(), n, 34, s, skeys, order));
    k_cid_scatter<<<grid_for(n), kBlock, 0, s>>>(order.as<uint32_t>(), n, ws.cid.as<uint32_t>());
    TIGR_CKL("pull oid");
    if (g->nchunks) {
        k_build_col_pr<<<grid_cap(g->nchunks, 16), kBlock, 0, s>>>(g->col.as<uint4>(), g->nchunks,
                                                                    ws.cid.as<uint32_t>(), ws.col_pr.as<uint4>());
        TIGR_CKL("pull col");
    }
    ws.cid_ready = true;
    return TIGR_OK;
}

template <int B, int T, int SLOTS, int MINB>
static void fill_plan(PrCidPlan& p, int layout, int unit) {
    static_assert(B >= 1, "");
    if (unit == 8)
        p.fn = layout == TIGR_LAYOUT_STRIDED ? &k_relax_pr_cid<TIGR_LAYOUT_STRIDED, 8, B, T, SLOTS, MINB>
                                             : &k_relax_pr_cid<TIGR_LAYOUT_CONSECUTIVE, 8, B, T, SLOTS, MINB>;
    else
        p.fn = layout == TIGR_LAYOUT_STRIDED ? &k_relax_pr_cid<TIGR_LAYOUT_STRIDED, 4, B, T, SLOTS, MINB>
                                             : &k_relax_pr_cid<TIGR_LAYOUT_CONSECUTIVE, 4, B, T, SLOTS, MINB>;
    p.threads = T;
    p.per_thread = B;
    p.smem = sizeof(double) * SLOTS;
    p.hot = SLOTS;
}

// Kernel shape: one 1024-thread block per SM (32 warps), 24576 hot slots (192 KB of shared
// memory: one table per SM instead of two 8192-slot copies), 2 virtual nodes per thread (45
// registers).  Measured at cfg4 (relax ms/launch): rounds 1-2 -- 256x2 blocks, 8192 slots 1.53;
// 512x1, 24576 1.15; 768x1 with 4 vnodes/thread, 24576 1.12-1.17 (the round-2b shape); 768x1,
// 28672 1.21; 1024x1 with 4 vnodes/thread (spills) 1.16.  Round 2d on one box (dev build):
// 1024x2v 1.129, 1024x3v 1.149, 1024x1v 1.138, 1024x2v with 26624 / 28672 slots 1.148 / 1.141
// (more shared memory leaves less L1 for the per-vnode gathers; fewer slots lose hot coverage:
// 20480 / 16384 / 12288 slots 1.150 / 1.160 / 1.371); shipped build, alternating
// runs: 1024x2v 1.139 against 768x4v 1.174 (with the probe test in the push, see the kernel).
// Timing decomposition (TIGR_PR_EXP): without the global reductions 0.78 ms, without the
// hot-slot adds 1.17 ms -- the reductions and the per-vnode gathers are what overlap.
// TIGR_PR_CFG selects the alternatives in development builds (dev_knob).
PrCidPlan pr_cid_plan(tigr_vgraph* vg) {
    PrCidPlan p;
    switch (dev_knob("TIGR_PR_CFG", 7)) {
        case 0: fill_plan<4, 256, 8192, 2>(p, vg->layout, (int)vg->unit); break;
        case 1: fill_plan<4, 512, 24576, 1>(p, vg->layout, (int)vg->unit); break;
        case 5: fill_plan<4, 768, 24576, 1>(p, vg->layout, (int)vg->unit); break;
        case 6: fill_plan<4, 768, 28672, 1>(p, vg->layout, (int)vg->unit); break;
        default: fill_plan<2, 1024, 24576, 1>(p, vg->layout, (int)vg->unit); break;
    }
    cudaFuncSetAttribute(p.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem);
    int per_sm = 0, dev = 0, sms = 148;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, p.fn, p.threads, p.smem);
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t per_tile = (uint64_t)p.threads * p.per_thread;
    p.tiles = (unsigned)(((uint64_t)(vg->hi - vg->lo) + per_tile - 1) / per_tile);
    p.grid = (unsigned)std::min<uint64_t>(p.tiles, (uint64_t)sms * (per_sm > 0 ? per_sm : 1));
    return p;
}

// arcs (non-pad slots) of the vnode range [lo, hi) and those among them with id >= hot
__global__ void k_count_reds(const uint32_t* __restrict__ col_pr,
                             const uint32_t* __restrict__ cptr, const uint32_t* __restrict__ vptr, uint32_t n,
                             uint32_t lo, uint32_t hi, uint32_t hot, unsigned long long* __restrict__ out) {
    unsigned long long a = 0, r = 0;
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint32_t f = vptr[v];
        if (vptr[v + 1] == f || f < lo || f >= hi) continue;  // no arcs, or another rank's family
        for (uint64_t q = (uint64_t)cptr[v] * kSpan; q < (uint64_t)cptr[v + 1] * kSpan; ++q) {
            const uint32_t c = col_pr[q];
            if (c == kPad) continue;
            ++a;
            r += c >= hot;
        }
    }
    for (int o = 16; o > 0; o >>= 1) {
        a += __shfl_xor_sync(0xffffffffu, a, o);
        r += __shfl_xor_sync(0xffffffffu, r, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(out, a); atomicAdd(out + 1, r); }
}

tigr_status pr_cid_profile(tigr_vgraph* vg, cudaStream_t s, uint64_t* arcs, uint64_t* reds, uint32_t* hot,
                           uint32_t* n_in) {
    if (!vg->vec) return fail(TIGR_EUNSUPPORTED, "vgraph_pr_profile: the accumulator-order relax needs 4 | K");
    if (vg->g->transposed) return fail(TIGR_EUNSUPPORTED, "vgraph_pr_profile: push PageRank only");
    TIGR_TRY(pr_cid_prepare(vg, s));
    const PrCidPlan p = pr_cid_plan(vg);
    TmpBuf cnt;
    TIGR_TRY(cnt.alloc(2 * sizeof(unsigned long long), s));
    TIGR_CK(cudaMemsetAsync(cnt.p, 0, 2 * sizeof(unsigned long long), s));
    const uint32_t n = vg->g->n;
    k_count_reds<<<grid_cap(n, 16), kBlock, 0, s>>>(vg->ws.col_pr.as<uint32_t>(), vg->g->cptr.as<uint32_t>(),
                                                    vg->vnode_ptr.as<uint32_t>(), n, vg->lo, vg->hi, p.hot,
                                                    cnt.as<unsigned long long>());
    TIGR_CKL("pr profile");
    unsigned long long h[2] = {0, 0};
    TIGR_CK(cudaMemcpyAsync(h, cnt.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    if (arcs) *arcs = h[0];
    if (reds) *reds = h[1];
    if (hot) *hot = p.hot;
    if (n_in) *n_in = (uint32_t)vg->ws.n_in;
    return TIGR_OK;
}

tigr_status pr_cid_apply(tigr_vgraph* vg, double base, double damping, int dangling, const double* dsum_cur,
                         double* dsum_next, cudaStream_t s, double* acc, bool reset) {
    Workspace& ws = vg->ws;
    const uint32_t n = vg->g->n;
    if (!acc) acc = ws.acc.as<double>();
    k_pr_apply_cid<<<grid_for(n), kBlock, 0, s>>>(n, vg->g->deg.as<uint32_t>(), ws.cid.as<uint32_t>(), ws.n_in, base,
                                                  damping, dangling, ws.x.as<double>(), ws.contrib.as<double>(),
                                                  acc, dsum_cur, dsum_next);
    TIGR_CKL("pr apply (cid)");
    // only the first n_in accumulator entries are ever written
    if (reset) TIGR_CK(cudaMemsetAsync(acc, 0, sizeof(double) * ws.n_in, s));
    return TIGR_OK;
}

}  // namespace tigr

// ==========================================================================================
// Pull-based PageRank: the relax runs on a virtual split of the
// TRANSPOSED graph (tigr_graph_transpose).  Virtual node i of node v owns <= K in-arcs u->v
// and gathers partial = sum contrib[u]; Thm. 3 (L1047-1073): pull is correct on a virtual split
// iff the combine is associative and the family's partials meet with atomics.  Lanes of one
// family are consecutive virtual nodes, so a warp first reduces its family segments with a
// key-equality segmented scan (shfl_up); the segment's last lane then stores (the segment is
// the whole family) or adds atomically (the family spans warps).  No arc-level atomics at all.
// ==========================================================================================
namespace tigr {
namespace {

template <int LAYOUT, int U, int B>
__global__ void __launch_bounds__(256) k_relax_pr_pull(RelaxArgs a) {
    const int lane = threadIdx.x & 31;
    const uint64_t base = (uint64_t)a.lo + (uint64_t)blockIdx.x * (B * 256) + threadIdx.x;
    const uint4* c4 = reinterpret_cast<const uint4*>(a.col);
    uint32_t v[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint64_t i = base + (uint64_t)r * 256;
        v[r] = i < a.hi ? __ldg(a.vn_phys + i) : kPad;
    }
    uint4 info[B];
#pragma unroll
    for (int r = 0; r < B; ++r) info[r] = v[r] != kPad ? __ldg(a.vinfo + v[r]) : make_uint4(0, 0, 0, 1);
    uint4 c0[B], c1[B];
    uint32_t kn[B], kend[B], step[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint64_t i = base + (uint64_t)r * 256;
        uint32_t k;
        if (v[r] == kPad) { k = 0; step[r] = 1; kend[r] = 0; }
        else unit_range<U, LAYOUT>(info[r].y, (uint32_t)(i - info[r].z), info[r].w, a.K, k, step[r], kend[r]);
        kn[r] = load8<U>(c4, info[r].x, k, step[r], kend[r], c0[r], c1[r], make_uint4(kPad, kPad, kPad, kPad));
    }
    double part[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint32_t nb[8] = {c0[r].x, c0[r].y, c0[r].z, c0[r].w, c1[r].x, c1[r].y, c1[r].z, c1[r].w};
        double g[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) g[q] = nb[q] != kPad ? __ldg(a.contrib + nb[q]) : 0.0;
        double s = 0.0;
#pragma unroll
        for (int q = 0; q < 8; ++q) s += g[q];
        for (uint32_t k = kn[r]; k < kend[r];) {  // units beyond the first 8 slots
            uint4 c, d;
            k = load8<U>(c4, info[r].x, k, step[r], kend[r], c, d, make_uint4(kPad, kPad, kPad, kPad));
            const uint32_t nb2[8] = {c.x, c.y, c.z, c.w, d.x, d.y, d.z, d.w};
#pragma unroll
            for (int q = 0; q < 8; ++q) s += nb2[q] != kPad ? __ldg(a.contrib + nb2[q]) : 0.0;
        }
        part[r] = s;
    }
#pragma unroll
    for (int r = 0; r < B; ++r) {
        // segmented (by node) inclusive sum across the warp's consecutive virtual nodes
        const uint32_t key = v[r];
        double val = part[r];
        uint32_t len = 1;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const double ov = __shfl_up_sync(0xffffffffu, val, o);
            const uint32_t ok = __shfl_up_sync(0xffffffffu, key, o);
            const uint32_t ol = __shfl_up_sync(0xffffffffu, len, o);
            if (lane >= o && ok == key) { val += ov; len += ol; }
        }
        const uint32_t next = __shfl_down_sync(0xffffffffu, key, 1);
        const bool last = (lane == 31) || (next != key);
        if (key != kPad && last) {
            const uint64_t i_last = base + (uint64_t)r * 256;
            const bool whole = (i_last + 1 - len == info[r].z) && (len == info[r].w);
            if (whole) a.acc[key] = val;
            else atomicAdd(a.acc + key, val);
        }
    }
}

}  // namespace

RelaxFn relax_pr_pull_kernel(int layout, int unit, int* per_thread) {
    *per_thread = 4;
    if (unit == 8)
        return layout == TIGR_LAYOUT_STRIDED ? &k_relax_pr_pull<TIGR_LAYOUT_STRIDED, 8, 4>
                                             : &k_relax_pr_pull<TIGR_LAYOUT_CONSECUTIVE, 8, 4>;
    return layout == TIGR_LAYOUT_STRIDED ? &k_relax_pr_pull<TIGR_LAYOUT_STRIDED, 4, 4>
                                         : &k_relax_pr_pull<TIGR_LAYOUT_CONSECUTIVE, 4, 4>;
}

}  // namespace tigr
