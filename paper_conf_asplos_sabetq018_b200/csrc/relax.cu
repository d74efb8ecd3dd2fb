// relax.cu -- relax kernels and iteration control.
//
// One thread per virtual node (the paper's scheduling unit: "threads are scheduled based on
// the virtually transformed graph ... each thread is assigned to process a virtual node",
// §4.4; Alg. 2, Alg. 3):
//   v = vn_phys[i]                                   (Alg. 2 line 2, "main difference")
//   x = value[v]                                     (Alg. 2 line 3; BSP: previous iteration)
//   for its <= K edges e (stride order, Alg. 3 line 7):
//       alt = f(x, w_e);  if better(alt, value[nbr]) then atomic{Min,Max}(&value[nbr], alt)
//                                                     and mark nbr active (worklist, §5)
// PageRank pushes contrib[v] = x[v]/d_v with a float64 atomic add (fn. 7 L1078: the vertex
// function is split into an associative accumulate and a separate apply; Thm. 3).
// B200 specifics: edges and weights move as 16-byte chunks through the non-coherent read-only
// path; the value gathers of a thread's edges are issued together before its atomics; all of
// a family's virtual nodes share one 16-byte node record; the worklist is an iteration stamp
// per node (no per-iteration clearing pass); the loop runs on the device as a CUDA graph.
#include "internal.cuh"
#include "vgraph.cuh"
#include "relax.cuh"
#include "devutil.cuh"

#include <algorithm>

namespace tigr {

// ------------------------------------------------------------------------------------------
// edge walk: the set of (nbr, w) slots a virtual node owns, in the layout's order
// ------------------------------------------------------------------------------------------
// Calls f(nbr[8], w[8]) on batches of up to 8 slots (pads/absent = kPad).  U: arcs per
// assignment unit -- 8 (32-byte span), 4 (16-byte chunk) or 1 (one arc; 4 does not divide K).
template <int LAYOUT, int U, bool W, class F>
__device__ __forceinline__ void walk(const uint32_t* __restrict__ col, const uint32_t* __restrict__ wt,
                                     uint32_t cbase, uint32_t d, uint32_t j, uint32_t mv, uint32_t K, F&& f) {
    uint32_t nb[8], ww[8];
    if (U > 1) {
        const uint4* c4 = reinterpret_cast<const uint4*>(col);
        const uint4* w4 = reinterpret_cast<const uint4*>(wt);
        uint32_t k, step, kend;
        unit_range<(U > 1 ? U : 4), LAYOUT>(d, j, mv, K, k, step, kend);
        while (k < kend) {
            uint4 a, b, wa = make_uint4(0, 0, 0, 0), wb = wa;
            const uint32_t next = load8<(U > 1 ? U : 4)>(c4, cbase, k, step, kend, a, b, make_uint4(kPad, kPad, kPad, kPad));
            if (W) load8<(U > 1 ? U : 4)>(w4, cbase, k, step, kend, wa, wb, make_uint4(0, 0, 0, 0));
            k = next;
            nb[0] = a.x; nb[1] = a.y; nb[2] = a.z; nb[3] = a.w;
            nb[4] = b.x; nb[5] = b.y; nb[6] = b.z; nb[7] = b.w;
            ww[0] = wa.x; ww[1] = wa.y; ww[2] = wa.z; ww[3] = wa.w;
            ww[4] = wb.x; ww[5] = wb.y; ww[6] = wb.z; ww[7] = wb.w;
            f(nb, ww);
        }
    } else {
        const uint32_t* cs = col + (uint64_t)cbase * kChunk;
        const uint32_t* ws = wt + (uint64_t)cbase * kChunk;
        uint32_t p, step, pend;
        if (LAYOUT == TIGR_LAYOUT_STRIDED) { p = j; step = mv; pend = d; }
        else { p = j * K; step = 1; pend = (K >= d - p) ? d : p + K; }
        while (p < pend) {
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const uint32_t pt = p + t * step;
                const bool ok = pt < pend;
                nb[t] = ok ? ldg_u32(cs + pt) : kPad;
                ww[t] = (W && ok) ? ldg_u32(ws + pt) : 0;
            }
            f(nb, ww);
            p += 8 * step;
        }
    }
}

// ------------------------------------------------------------------------------------------
// relax kernel
// ------------------------------------------------------------------------------------------
template <int A, int LAYOUT, int U, int FRONT, bool BSP, bool STATS>
__global__ void __launch_bounds__(kRelaxThreads) k_relax(RelaxArgs a) {
    constexpr bool W = (A == TIGR_SSSP || A == TIGR_SSWP);
    if (!a.ctl->cont) return;  // an iteration enqueued past the fixed point (batched host loop, run.cu)
    const uint64_t i = (uint64_t)a.lo + (uint64_t)blockIdx.x * kRelaxThreads + threadIdx.x;
    const uint32_t it = (FRONT == TIGR_FRONTIER_DENSE) ? a.ctl->it : 0;
    bool touched = false;
    uint32_t n_edges = 0, n_upd = 0, n_vn = 0;
    if (i < a.hi) {
        const uint32_t v = a.vn_phys[i];
        bool act = true;
        if (FRONT == TIGR_FRONTIER_DENSE) act = a.stamp[(uint64_t)(it & 1u) * a.n + v] == stamp_of(it);
        uint32_t x = 0;
        if (act) {
            x = BSP ? a.prev[v] : a.val[v];
            if (FRONT == TIGR_FRONTIER_NONE) {
                if ((A == TIGR_BFS || A == TIGR_SSSP) && x == kInf) act = false;
                if (A == TIGR_SSWP && x == 0) act = false;
            }
        }
        if (act) {
            const uint4 info = a.vinfo[v];  // {chunk base, degree, first vnode, family size}
            const uint32_t j = (uint32_t)(i - info.z);
            if (STATS) n_vn = 1;
            walk<LAYOUT, U, W>(a.col, a.wt, info.x, info.y, j, info.w, a.K,
                                 [&](const uint32_t* nb, const uint32_t* ww) {
                uint32_t cur[8];
#pragma unroll
                for (int t = 0; t < 8; ++t) cur[t] = (nb[t] != kPad) ? a.val[nb[t]] : 0u;
#pragma unroll
                for (int t = 0; t < 8; ++t) {
                    if (nb[t] == kPad) continue;
                    if (STATS) ++n_edges;
                    const uint32_t alt = combine<A>(x, ww[t]);
                    if (better<A>(alt, cur[t])) {
                        if (A == TIGR_SSWP) atomicMax(a.val + nb[t], alt);
                        else atomicMin(a.val + nb[t], alt);
                        if (FRONT == TIGR_FRONTIER_DENSE) a.stamp[(uint64_t)((it + 1) & 1u) * a.n + nb[t]] = stamp_of(it + 1);
                        touched = true;
                        if (STATS) ++n_upd;
                    }
                }
            });
        }
    }
    if (__any_sync(0xffffffffu, touched) && (threadIdx.x & 31) == 0) a.ctl->changed = 1;
    if (STATS) {
        unsigned long long e = n_edges, u = n_upd, q = n_vn;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            e += __shfl_xor_sync(0xffffffffu, e, o);
            u += __shfl_xor_sync(0xffffffffu, u, o);
            q += __shfl_xor_sync(0xffffffffu, q, o);
        }
        if ((threadIdx.x & 31) == 0) {
            if (e) atomicAdd(&a.ctl->edges, e);
            if (u) atomicAdd(&a.ctl->updates, u);
            if (q) atomicAdd(&a.ctl->vnodes, q);
        }
    }
}

// Frontier relax with B virtual nodes per thread (16-byte-chunk layouts, no stats): every
// stage -- vnode -> node id, activity stamp, node record + value, the first two edge (and
// weight) chunks, the target-value gathers -- is issued for all B vnodes before the first
// use, so a warp keeps ~8B independent loads in flight instead of one dependent chain.
template <int A, int LAYOUT, int U, int FRONT, bool BSP, int B>
__global__ void __launch_bounds__(kRelaxThreads) k_relax_mlp(RelaxArgs a) {
    constexpr bool W = (A == TIGR_SSSP || A == TIGR_SSWP);
    if (!a.ctl->cont) return;  // past the fixed point (batched host loop)
    const uint64_t base = (uint64_t)a.lo + (uint64_t)blockIdx.x * (B * kRelaxThreads) + threadIdx.x;
    const uint32_t it = (FRONT == TIGR_FRONTIER_DENSE) ? a.ctl->it : 0;
    const stamp_t* stamp_cur = a.stamp + (uint64_t)(it & 1u) * a.n;   // not written in this launch
    stamp_t* stamp_next = a.stamp + (uint64_t)((it + 1) & 1u) * a.n;
    const stamp_t s_cur = stamp_of(it), s_next = stamp_of(it + 1);
    const uint4* c4 = reinterpret_cast<const uint4*>(a.col);
    const uint4* w4 = reinterpret_cast<const uint4*>(a.wt);
    bool touched = false;

    uint32_t v[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint64_t i = base + (uint64_t)r * kRelaxThreads;
        v[r] = i < a.hi ? __ldg(a.vn_phys + i) : kPad;
    }
    bool act[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        act[r] = v[r] != kPad;
        if (FRONT == TIGR_FRONTIER_DENSE && act[r]) act[r] = __ldg(stamp_cur + v[r]) == s_cur;
    }
    uint32_t x[B];
    uint4 info[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        x[r] = 0;
        info[r] = make_uint4(0, 0, 0, 1);
        if (act[r]) {
            x[r] = BSP ? __ldg(a.prev + v[r]) : a.val[v[r]];
            info[r] = __ldg(a.vinfo + v[r]);
        }
    }
    bool any = false;
#pragma unroll
    for (int r = 0; r < B; ++r) {
        if (FRONT == TIGR_FRONTIER_NONE) {
            if ((A == TIGR_BFS || A == TIGR_SSSP) && x[r] == kInf) act[r] = false;
            if (A == TIGR_SSWP && x[r] == 0) act[r] = false;
        }
        any |= act[r];
    }
    // a warp whose 4x32 virtual nodes are all inactive leaves now: sparse iterations cost one
    // coalesced vn_phys read and one stamp gather per virtual node, not the whole relax body
    if (!__any_sync(0xffffffffu, any)) return;
    uint4 c0[B], c1[B], w0[B], w1[B];
    uint32_t kn[B], kend[B], step[B];
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint64_t i = base + (uint64_t)r * kRelaxThreads;
        uint32_t k;
        if (!act[r]) { k = 0; step[r] = 1; kend[r] = 0; }
        else unit_range<U, LAYOUT>(info[r].y, (uint32_t)(i - info[r].z), info[r].w, a.K, k, step[r], kend[r]);
        kn[r] = load8<U>(c4, info[r].x, k, step[r], kend[r], c0[r], c1[r], make_uint4(kPad, kPad, kPad, kPad));
        if (W) load8<U>(w4, info[r].x, k, step[r], kend[r], w0[r], w1[r], make_uint4(0, 0, 0, 0));
    }
    auto relax8 = [&](const uint32_t* nb, const uint32_t* ww, uint32_t xv) {
        uint32_t cur[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) cur[q] = (nb[q] != kPad) ? a.val[nb[q]] : 0u;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (nb[q] == kPad) continue;
            const uint32_t alt = combine<A>(xv, W ? ww[q] : 0u);
            if (better<A>(alt, cur[q])) {
                if (A == TIGR_SSWP) atomicMax(a.val + nb[q], alt);
                else atomicMin(a.val + nb[q], alt);
                if (FRONT == TIGR_FRONTIER_DENSE) stamp_next[nb[q]] = s_next;
                touched = true;
            }
        }
    };
#pragma unroll
    for (int r = 0; r < B; ++r) {
        const uint32_t nb[8] = {c0[r].x, c0[r].y, c0[r].z, c0[r].w, c1[r].x, c1[r].y, c1[r].z, c1[r].w};
        uint32_t ww[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        if (W) { ww[0] = w0[r].x; ww[1] = w0[r].y; ww[2] = w0[r].z; ww[3] = w0[r].w;
                 ww[4] = w1[r].x; ww[5] = w1[r].y; ww[6] = w1[r].z; ww[7] = w1[r].w; }
        relax8(nb, ww, x[r]);
    }
#pragma unroll
    for (int r = 0; r < B; ++r) {  // units beyond the first 8 slots (K > 8 or no split)
        for (uint32_t k = kn[r]; k < kend[r];) {
            uint4 a0, a1, b0 = make_uint4(0, 0, 0, 0), b1 = b0;
            const uint32_t next = load8<U>(c4, info[r].x, k, step[r], kend[r], a0, a1, make_uint4(kPad, kPad, kPad, kPad));
            if (W) load8<U>(w4, info[r].x, k, step[r], kend[r], b0, b1, make_uint4(0, 0, 0, 0));
            k = next;
            const uint32_t nb[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
            const uint32_t ww[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
            relax8(nb, ww, x[r]);
        }
    }
    if (__any_sync(0xffffffffu, touched) && (threadIdx.x & 31) == 0) a.ctl->changed = 1;
}

template <int A, int LAYOUT, int U>
static RelaxFn pick_mlp(int front, bool bsp) {
#define TIGR_MLP(F, BS) if (front == F && bsp == BS) return &k_relax_mlp<A, LAYOUT, U, F, BS, 4>;
    TIGR_MLP(TIGR_FRONTIER_DENSE, false) TIGR_MLP(TIGR_FRONTIER_DENSE, true)
    TIGR_MLP(TIGR_FRONTIER_NONE, false) TIGR_MLP(TIGR_FRONTIER_NONE, true)
#undef TIGR_MLP
    return nullptr;
}

template <int A>
static RelaxFn pick_mlp_lu(int layout, int unit, int front, bool bsp) {
    if (layout == TIGR_LAYOUT_STRIDED)
        return unit == 8 ? pick_mlp<A, TIGR_LAYOUT_STRIDED, 8>(front, bsp) : pick_mlp<A, TIGR_LAYOUT_STRIDED, 4>(front, bsp);
    return unit == 8 ? pick_mlp<A, TIGR_LAYOUT_CONSECUTIVE, 8>(front, bsp)
                     : pick_mlp<A, TIGR_LAYOUT_CONSECUTIVE, 4>(front, bsp);
}

// multi-vnode frontier kernel (4 virtual nodes per thread; the 2-per-thread shape measured
// slower), or nullptr (then relax_kernel's one-vnode-per-thread kernel)
RelaxFn relax_mlp_kernel(int algo, int layout, int unit, int front, bool bsp, bool stats, int* per_thread) {
    if (unit < 4 || stats || algo == TIGR_PR) return nullptr;
    *per_thread = 4;
    switch (algo) {
        case TIGR_BFS: return pick_mlp_lu<TIGR_BFS>(layout, unit, front, bsp);
        case TIGR_SSSP: return pick_mlp_lu<TIGR_SSSP>(layout, unit, front, bsp);
        case TIGR_CC: return pick_mlp_lu<TIGR_CC>(layout, unit, front, bsp);
        case TIGR_SSWP: return pick_mlp_lu<TIGR_SSWP>(layout, unit, front, bsp);
    }
    return nullptr;
}

template <int LAYOUT, int U, bool STATS>
__global__ void __launch_bounds__(kRelaxThreads) k_relax_pr(RelaxArgs a) {
    const uint64_t i = (uint64_t)a.lo + (uint64_t)blockIdx.x * kRelaxThreads + threadIdx.x;
    uint32_t n_edges = 0;
    if (i < a.hi) {
        const uint32_t v = a.vn_phys[i];
        const double x = a.contrib[v];
        const uint4 info = a.vinfo[v];
        const uint32_t j = (uint32_t)(i - info.z);
        walk<LAYOUT, U, false>(a.col, a.wt, info.x, info.y, j, info.w, a.K,
                                 [&](const uint32_t* nb, const uint32_t*) {
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                if (nb[t] == kPad) continue;
                atomicAdd(a.acc + nb[t], x);  // RED.ADD.F64 (result unused)
                if (STATS) ++n_edges;
            }
        });
    }
    if (STATS) {
        unsigned long long e = n_edges;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
        if ((threadIdx.x & 31) == 0 && e) atomicAdd(&a.ctl->edges, e);
        if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(&a.ctl->vnodes, (unsigned long long)(a.hi - a.lo));
    }
}

// sampled in-degree (PageRank accumulator order, pr.cu): every kHotSampleStride-th 16-byte
// chunk of the arc array
constexpr int kHotSampleStride = 16;

__global__ void k_hot_sample(const uint4* __restrict__ c4, uint64_t nchunks, uint32_t* __restrict__ cnt) {
    for (uint64_t k = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * kHotSampleStride; k < nchunks;
         k += (uint64_t)gridDim.x * blockDim.x * kHotSampleStride) {
        const uint4 c = __ldg(c4 + k);
        if (c.x != kPad) atomicAdd(cnt + c.x, 1u);
        if (c.y != kPad) atomicAdd(cnt + c.y, 1u);
        if (c.z != kPad) atomicAdd(cnt + c.z, 1u);
        if (c.w != kPad) atomicAdd(cnt + c.w, 1u);
    }
}

// ------------------------------------------------------------------------------------------
// dispatch
// ------------------------------------------------------------------------------------------
template <int A, int LAYOUT, int U>
static RelaxFn pick_front(int front, bool bsp, bool stats) {
#define TIGR_PICK(F, B, S) if (front == F && bsp == B && stats == S) return &k_relax<A, LAYOUT, U, F, B, S>;
    TIGR_PICK(TIGR_FRONTIER_DENSE, false, false)
    TIGR_PICK(TIGR_FRONTIER_DENSE, false, true)
    TIGR_PICK(TIGR_FRONTIER_DENSE, true, false)
    TIGR_PICK(TIGR_FRONTIER_DENSE, true, true)
    TIGR_PICK(TIGR_FRONTIER_NONE, false, false)
    TIGR_PICK(TIGR_FRONTIER_NONE, false, true)
    TIGR_PICK(TIGR_FRONTIER_NONE, true, false)
    TIGR_PICK(TIGR_FRONTIER_NONE, true, true)
#undef TIGR_PICK
    return nullptr;
}

template <int A, int LAYOUT>
static RelaxFn pick_unit(int unit, int front, bool bsp, bool stats) {
    if (unit == 8) return pick_front<A, LAYOUT, 8>(front, bsp, stats);
    if (unit == 4) return pick_front<A, LAYOUT, 4>(front, bsp, stats);
    return pick_front<A, LAYOUT, 1>(front, bsp, stats);
}

template <int A>
static RelaxFn pick_layout(int layout, int unit, int front, bool bsp, bool stats) {
    if (layout == TIGR_LAYOUT_STRIDED) return pick_unit<A, TIGR_LAYOUT_STRIDED>(unit, front, bsp, stats);
    return pick_unit<A, TIGR_LAYOUT_CONSECUTIVE>(unit, front, bsp, stats);
}

template <int LAYOUT>
static RelaxFn pick_pr(int unit, bool stats) {
    if (unit == 8) return stats ? &k_relax_pr<LAYOUT, 8, true> : &k_relax_pr<LAYOUT, 8, false>;
    if (unit == 4) return stats ? &k_relax_pr<LAYOUT, 4, true> : &k_relax_pr<LAYOUT, 4, false>;
    return stats ? &k_relax_pr<LAYOUT, 1, true> : &k_relax_pr<LAYOUT, 1, false>;
}

RelaxFn relax_kernel(int algo, int layout, int unit, int front, bool bsp, bool stats) {
    switch (algo) {
        case TIGR_BFS: return pick_layout<TIGR_BFS>(layout, unit, front, bsp, stats);
        case TIGR_SSSP: return pick_layout<TIGR_SSSP>(layout, unit, front, bsp, stats);
        case TIGR_CC: return pick_layout<TIGR_CC>(layout, unit, front, bsp, stats);
        case TIGR_SSWP: return pick_layout<TIGR_SSWP>(layout, unit, front, bsp, stats);
        case TIGR_PR:
            return layout == TIGR_LAYOUT_STRIDED ? pick_pr<TIGR_LAYOUT_STRIDED>(unit, stats)
                                                 : pick_pr<TIGR_LAYOUT_CONSECUTIVE>(unit, stats);
    }
    return nullptr;
}

// ------------------------------------------------------------------------------------------
// init / control / PR apply / multi-GPU diff / assignment dump
// ------------------------------------------------------------------------------------------
__global__ void k_init(int algo, uint32_t n, uint32_t source, uint32_t* __restrict__ val,
                       stamp_t* __restrict__ stamp, Ctl* ctl, uint32_t max_iters,
                       const uint32_t* __restrict__ cid, const uint32_t* __restrict__ order,
                       uint32_t* __restrict__ settled) {
    // reordered graphs (tigr_graph_reorder): the source is an original id, CC labels are
    // original ids (the minimum original id of the component)
    const uint32_t src = cid ? cid[source] : source;
    // four nodes per thread (16-byte value and 4-byte stamp stores) when n % 4 == 0
    const bool vec = (n & 3u) == 0;
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    auto init_val = [&](uint32_t v) -> uint32_t {
        uint32_t x = kInf;
        if (algo == TIGR_CC) x = order ? order[v] : v;
        else if (algo == TIGR_SSWP) x = 0;
        if (v == src && algo != TIGR_CC) x = (algo == TIGR_SSWP) ? kInf : 0;
        return x;
    };
    auto init_stamp1 = [&](uint32_t v) -> uint32_t {  // parity 1: active in iteration 1
        return (algo == TIGR_CC || v == src) ? stamp_of(1) : 0;
    };
    const uint32_t v0 = vec ? 4 * t : t;
    if (vec && v0 < n) {
        reinterpret_cast<uint4*>(val)[t] = make_uint4(init_val(v0), init_val(v0 + 1), init_val(v0 + 2), init_val(v0 + 3));
        reinterpret_cast<uint32_t*>(stamp)[t] = 0u;  // parity 0: never stamped
        reinterpret_cast<uint32_t*>(stamp + n)[t] = init_stamp1(v0) | (init_stamp1(v0 + 1) << 8) |
                                                    (init_stamp1(v0 + 2) << 16) | (init_stamp1(v0 + 3) << 24);
    } else if (!vec && v0 < n) {
        val[v0] = init_val(v0);
        stamp[v0] = 0;
        stamp[(uint64_t)n + v0] = (stamp_t)init_stamp1(v0);
    }
    // BFS: the source's level 0 is final from the start; its settled bit (cleared before this
    // kernel; frontier_kernel.cuh) spares every gather of it -- R-MAT's source is a hub
    if (settled && t == 0 && algo == TIGR_BFS && src < n) atomicOr(settled + (src >> 5), 1u << (src & 31u));
    if (t == 0) {
        ctl->changed = 0; ctl->it = 1; ctl->max_iters = max_iters; ctl->cont = 1; ctl->notconv = 0;
        ctl->xchanged[0] = 0; ctl->xchanged[1] = 0;
        ctl->edges = 0; ctl->updates = 0; ctl->vnodes = 0; ctl->dsum[0] = 0.0; ctl->dsum[1] = 0.0;
        ctl->qpack[0] = 0ull; ctl->qpack[1] = 0ull; ctl->queue_iters = 0; ctl->nodes = 0;
    }
}

// results of a reordered graph back to original ids: out[v] = val[cid[v]]
template <class T>
__global__ void k_unpermute(uint32_t n, const uint32_t* __restrict__ cid, const T* __restrict__ val,
                            T* __restrict__ out) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v < n) out[v] = val[cid[v]];
}

tigr_status unpermute(uint32_t n, const uint32_t* cid, const void* val, void* out, bool f64, cudaStream_t s) {
    if (f64) k_unpermute<double><<<grid_for(n), kBlock, 0, s>>>(n, cid, (const double*)val, (double*)out);
    else k_unpermute<uint32_t><<<grid_for(n), kBlock, 0, s>>>(n, cid, (const uint32_t*)val, (uint32_t*)out);
    TIGR_CKL("unpermute");
    return TIGR_OK;
}

// end of one iteration: decide whether to continue; sets the graph's WHILE condition
__global__ void k_control(Ctl* ctl, cudaGraphConditionalHandle h, int use_handle) {
    if (!ctl->cont) {  // already stopped: an iteration enqueued past the fixed point (run.cu)
        if (use_handle) cudaGraphSetConditional(h, 0);
        return;
    }
    const uint32_t changed = ctl->changed;
    ctl->nodes += ctl->qpack[ctl->it & 1u] >> 32;
    ctl->qpack[ctl->it & 1u] = 0ull;  // queue slot consumed by this iteration (frontier.cu)
    uint32_t cont = changed ? 1u : 0u;
    if (changed && ctl->it >= ctl->max_iters) { cont = 0; ctl->notconv = 1; }
    ctl->changed = 0;
    if (cont) ctl->it += 1;
    ctl->cont = cont;
    if (use_handle) cudaGraphSetConditional(h, cont);
}

// multi-GPU: after the all-reduce, activate every node whose replica value moved
__global__ void k_diff(uint32_t n, const uint32_t* __restrict__ val, uint32_t* __restrict__ prev,
                       stamp_t* __restrict__ stamp, Ctl* ctl) {
    if (!ctl->cont) return;  // past the fixed point (batched host loop, run.cu)
    const uint32_t it = ctl->it;
    bool moved = false;
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v < n) {
        const uint32_t x = val[v];
        if (x != prev[v]) { prev[v] = x; stamp[(uint64_t)((it + 1) & 1u) * n + v] = stamp_of(it + 1); moved = true; }
    }
    if (__any_sync(0xffffffffu, moved) && (threadIdx.x & 31) == 0) ctl->changed = 1;
}

// block-reduce a double and add it to *dst with one atomic per block (kBlock threads)
__device__ __forceinline__ void block_add(double v, double* dst) {
    __shared__ double part[kBlock / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < kBlock / 32; ++w) t += part[w];
        if (t != 0.0) atomicAdd(dst, t);
    }
}

__global__ void k_pr_init(uint32_t n, const uint32_t* __restrict__ deg, double* __restrict__ x,
                          double* __restrict__ contrib, double* __restrict__ acc, Ctl* ctl,
                          const uint32_t* __restrict__ oid) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    double dang = 0.0;
    if (v < n) {
        const double x0 = 1.0 / (double)n;
        const uint32_t d = deg[v];
        x[v] = x0;
        contrib[oid ? oid[v] : v] = d ? __ddiv_rn(x0, (double)d) : 0.0;
        acc[v] = 0.0;
        if (!d) dang = x0;
    }
    block_add(dang, &ctl->dsum[0]);
}

// x = (1-d)/n + d*(acc + dsum/n);  contrib = x/deg;  acc = 0;  next dangling mass -> dsum_next
__global__ void k_pr_apply(uint32_t n, const uint32_t* __restrict__ deg, double base, double damping,
                           int dangling, double* __restrict__ x, double* __restrict__ contrib,
                           double* __restrict__ acc, const double* dsum_cur, double* dsum_next,
                           const uint32_t* __restrict__ oid) {
    const uint32_t v = blockIdx.x * blockDim.x + threadIdx.x;
    double dang = 0.0;
    if (v < n) {
        double s = acc[v];
        if (dangling) s = __dadd_rn(s, __ddiv_rn(*dsum_cur, (double)n));
        const double r = __dadd_rn(base, __dmul_rn(damping, s));  // no FMA: matches the oracle
        const uint32_t d = deg[v];
        x[v] = r;
        contrib[oid ? oid[v] : v] = d ? __ddiv_rn(r, (double)d) : 0.0;
        acc[v] = 0.0;
        if (!d) dang = r;
    }
    if (dangling) block_add(dang, dsum_next);
}

// per-vnode edge lists, walked with the relax kernels' own arithmetic (layout parity tests)
template <int LAYOUT, int U>
__global__ void k_assign(RelaxArgs a, const uint32_t* __restrict__ offs, uint32_t* __restrict__ counts,
                         uint32_t* __restrict__ nbr, uint32_t* __restrict__ wout, int weighted, int pass) {
    const uint64_t i = (uint64_t)blockIdx.x * kRelaxThreads + threadIdx.x;
    if (i >= a.hi) return;
    const uint32_t v = a.vn_phys[i];
    const uint4 info = a.vinfo[v];
    const uint32_t j = (uint32_t)(i - info.z);
    uint32_t c = 0;
    const uint32_t base = pass ? offs[i] : 0;
    const uint32_t* wt = weighted ? a.wt : a.col;
    walk<LAYOUT, U, true>(a.col, wt, info.x, info.y, j, info.w, a.K,
                            [&](const uint32_t* nb, const uint32_t* ww) {
        for (int t = 0; t < 8; ++t) {
            if (nb[t] == kPad) continue;
            if (pass) {
                nbr[base + c] = nb[t];
                if (wout && weighted) wout[base + c] = ww[t];
            }
            ++c;
        }
    });
    if (!pass) counts[i] = c;
}

AssignFn assign_kernel(int layout, int unit) {
    if (layout == TIGR_LAYOUT_STRIDED)
        return unit == 8 ? &k_assign<TIGR_LAYOUT_STRIDED, 8>
                         : (unit == 4 ? &k_assign<TIGR_LAYOUT_STRIDED, 4> : &k_assign<TIGR_LAYOUT_STRIDED, 1>);
    return unit == 8 ? &k_assign<TIGR_LAYOUT_CONSECUTIVE, 8>
                     : (unit == 4 ? &k_assign<TIGR_LAYOUT_CONSECUTIVE, 4> : &k_assign<TIGR_LAYOUT_CONSECUTIVE, 1>);
}

}  // namespace tigr
