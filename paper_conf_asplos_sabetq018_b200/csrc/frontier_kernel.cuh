// frontier_kernel.cuh -- queue-driven frontier relax with dynamic virtual-node mapping
// (§8(f) NEXT-3 "dynamic mapping reasoning").
//
// The paper's worklist (§5) keeps the nodes whose value changed; its "dynamic
// mapping reasoning" (§4.1) derives a node's virtual nodes from the degree bound at
// run time instead of storing the virtual node array ("before processing node v2, a
// reasoning runtime finds its degree is 6, which is greater than K, hence splits it into two
// virtual nodes (ceil(6/3))").  Here both meet:
//
//   k_compact  after each iteration, the nodes stamped active for the next iteration that own
//              virtual nodes in this rank's range are appended to a queue {node, offset}, where
//              offset is the exclusive prefix of the family sizes m_v = ceil(d_v/K) in queue
//              order (one 64-bit atomic per 2048-node tile packs entry and vnode counts, so
//              offsets increase with the entry index).
//   k_relax_fq the next relax covers the queue's virtual nodes t in [0, total): a warp takes 32
//              consecutive t per round, finds the queue entry of its first t with a 32-ary
//              search over the offsets (ballot per step), and maps every lane to its entry with
//              one OR-reduction of entry-start bits (entries own >= 1 vnode, so 32 entries
//              always cover 32 vnodes).  Lane t then is virtual node j = t - offset of node v,
//              and walks the same <= K arcs, in the same strided (Fig. 12) or consecutive
//              (Fig. 10) order, as virtual node vnode_ptr[v] + j of the stored array would.
//              No vn_phys read at all: the mapping is reasoned from the queue and the node
//              record.
//   When the queue holds many virtual nodes (>= 1/div of this rank's), the same kernel
//   instead sweeps the stored virtual node array with the stamp test (the dense frontier of
//   relax.cu): per-iteration cost then tracks the active work in sparse iterations and the
//   streaming rate in dense ones.  The choice is made on the device from the queue size, so
//   the whole loop stays one CUDA graph launch.
//
// The relax itself is Alg. 2/3 unchanged: x = value[v]; for each arc alt = f(x, w); if
// better(alt, value[nbr]) then atomic{Min,Max} and stamp nbr for the next iteration.
//
// BFS settled bitmap.  The relax is bound by the L1/L2 sector traffic of the random 4-byte
// target gathers (profiles/r01_ncu_frontier_units.csv), so BFS first tests one bit of a 2 MB
// bitmap (hot targets stay L1-resident) and gathers the level only for targets whose bit is
// clear.  This is exact because BFS levels are final on first assignment under this
// worklist, asynchronous schedule included: by induction, the nodes active in iteration it
// all hold level it-1 (they were lowered to it-1 in iteration it-1, and every candidate of
// iteration it-1 was it-1), so every candidate of iteration it equals it and can never lower
// a value assigned earlier; on replicas the same holds rank-wide.  A bit is set next to an
// atomicMin whose candidate beat the observed level (the level then ends at it, final), so a
// set bit never hides an improvement; a stale clear bit (another SM's atomicOr not yet
// visible through this SM's L1) only costs the level gather the plain test would have done.
// CC uses the same bitmap for one exact case: a label lowered to 0, the smallest id, is
// final (nothing is better than 0), and on power-law graphs the giant component -- most
// targets -- carries label 0 after the first iterations.
// SSSP and SSWP test the value itself: a bitmap settled by the frontier bound (values below the
// minimum active value, SSSP, or at least the maximum, SSWP, are final) was built and measured
// slower (cfg4 SSSP 2.68 -> 4.03 ms): in their heavy iterations few targets are
// final, so the bit test only adds a second dependent access before the value gather.
//
// This header holds the relax kernel template; frontier_{bfs,sssp,sswp,cc}.cu instantiate it
// for one algorithm each (parallel compilation), frontier.cu holds the queue build and the
// dispatch.  Everything here has internal linkage (anonymous namespace): each translation
// unit owns the kernels it instantiates.
#pragma once

#include <cstdlib>

#include "devutil.cuh"
#include "internal.cuh"
#include "relax.cuh"
#include "vgraph.cuh"

namespace tigr {
namespace {

constexpr int kFqThreads = 256;
constexpr uint32_t kFull = 0xffffffffu;

// largest k in [0, qn) with qo[k] <= t (qo increasing, qo[0] == 0 <= t): 32-ary search, one
// ballot per step
__device__ __forceinline__ uint32_t warp_search(const uint32_t* __restrict__ qo, uint32_t qn, uint32_t t, int lane) {
    uint32_t lo = 0, hi = qn;
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t idx = lo + (uint32_t)lane * step;
        const bool p = idx < hi && __ldg(qo + idx) <= t;
        const uint32_t b = __ballot_sync(kFull, p);
        const uint32_t L = 31u - __clz(b);  // lane 0 always holds (qo[lo] <= t)
        lo += L * step;
        hi = min(hi, lo + step);
    }
    const uint32_t idx = lo + (uint32_t)lane;
    const uint32_t b = __ballot_sync(kFull, idx < hi && __ldg(qo + idx) <= t);
    return lo + (31u - __clz(b));
}

// map lanes of round start tr (vnodes tr + lane) to queue entries, starting from a window
// whose first entry starts at or before tr.  Returns the lane's (node, vnode index j) and the
// entry index the next round may start from.
__device__ __forceinline__ void map_round(const uint32_t* __restrict__ qv, const uint32_t* __restrict__ qo,
                                          uint32_t qn, uint32_t& k, uint32_t tr, int lane, uint32_t& v,
                                          uint32_t& j) {
    uint32_t idx = k + (uint32_t)lane;
    uint32_t off = idx < qn ? __ldg(qo + idx) : kInf;
    // entries starting at or before tr form a prefix of the window; its last one owns tr.
    // Rebase the window there, so that its 32 entries (>= 1 vnode each) cover tr .. tr + 31.
    const uint32_t le = __ballot_sync(kFull, off <= tr);
    const int first = 31 - __clz(le);  // le != 0: the window's first entry starts at or before tr
    if (first > 0) {                   // warp-uniform
        k += (uint32_t)first;
        idx = k + (uint32_t)lane;
        off = idx < qn ? __ldg(qo + idx) : kInf;
    }
    const uint32_t node = idx < qn ? __ldg(qv + idx) : kPad;
    uint32_t bit = 0;
    if (lane == 0) bit = 1u;
    else if (off < tr + 32u) bit = 1u << (off - tr);  // off > tr here
    const uint32_t starts = __reduce_or_sync(kFull, bit);
    const uint32_t upto = lane == 31 ? kFull : ((2u << lane) - 1u);
    const int e = __popc(starts & upto) - 1;  // window lane of this lane's entry
    v = __shfl_sync(kFull, node, e);
    const uint32_t eo = __shfl_sync(kFull, off, e);
    j = (tr + (uint32_t)lane) - eo;
    k += (uint32_t)__shfl_sync(kFull, e, 31);
}

// Fused exchange (TIGR_EXCHANGE_FUSED, exchange.cu): an improvement found by this rank is
// applied, in the same branch, to every peer's replica with the relax's own atomic (over
// NVLink when the peer is another GPU) and activates the node there too -- the peers see it
// like an update from one more SM.  Only improvements travel: bytes ~ updates x (P-1) x 8.
// Scope: a replica word receives atomics from its owner GPU and from every peer GPU at once, so
// with peers every atomic on a replica -- the owner's own included (apply8) -- is system-scope
// (atom.sys): only atomics whose scopes include each other are atomic with respect to each other
// in the PTX memory model, and a gpu-scope atomic does not include another GPU's threads.  The
// stamp stores and the plain value gathers are ordered by the end-of-iteration barrier (kernel
// completion, stream sync, host barrier); a gather that misses a concurrent peer update reads a
// stale larger (smaller, SSWP) value, which only costs an atomic that cannot lower it -- the same
// benign staleness as between the SMs of one GPU.
template <int A>
__device__ __forceinline__ void atomic_better_sys(uint32_t* p, uint32_t alt) {
    if (A == TIGR_SSWP) atomicMax_system(p, alt);
    else atomicMin_system(p, alt);
}

template <int A>
__device__ __forceinline__ void push_peers(const FusedPeers* __restrict__ pp, uint32_t n, uint32_t it, uint32_t v,
                                           uint32_t alt) {
    const uint64_t slot = (uint64_t)((it + 1) & 1u) * n;
    for (int r = 0; r < pp->P; ++r) {
        if (r == pp->me) continue;
        atomic_better_sys<A>(pp->val[r] + v, alt);
        pp->stamp[r][slot + v] = stamp_of(it + 1);
    }
}


// PK (SSSP / SSWP): the arcs come from the packed array f.cw -- target | (w - wmin) << idbits in
// one 32-bit slot (run.cu packs it once per virtual graph when ids and weights fit), so one span
// load per 8 arcs brings targets and weights together instead of two.
template <int A, int LAYOUT, int U, bool BSP, int B, bool STATS, int MINB, bool PRE, bool PK = false>
__global__ void __launch_bounds__(kFqThreads, MINB) k_relax_fq(RelaxArgs a, FqArgs f) {
    constexpr bool W = (A == TIGR_SSSP || A == TIGR_SSWP);
    static_assert(!PK || W, "packed arcs carry weights");
    constexpr uint32_t kFinal = 0u;  // a settled BFS / CC target reads as 0: never improvable
    const bool BITS = (A == TIGR_BFS || A == TIGR_CC) && f.settled != nullptr;  // uniform per launch
    if (!a.ctl->cont) return;  // an iteration enqueued past the fixed point (batched host loop, run.cu)
    const int lane = threadIdx.x & 31;
    const uint32_t it = a.ctl->it;
    const unsigned long long qp = a.ctl->qpack[it & 1u];
    const uint32_t qn = (uint32_t)(qp >> 32), qt = (uint32_t)qp;
    const uint64_t span = (uint64_t)(a.hi - a.lo);
    const bool queue = f.mode == 1 || (f.mode == 0 && (uint64_t)qt * f.dense_div < span);
    const uint32_t* qv = f.qv + (uint64_t)(it & 1u) * a.n;
    const uint32_t* qo = f.qo + (uint64_t)(it & 1u) * a.n;
    const stamp_t* stamp_cur = a.stamp + (uint64_t)(it & 1u) * a.n;
    stamp_t* stamp_next = a.stamp + (uint64_t)((it + 1) & 1u) * a.n;
    const stamp_t s_cur = stamp_of(it), s_next = stamp_of(it + 1);
    const uint4* c4 = reinterpret_cast<const uint4*>(PK ? f.cw : a.col);
    const uint4* w4 = reinterpret_cast<const uint4*>(a.wt);
    if (blockIdx.x == 0 && threadIdx.x == 0 && queue) atomicAdd(&a.ctl->queue_iters, 1u);
    // 8 slots -> targets (kPad for pads) and weights
    auto decode8 = [&](const uint4& c, const uint4& d, const uint4& wc, const uint4& wd, uint32_t* nb, uint32_t* ww) {
        const uint32_t raw[8] = {c.x, c.y, c.z, c.w, d.x, d.y, d.z, d.w};
        const uint32_t wr[8] = {wc.x, wc.y, wc.z, wc.w, wd.x, wd.y, wd.z, wd.w};
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (PK) {
                const uint32_t t = raw[q] & f.idmask;
                nb[q] = t == f.idmask ? kPad : t;
                ww[q] = (raw[q] >> f.idbits) + f.wmin;
            } else {
                nb[q] = raw[q];
                ww[q] = W ? wr[q] : 0u;
            }
        }
    };
    const uint64_t total = queue ? (uint64_t)qt : span;
    constexpr uint32_t kTile = 32u * B;
    const uint64_t tiles = (total + kTile - 1) / kTile;
    const uint64_t warp0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    bool touched = false;
    uint32_t n_edges = 0, n_upd = 0, n_vn = 0;
    // Tiles go to warps in runs of kRun consecutive tiles, the runs interleaved across warps:
    // within a run the queue entry index carries over from one tile to the next (map_round
    // leaves it at an entry that starts at or before the next round), so the 32-ary search --
    // a chain of dependent loads -- runs once per run, while the interleaving keeps all warps
    // sweeping the queue front to back together.  Measured at cfg4 (profiles/r02_frontier_tiles.txt,
    // reordered graph, ms): runs of 1 / 2 / 4 / 8 tiles: BFS 1.32 / 1.27 / 1.27 / 1.37, SSSP 2.20 /
    // 2.15 / 2.18 / 2.27, CC 2.96 / 2.92 / 2.90 / 2.95.  One contiguous range per warp saved the
    // most searches but raised the asynchronous schedule's redundant work (SSSP +10 % time).
    const uint32_t kRun = f.run;  // tiles per run (2; FqArgs)
    const uint32_t nruns = (uint32_t)((tiles + kRun - 1) / kRun);  // tiles < 2^32 / 32
    uint32_t kq = 0;
    for (uint32_t run = (uint32_t)warp0; run < nruns; run += (uint32_t)nwarps)
    for (uint32_t tile = run * kRun; tile < min(run * kRun + kRun, (uint32_t)tiles); ++tile) {
        const uint64_t t0 = (uint64_t)tile * kTile;
        uint32_t v[B], j[B];
        bool act[B];
        if (queue) {
            if (tile == run * kRun) kq = warp_search(qo, qn, (uint32_t)t0, lane);
            uint32_t k = kq;
#pragma unroll
            for (int r = 0; r < B; ++r) {
                const uint32_t tr = (uint32_t)t0 + 32u * r;
                if (tr < qt) {  // warp-uniform
                    map_round(qv, qo, qn, k, tr, lane, v[r], j[r]);
                    act[r] = tr + (uint32_t)lane < qt;
                } else {
                    v[r] = kPad; j[r] = 0; act[r] = false;
                }
                if (!act[r]) v[r] = kPad;
            }
            kq = k;
        } else {
#pragma unroll
            for (int r = 0; r < B; ++r) {
                const uint64_t i = (uint64_t)a.lo + t0 + 32u * r + lane;
                v[r] = i < a.hi ? __ldg(a.vn_phys + i) : kPad;
                j[r] = (uint32_t)i;  // absolute vnode index; made family-relative below
            }
#pragma unroll
            for (int r = 0; r < B; ++r) act[r] = v[r] != kPad && __ldg(stamp_cur + v[r]) == s_cur;
        }
        uint32_t x[B];
        uint4 info[B];
        bool any = false;
#pragma unroll
        for (int r = 0; r < B; ++r) {
            x[r] = 0;
            info[r] = make_uint4(0, 0, 0, 1);
            if (act[r]) {
                x[r] = BSP ? __ldg(a.prev + v[r]) : a.val[v[r]];
                info[r] = __ldg(a.vinfo + v[r]);
            }
            any |= act[r];
        }
        if (!__any_sync(kFull, any)) continue;
        uint4 c0[B], c1[B], w0[B], w1[B];
        uint32_t kn[B], kend[B], step[B];
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t jj = queue ? j[r] : j[r] - info[r].z;  // offset within the family
            uint32_t k;
            if (!act[r]) { k = 0; step[r] = 1; kend[r] = 0; }
            else unit_range<U, LAYOUT>(info[r].y, jj, info[r].w, a.K, k, step[r], kend[r]);
            // the first 8 slots: one span (U = 8) or two chunks (U = 4)
            kn[r] = load8<U>(c4, info[r].x, k, step[r], kend[r], c0[r], c1[r], make_uint4(kPad, kPad, kPad, kPad));
            if (W && !PK) load8<U>(w4, info[r].x, k, step[r], kend[r], w0[r], w1[r], make_uint4(0, 0, 0, 0));
            else w0[r] = w1[r] = make_uint4(0, 0, 0, 0);
            if (STATS && act[r]) ++n_vn;
        }
        // settled bitmap (f.settled): the test reads one bit of an n/8-byte array instead of the
        // 4-byte value (see the header); a settled target reads as kFinal (never improvable)
        auto gather8 = [&](const uint32_t* nb, uint32_t* cur) {
            if (BITS) {
                uint32_t b[8];
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    b[q] = (nb[q] == kPad) ? 1u : (f.settled[nb[q] >> 5] >> (nb[q] & 31u)) & 1u;
#pragma unroll
                for (int q = 0; q < 8; ++q) cur[q] = b[q] ? kFinal : a.val[nb[q]];
                return;
            }
#pragma unroll
            for (int q = 0; q < 8; ++q) cur[q] = (nb[q] == kPad) ? kFinal : a.val[nb[q]];
        };
        auto apply8 = [&](const uint32_t* nb, const uint32_t* ww, uint32_t xv, const uint32_t* cur) {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                if (nb[q] == kPad) continue;
                if (STATS) ++n_edges;
                const uint32_t alt = combine<A>(xv, W ? ww[q] : 0u);
                if (better<A>(alt, cur[q])) {
                    if (f.peers) {  // fused exchange: system-scope on every replica (push_peers)
                        atomic_better_sys<A>(a.val + nb[q], alt);
                        push_peers<A>(f.peers, a.n, it, nb[q], alt);
                    } else if (A == TIGR_SSWP) {
                        atomicMax(a.val + nb[q], alt);
                    } else {
                        atomicMin(a.val + nb[q], alt);
                    }
                    // BFS: the level becomes alt = it, final (see the header); CC: label 0 is final
                    if (BITS && (A == TIGR_BFS || (A == TIGR_CC && alt == 0u)))
                        atomicOr(f.settled + (nb[q] >> 5), 1u << (nb[q] & 31u));
                    stamp_next[nb[q]] = s_next;
                    touched = true;
                    if (STATS) ++n_upd;
                }
            }
        };
        auto relax8 = [&](const uint32_t* nb, const uint32_t* ww, uint32_t xv) {
            uint32_t cur[8];
            gather8(nb, cur);
            apply8(nb, ww, xv, cur);
        };
        if (PRE) {  // every target value of the first two chunks of all B vnodes in flight at once
            uint32_t cur[B][8];
#pragma unroll
            for (int r = 0; r < B; ++r) {
                uint32_t nb[8], ww[8];
                decode8(c0[r], c1[r], w0[r], w1[r], nb, ww);
                gather8(nb, cur[r]);
            }
#pragma unroll
            for (int r = 0; r < B; ++r) {
                uint32_t nb[8], ww[8];
                decode8(c0[r], c1[r], w0[r], w1[r], nb, ww);
                apply8(nb, ww, x[r], cur[r]);
            }
        } else {
#pragma unroll
            for (int r = 0; r < B; ++r) {
                uint32_t nb[8], ww[8];
                decode8(c0[r], c1[r], w0[r], w1[r], nb, ww);
                relax8(nb, ww, x[r]);
            }
        }
#pragma unroll
        for (int r = 0; r < B; ++r) {  // units beyond the first 8 slots (K > 8 or no split)
            for (uint32_t k = kn[r]; k < kend[r];) {
                uint4 a0, a1, b0 = make_uint4(0, 0, 0, 0), b1 = b0;
                const uint32_t next = load8<U>(c4, info[r].x, k, step[r], kend[r], a0, a1, make_uint4(kPad, kPad, kPad, kPad));
                if (W && !PK) load8<U>(w4, info[r].x, k, step[r], kend[r], b0, b1, make_uint4(0, 0, 0, 0));
                k = next;
                uint32_t nb[8], ww[8];
                decode8(a0, a1, b0, b1, nb, ww);
                relax8(nb, ww, x[r]);
            }
        }
    }
    if (__any_sync(kFull, touched) && lane == 0) {
        if (f.peers) {  // every rank's verdict for this iteration, read after the group barrier
            for (int r = 0; r < f.peers->P; ++r)
                *reinterpret_cast<volatile uint32_t*>(&f.peers->ctl[r]->xchanged[it & 1u]) = 1u;
        } else {
            a.ctl->changed = 1;
        }
    }
    if (STATS) {
        unsigned long long e = n_edges, u = n_upd, q = n_vn;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            e += __shfl_xor_sync(kFull, e, o);
            u += __shfl_xor_sync(kFull, u, o);
            q += __shfl_xor_sync(kFull, q, o);
        }
        if (lane == 0) {
            if (e) atomicAdd(&a.ctl->edges, e);
            if (u) atomicAdd(&a.ctl->updates, u);
            if (q) atomicAdd(&a.ctl->vnodes, q);
        }
    }
}

// Kernel shape per algorithm (cfg4 sweep, tools/dev/fq_sweep.sh): the relax
// is bound by L1tex wavefronts of the random target-value gathers and by latency, so
// occupancy matters more than per-thread depth.  BFS and CC (settled bitmap): see pick_fq;
// BSP / stats variants: 4 vnodes per thread, 80 registers, 3 blocks/SM.  Weighted (SSSP, SSWP; one more 16-byte load per chunk): 2 vnodes
// per thread with all target gathers of both issued before the first atomic, 3 blocks/SM.
template <int A, int LAYOUT, int U>
FqFn pick_fq_u(bool bsp, bool stats, bool packed) {
    constexpr bool W = (A == TIGR_SSSP || A == TIGR_SSWP);
    constexpr int B = W ? 2 : 4;
    constexpr bool PRE = W;
    if constexpr (W) {  // packed target | weight arcs (asynchronous schedule, no stats)
        if (packed && !bsp && !stats) return &k_relax_fq<A, LAYOUT, U, false, B, false, 3, PRE, true>;
    }
    if (!bsp && !stats) {  // TIGR_FQ_SHAPE: alternative shapes in development builds
        // BFS and CC with their settled bitmap are latency-bound rather than L1/L2-bound
        // (profiles/README.md): 2 virtual nodes per thread with all gathers issued first,
        // 4 blocks/SM (64 registers, no spills); cfg4 BFS 1.47 -> 1.34 ms, CC 3.44 -> 3.07 ms
        const int dflt = (A == TIGR_BFS || A == TIGR_CC) ? 1 : 0;
        switch (dev_knob("TIGR_FQ_SHAPE", dflt)) {
            case 1: return &k_relax_fq<A, LAYOUT, U, false, 2, false, 4, true>;
            default: break;
        }
    }
    if (bsp) return stats ? &k_relax_fq<A, LAYOUT, U, true, B, true, 3, PRE> : &k_relax_fq<A, LAYOUT, U, true, B, false, 3, PRE>;
    return stats ? &k_relax_fq<A, LAYOUT, U, false, B, true, 3, PRE> : &k_relax_fq<A, LAYOUT, U, false, B, false, 3, PRE>;
}

template <int A>
FqFn pick_fq(int layout, int unit, bool bsp, bool stats, bool packed) {
    if (layout == TIGR_LAYOUT_STRIDED)
        return unit == 8 ? pick_fq_u<A, TIGR_LAYOUT_STRIDED, 8>(bsp, stats, packed)
                         : pick_fq_u<A, TIGR_LAYOUT_STRIDED, 4>(bsp, stats, packed);
    return unit == 8 ? pick_fq_u<A, TIGR_LAYOUT_CONSECUTIVE, 8>(bsp, stats, packed)
                     : pick_fq_u<A, TIGR_LAYOUT_CONSECUTIVE, 4>(bsp, stats, packed);
}

}  // namespace
}  // namespace tigr
