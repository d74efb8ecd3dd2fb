// exchange.cu -- the per-iteration merge of the replicated value array across ranks for the
// frontier algorithms (§8(f) NEXT-2 "exchange only changed vertices").
//
// Each rank relaxes only its own virtual nodes (a contiguous, family-aligned range) against a
// full replica of the values, so after the relax the replicas differ exactly at the nodes some
// rank improved.  Every local improvement is stamped for the next iteration in the same branch
// that issues the atomic (frontier rule), so a rank's stamps for it+1 are a superset
// of the nodes whose value it changed.  Two ways to merge:
//
//   dense   in-place all-reduce of all n values (MIN / MAX), then k_diff activates the nodes whose
//           replica value moved against the snapshot `prev` -- 2(P-1)/P * 4n bytes per rank.
//   sparse  each rank packs {node, value} of its stamped nodes (k_pack), the list lengths are
//           all-gathered, every rank reads all P lists and applies them with the same atomic as
//           the relax (k_apply_lists), stamping every listed node; then `prev` is refreshed at
//           the listed nodes (k_lists_prev).  8 bytes per changed node.
//
// Both leave every replica with the elementwise MIN (MAX) of the replicas and the same set of
// nodes active on every rank (in sparse mode: the union of the lists, which every rank sees),
// so every rank takes the same termination decision with no extra collective, and the fixed
// point -- hence the result -- is the single-GPU one (min/max are associative, commutative,
// idempotent; Thm. 2 L1030-1045 carries over to replicas).  AUTO picks sparse while the lists
// hold at most n/2 records in total (the dense all-reduce moves 4n bytes either way).
#include <algorithm>

#include "internal.cuh"
#include "relax.cuh"
#include "vgraph.cuh"

namespace tigr {

tigr_status comm_allreduce(tigr_comm* c, void* buf, size_t count, int algo, cudaStream_t s);
tigr_status comm_allgather_count(tigr_comm* c, const uint32_t* dev_count, uint32_t* host_counts, cudaStream_t s);
tigr_status comm_share_lists(tigr_comm* c, const void* mine, const uint32_t* counts, const void** ptrs,
                             cudaStream_t s);
tigr_status comm_release_lists(tigr_comm* c, cudaStream_t s);
tigr_status comm_share_ptrs(tigr_comm* c, const void* const* mine, int k, const void** all);
tigr_status comm_sync_barrier(tigr_comm* c, cudaStream_t s);

namespace {

constexpr int kMaxLists = 16;
struct Lists {
    const uint2* p[kMaxLists];
    uint32_t cnt[kMaxLists];
};

// {node, value} of every node stamped for iteration it + 1 (warp-aggregated append)
__global__ void k_pack(uint32_t n, const uint32_t* __restrict__ val, const stamp_t* __restrict__ stamp, Ctl* ctl,
                       uint2* __restrict__ out) {
    const uint32_t it = ctl->it;
    const stamp_t* st = stamp + (uint64_t)((it + 1) & 1u) * n;
    const stamp_t sn = stamp_of(it + 1);
    const int lane = threadIdx.x & 31;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t b = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); b < n; b += stride) {
        const uint64_t v = b + lane;
        const bool on = v < n && st[v] == sn;
        const uint32_t mask = __ballot_sync(0xffffffffu, on);
        if (!mask) continue;
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(&ctl->xcount, (uint32_t)__popc(mask));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (on) out[base + __popc(mask & ((1u << lane) - 1u))] = make_uint2((uint32_t)v, val[v]);
    }
}

// apply the other ranks' records with the relax's own atomic; activate every listed node
template <int A>
__global__ void k_apply_lists(Lists L, int me, uint32_t n, uint32_t* __restrict__ val, stamp_t* __restrict__ stamp,
                              const Ctl* ctl) {
    const int r = blockIdx.y;
    if (r == me) return;  // this rank's own records are already in its replica and its stamps
    const uint32_t it = ctl->it;
    stamp_t* st = stamp + (uint64_t)((it + 1) & 1u) * n;
    const uint2* p = L.p[r];
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < L.cnt[r]; i += gridDim.x * blockDim.x) {
        const uint2 e = p[i];
        if (A == TIGR_SSWP) atomicMax(val + e.x, e.y);
        else atomicMin(val + e.x, e.y);
        st[e.x] = stamp_of(it + 1);
    }
}

// prev := val at every listed node (all ranks' lists, this rank's included): outside the
// lists no replica value moved, so prev == val holds again everywhere
__global__ void k_lists_prev(Lists L, const uint32_t* __restrict__ val, uint32_t* __restrict__ prev) {
    const int r = blockIdx.y;
    const uint2* p = L.p[r];
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < L.cnt[r]; i += gridDim.x * blockDim.x) {
        const uint32_t v = p[i].x;
        prev[v] = val[v];
    }
}

// fused exchange, end of an iteration: this rank's verdict is every rank's flag for it
__global__ void k_fused_settle(Ctl* ctl) {
    const uint32_t slot = ctl->it & 1u;
    ctl->changed = ctl->xchanged[slot];
    ctl->xchanged[slot] = 0;  // no rank writes this slot again before iteration it + 2
}

tigr_status dense(const ExchangeArgs& x, cudaStream_t s) {
    TIGR_TRY(comm_allreduce(x.comm, x.val, x.n, x.algo, s));
    // the local `changed` flag is rank-local: reset it so k_control only sees k_diff's verdict
    TIGR_CK(cudaMemsetAsync(&x.ctl->changed, 0, sizeof(uint32_t), s));
    k_diff<<<grid_for(x.n), kBlock, 0, s>>>(x.n, x.val, x.prev, x.stamp, x.ctl);
    TIGR_CKL("exchange diff");
    return TIGR_OK;
}

}  // namespace

// Fused exchange (TIGR_EXCHANGE_FUSED; peer-group transports: thread group or node group).  There is no exchange step:
// the relax itself applies each improvement to every peer's replica and stamp array
// (frontier.cu push_peers) and raises every rank's xchanged flag.  What remains per iteration
// is ordering: a barrier once every rank's relax has drained (all remote updates have landed),
// then each rank reads the common verdict.  Before the first iteration every replica must be
// initialised (barrier after init); in BSP mode the snapshot is taken between two barriers so
// that no peer's update of the new iteration leaks into it.
tigr_status fused_setup(tigr_comm* c, uint32_t* val, stamp_t* stamp, Ctl* ctl, DevBuf& peers_buf,
                        cudaStream_t s, const FusedPeers** out) {
    if (!c->local) return fail(TIGR_EUNSUPPORTED, "fused exchange needs a thread-group or node communicator");
    if (c->nranks > kMaxPeers) return fail(TIGR_EUNSUPPORTED, "fused exchange: more than 16 ranks");
    const void* mine[3] = {val, stamp, ctl};
    const void* all[3 * kMaxPeers] = {};
    TIGR_TRY(comm_share_ptrs(c, mine, 3, all));
    FusedPeers h{};
    h.P = c->nranks;
    h.me = c->rank;
    for (int r = 0; r < c->nranks; ++r) {
        h.val[r] = const_cast<uint32_t*>(static_cast<const uint32_t*>(all[3 * r]));
        h.stamp[r] = const_cast<stamp_t*>(static_cast<const stamp_t*>(all[3 * r + 1]));
        h.ctl[r] = const_cast<Ctl*>(static_cast<const Ctl*>(all[3 * r + 2]));
    }
    if (!peers_buf.p) TIGR_TRY(peers_buf.alloc(sizeof(FusedPeers), s));
    TIGR_CK(cudaMemcpyAsync(peers_buf.p, &h, sizeof(FusedPeers), cudaMemcpyHostToDevice, s));
    TIGR_CK(cudaStreamSynchronize(s));  // h is a stack copy
    *out = peers_buf.as<FusedPeers>();
    return TIGR_OK;
}

tigr_status fused_barrier(tigr_comm* c, cudaStream_t s) { return comm_sync_barrier(c, s); }

tigr_status fused_end_iteration(tigr_comm* c, Ctl* ctl, cudaStream_t s) {
    TIGR_TRY(comm_sync_barrier(c, s));
    k_fused_settle<<<1, 1, 0, s>>>(ctl);
    TIGR_CKL("fused settle");
    return TIGR_OK;
}

tigr_status exchange_frontier(const ExchangeArgs& x, cudaStream_t s, bool* sparse_used) {
    *sparse_used = false;
    if (x.mode == TIGR_EXCHANGE_DENSE) return dense(x, s);
    tigr_comm* c = x.comm;
    if (c->nranks > kMaxLists) return fail(TIGR_EUNSUPPORTED, "sparse exchange: more than 16 ranks");
    TIGR_CK(cudaMemsetAsync(&x.ctl->xcount, 0, sizeof(uint32_t), s));
    if (x.n) {
        int dev = 0, sms = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const unsigned grid = (unsigned)std::min<uint64_t>(grid_for(x.n), (uint64_t)sms * 8);
        k_pack<<<grid, kBlock, 0, s>>>(x.n, x.val, x.stamp, x.ctl, x.list);
        TIGR_CKL("exchange pack");
    }
    uint32_t counts[kMaxLists] = {};
    TIGR_TRY(comm_allgather_count(c, &x.ctl->xcount, counts, s));
    uint64_t total = 0, most = 0;
    for (int r = 0; r < c->nranks; ++r) {
        total += counts[r];
        most = std::max<uint64_t>(most, counts[r]);
    }
    if (x.mode == TIGR_EXCHANGE_AUTO && 2 * total > (uint64_t)x.n) return dense(x, s);  // same verdict on every rank
    const void* ptrs[kMaxLists] = {};
    TIGR_TRY(comm_share_lists(c, x.list, counts, ptrs, s));
    Lists L{};
    for (int r = 0; r < c->nranks; ++r) {
        L.p[r] = static_cast<const uint2*>(ptrs[r]);
        L.cnt[r] = counts[r];
    }
    if (most) {
        const dim3 grid((unsigned)std::min<uint64_t>(grid_for(most), 1024), (unsigned)c->nranks);
        switch (x.algo) {
            case TIGR_SSWP: k_apply_lists<TIGR_SSWP><<<grid, kBlock, 0, s>>>(L, c->rank, x.n, x.val, x.stamp, x.ctl); break;
            default: k_apply_lists<TIGR_BFS><<<grid, kBlock, 0, s>>>(L, c->rank, x.n, x.val, x.stamp, x.ctl); break;
        }
        TIGR_CKL("exchange apply");
        k_lists_prev<<<grid, kBlock, 0, s>>>(L, x.val, x.prev);
        TIGR_CKL("exchange prev");
    }
    TIGR_TRY(comm_release_lists(c, s));
    // converged iff no rank changed anything: every rank sees the same counts
    TIGR_CK(cudaMemsetAsync(&x.ctl->changed, total ? 1 : 0, sizeof(uint32_t), s));
    *sparse_used = true;
    return TIGR_OK;
}

}  // namespace tigr
