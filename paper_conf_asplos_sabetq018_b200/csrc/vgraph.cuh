// vgraph.cuh -- the virtual graph handle and its run workspace (internal).
#pragma once

#include <map>
#include <vector>
#include <tuple>

#include "internal.cuh"

namespace tigr {

// Device-side control block of one run (one per vgraph workspace).
struct Ctl {
    uint32_t changed;      // set by relax when any value improved this iteration
    uint32_t it;           // current iteration (1-based; node v is active iff stamp[v] == stamp_of(it))
    uint32_t max_iters;
    uint32_t cont;         // 1 while the loop should continue (host-loop mode reads it)
    uint32_t notconv;      // 1 if the cap was hit while values still changed
    uint32_t xchanged[2];  // fused multi-GPU exchange: set by any rank's relax in iteration it (slot it&1)
    uint32_t pad;
    unsigned long long edges, updates, vnodes;
    double dsum[2];        // PR: dangling mass of the iterate (parity of the iteration)
    // active-node queue of iteration it (frontier.cu): slot it&1 packs (entries << 32) | vnodes
    unsigned long long qpack[2];
    uint32_t queue_iters;  // iterations the queue-driven (dynamic-mapping) path ran
    uint32_t xcount;       // multi-GPU sparse exchange: records this rank packed (exchange.cu)
    unsigned long long nodes;  // sum over iterations of active nodes with arcs (queue entries)
};

struct GraphKey {
    int algo, layout_vec, frontier, schedule, stats, comm;
    uint32_t lo, hi;
    const void* relax;  // the relax kernel the graph launches (it depends on packed arcs, dev knobs)
    bool operator<(const GraphKey& o) const {
        return std::tie(algo, layout_vec, frontier, schedule, stats, comm, lo, hi, relax) <
               std::tie(o.algo, o.layout_vec, o.frontier, o.schedule, o.stats, o.comm, o.lo, o.hi, o.relax);
    }
};

struct CachedGraph {
    cudaGraphExec_t exec = nullptr;
    cudaStream_t stream = nullptr;
    int kernels_per_iter = 0;
};

struct Workspace {
    DevBuf val;      // uint32[n] values (BFS/SSSP/CC/SSWP)
    DevBuf prev;     // uint32[n] BSP snapshot / multi-GPU pre-exchange copy
    DevBuf stamp;    // uint8[2n] worklist: node v active in iteration it iff stamp[(it&1)n + v] == stamp_of(it);
                     // relax(it) writes only the other parity, so activations never race reads
    DevBuf x;        // double[n] PR rank
    DevBuf contrib;  // double[n] PR x/deg
    DevBuf acc;      // double[n] PR accumulator
    DevBuf acc2;     // double[n] second accumulator (fused apply alternates the two; pr.cu)
    DevBuf cid;      // uint32[n]: PR accumulator id (in-degree order; pr.cu)
    DevBuf col_pr;   // uint32[4 * nchunks]: arc targets as accumulator ids (PR only)
    uint32_t n_in = 0;       // nodes with in-arcs (= accumulator entries ever written)
    bool cid_ready = false;
    DevBuf qv;       // uint32[2][n]: active-node queue (node ids), one slot per iteration parity
    DevBuf qo;       // uint32[2][n]: first queue-space virtual node of each entry (exclusive prefix)
    DevBuf settled;  // uint32[n/32+1]: BFS / CC settled bitmap (frontier.cu)
    DevBuf cw;       // uint32[4 * nchunks]: SSSP / SSWP packed arcs target | (w - wmin) << idbits
    int cw_state = 0;         // 0 not prepared, 1 packed, 2 ids and weights do not fit 32 bits
    uint32_t cw_idbits = 0, cw_wmin = 0;
    DevBuf xlist;    // uint2[n]: multi-GPU sparse exchange records {node, value} (exchange.cu)
    DevBuf peers;    // FusedPeers (fused multi-GPU exchange, exchange.cu)
    DevBuf ctl;      // Ctl
    Ctl* ctl_host = nullptr;  // pinned mirror for the host loop (owned: pinned_ctl_acquire, run.cu)
    cudaEvent_t ev[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
    std::vector<cudaEvent_t> tev;  // per-relax-launch timing events (time_kernels)
    std::map<GraphKey, CachedGraph> graphs;
    ~Workspace();
};

}  // namespace tigr

struct tigr_vgraph {
    const tigr_graph* g = nullptr;
    uint32_t K = 8;
    tigr_layout layout = TIGR_LAYOUT_STRIDED;
    uint32_t unit = 8;           // arcs per assignment unit: 8 (32-byte span, 8 | K), 4 (16-byte chunk,
                                 // 4 | K) or 1 (virt.cu)
    bool vec = true;             // unit > 1: the chunked kernels (one vector load per unit)
    uint64_t nv = 0;
    tigr::DevBuf vnode_ptr;      // uint32[n+1]
    tigr::DevBuf vn_phys;        // uint32[nv]
    tigr::DevBuf vinfo;          // uint4[n] = {first 16-byte chunk, degree, first vnode, family size}
    uint32_t lo = 0, hi = 0;     // this rank's vnode range
    uint64_t n_out = 0;          // nodes with out-arcs whose virtual nodes lie in [lo, hi)
    uint64_t m_local = 0;        // arcs of the nodes whose virtual nodes lie in [lo, hi)
    double ms_build = 0.0;
    tigr::Workspace ws;
};
