// run.cu -- host orchestration of one algorithm run (SURVEY.md §3 "Build entry points" 3).
//
// Frontier algorithms (BFS/SSSP/CC/SSWP) iterate  [BSP snapshot] -> relax -> [all-reduce ->
// diff] -> control  until no value changes (the paper's `finished` flag, Alg. 2/3, and the
// BSP halting rule, §2.1).  By default the loop is ONE CUDA graph launch: the body is
// captured into the body graph of a conditional WHILE node and k_control sets the condition
// on the device, so there is no host round trip per iteration (the paper copies `finished`
// back every iteration).  PageRank runs pr_iters x (relax -> [all-reduce] -> apply).
#include <algorithm>
#include <mutex>
#include <vector>

#include "internal.cuh"
#include "relax.cuh"
#include "vgraph.cuh"

namespace tigr {

tigr_status comm_allreduce(tigr_comm* c, void* buf, size_t count, int algo, cudaStream_t s);

// Pinned host mirrors of the control block, one per workspace (a vgraph may be run from any
// thread, and two vgraphs may run at once on different threads, so the mirror is never shared).
// cudaMallocHost synchronises the device, and the bench rebuilds its vgraph every step, so
// mirrors come from a process-wide free list that grows in slabs and never shrinks.
namespace {
std::mutex g_ctl_mu;
std::vector<Ctl*> g_ctl_free;
}  // namespace

Ctl* pinned_ctl_acquire() {
    std::lock_guard<std::mutex> lk(g_ctl_mu);
    if (g_ctl_free.empty()) {
        constexpr int kSlab = 64;
        Ctl* slab = nullptr;
        if (cudaMallocHost(&slab, sizeof(Ctl) * kSlab) != cudaSuccess) return nullptr;
        for (int i = kSlab - 1; i >= 0; --i) g_ctl_free.push_back(slab + i);
    }
    Ctl* c = g_ctl_free.back();
    g_ctl_free.pop_back();
    return c;
}

void pinned_ctl_release(Ctl* c) {
    if (!c) return;
    std::lock_guard<std::mutex> lk(g_ctl_mu);
    g_ctl_free.push_back(c);
}

Workspace::~Workspace() {
    pinned_ctl_release(ctl_host);
    for (auto& kv : graphs) {
        if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
        if (kv.second.stream) cudaStreamDestroy(kv.second.stream);
    }
    for (auto& e : ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : tev) cudaEventDestroy(e);
}

namespace {

tigr_status ensure_ws(tigr_vgraph* vg, bool pr, cudaStream_t s) {
    Workspace& ws = vg->ws;
    const size_t n = vg->g->n ? vg->g->n : 1;
    if (!ws.ctl.p) {
        TIGR_TRY(ws.ctl.alloc(sizeof(Ctl), s));
        ws.ctl_host = pinned_ctl_acquire();
        if (!ws.ctl_host) return fail(TIGR_ENOMEM, "cudaMallocHost of the control-block mirror failed");
        for (auto& e : ws.ev) TIGR_CK(cudaEventCreate(&e));
    }
    if (pr) {
        if (!ws.x.p) {
            TIGR_TRY(ws.x.alloc(sizeof(double) * n, s));
            TIGR_TRY(ws.contrib.alloc(sizeof(double) * n, s));
            TIGR_TRY(ws.acc.alloc(sizeof(double) * n, s));
        }
    } else if (!ws.val.p) {
        TIGR_TRY(ws.val.alloc(sizeof(uint32_t) * n, s));
        TIGR_TRY(ws.prev.alloc(sizeof(uint32_t) * n, s));
        TIGR_TRY(ws.stamp.alloc(sizeof(stamp_t) * 2 * n, s));
    }
    if (!pr && vg->vec && !ws.qv.p) {  // active-node queues (frontier.cu), one per iteration parity
        TIGR_TRY(ws.qv.alloc(sizeof(uint32_t) * 2 * n, s));
        TIGR_TRY(ws.qo.alloc(sizeof(uint32_t) * 2 * n, s));
    }
    return TIGR_OK;
}

RelaxArgs make_args(tigr_vgraph* vg) {
    const tigr_graph* g = vg->g;
    RelaxArgs a;
    a.vn_phys = vg->vn_phys.as<uint32_t>();
    a.vinfo = vg->vinfo.as<uint4>();
    a.col = g->col.as<uint32_t>();
    a.wt = g->weighted ? g->wt.as<uint32_t>() : g->col.as<uint32_t>();
    a.lo = vg->lo;
    a.hi = vg->hi;
    a.K = vg->K;
    a.n = g->n;
    a.val = vg->ws.val.as<uint32_t>();
    a.prev = vg->ws.prev.as<uint32_t>();
    a.stamp = vg->ws.stamp.as<stamp_t>();
    a.acc = vg->ws.acc.as<double>();
    a.contrib = vg->ws.contrib.as<double>();
    a.ctl = vg->ws.ctl.as<Ctl>();
    return a;
}

struct FrontierPlan {
    RelaxFn relax;
    ExchangeArgs xa;       // multi-GPU merge (exchange.cu), when comm
    FqFn fq = nullptr;     // queue / dynamic-mapping relax (frontier.cu); relax unused when set
    FqArgs fa;
    const tigr_vgraph* vg = nullptr;
    RelaxArgs args;
    unsigned grid;
    bool bsp, comm;
    bool fused = false;    // TIGR_EXCHANGE_FUSED: the relax updates the peers' replicas itself
    int algo;
    tigr_comm* c;
    uint32_t n;
};

// enqueue one iteration body; returns number of kernels it launches
tigr_status enqueue_body(const FrontierPlan& p, cudaStream_t s, cudaGraphConditionalHandle h, int use_handle,
                         int* kernels, cudaEvent_t ev_a = nullptr, cudaEvent_t ev_b = nullptr,
                         uint32_t* sparse_count = nullptr, cudaEvent_t ev_c = nullptr) {
    int k = 0;
    if (p.bsp && (!p.comm || p.fused))
        TIGR_CK(cudaMemcpyAsync((void*)p.args.prev, p.args.val, sizeof(uint32_t) * p.n, cudaMemcpyDeviceToDevice, s));
    if (p.bsp && p.fused) TIGR_TRY(fused_barrier(p.c, s));  // every snapshot taken before any remote update
    if (ev_a) TIGR_CK(cudaEventRecord(ev_a, s));
    if (p.grid && p.fq) {
        p.fq<<<p.grid, relax_fq_threads(), 0, s>>>(p.args, p.fa);
        TIGR_CK(cudaGetLastError());
        ++k;
    } else if (p.grid) {
        p.relax<<<p.grid, kRelaxThreads, 0, s>>>(p.args);
        TIGR_CK(cudaGetLastError());
        ++k;
    }
    if (ev_b) TIGR_CK(cudaEventRecord(ev_b, s));
    if (p.fused) {  // host loop only: wait for every rank's relax (and its remote updates)
        TIGR_TRY(fused_end_iteration(p.c, p.args.ctl, s));
    } else if (p.comm) {  // host loop only (never captured): the exchange decides on the host
        bool sparse = false;
        TIGR_TRY(exchange_frontier(p.xa, s, &sparse));  // its kernels count their own launches
        if (sparse && sparse_count) ++*sparse_count;
    }
    if (ev_c) TIGR_CK(cudaEventRecord(ev_c, s));
    if (p.fq) {  // next iteration's queue from the stamps just written
        TIGR_TRY(compact_launch(p.vg, p.args.ctl, 1, s));
        ++k;
    }
    k_control<<<1, 1, 0, s>>>(p.args.ctl, h, use_handle);
    TIGR_CK(cudaGetLastError());
    ++k;
    *kernels = k;
    return TIGR_OK;
}

tigr_status run_frontier(tigr_vgraph* vg, int algo, uint32_t source, const tigr_run_opts& o, cudaStream_t s,
                         tigr_stats* st) {
    Workspace& ws = vg->ws;
    const uint32_t n = vg->g->n;
    int front = o.frontier;
    FrontierPlan p;
    p.vg = vg;
    if ((front == TIGR_FRONTIER_AUTO || front == TIGR_FRONTIER_QUEUE) && vg->vec) {
        // SSSP / SSWP: targets and weights packed into one slot when they fit (frontier.cu)
        bool packed = false;
        if ((algo == TIGR_SSSP || algo == TIGR_SSWP) && dev_knob("TIGR_PACK_ARCS", 1)) {
            TIGR_TRY(pack_arcs_prepare(vg, s));
            packed = ws.cw_state == 1;
        }
        p.fq = relax_fq_kernel(algo, vg->layout, (int)vg->unit, o.schedule == 1, o.collect_stats != 0, packed);
        p.fa.cw = packed ? ws.cw.as<uint32_t>() : nullptr;
        p.fa.idbits = packed ? ws.cw_idbits : 0u;
        p.fa.idmask = packed ? (uint32_t)((1ull << ws.cw_idbits) - 1) : 0u;
        p.fa.wmin = packed ? ws.cw_wmin : 0u;
        p.fa.qv = ws.qv.as<uint32_t>();
        p.fa.qo = ws.qo.as<uint32_t>();
        p.fa.mode = front == TIGR_FRONTIER_QUEUE ? 1 : 0;
        if (front == TIGR_FRONTIER_AUTO) p.fa.mode = dev_knob("TIGR_FQ_MODE", 0);  // 1 queue, 2 dense
        p.fa.dense_div = o.frontier_div ? o.frontier_div : 2u;
        p.fa.settled = nullptr;
        p.fa.peers = nullptr;
        p.fa.run = (uint32_t)std::max(1, dev_knob("TIGR_FQ_RUN", 2));
        // BFS / CC settled bitmap (frontier_kernel.cuh): a target whose value is final is never
        // gathered.  (SSSP / SSWP were measured slower with a bitmap settled by the frontier
        // bound: their targets are rarely final in the heavy iterations, so the bit test only
        // puts a second dependent access in front of the value gather -- DESIGN.md §5.)
        if ((algo == TIGR_BFS || algo == TIGR_CC) && dev_knob("TIGR_BFS_BITS", 1)) {
            if (!ws.settled.p) TIGR_TRY(ws.settled.alloc(sizeof(uint32_t) * ((size_t)n / 32 + 1), s));
            p.fa.settled = ws.settled.as<uint32_t>();
        }
    } else if (front == TIGR_FRONTIER_QUEUE) {
        return fail(TIGR_EUNSUPPORTED, "frontier QUEUE needs the 16-byte-chunk layout (4 | K)");
    }
    if (front == TIGR_FRONTIER_AUTO || front == TIGR_FRONTIER_QUEUE) front = TIGR_FRONTIER_DENSE;
    p.bsp = o.schedule == 1;
    p.comm = o.comm != nullptr;  // a 1-rank communicator still runs the exchange path (tests)
    p.c = o.comm;
    p.algo = algo;
    p.n = n;
    p.relax = relax_kernel(algo, vg->layout, (int)vg->unit, front, p.bsp, o.collect_stats != 0);
    if (!p.relax) return fail(TIGR_EUNSUPPORTED, "no relax kernel for this option combination");
    p.args = make_args(vg);
    if (p.comm) {
        if (o.exchange < TIGR_EXCHANGE_AUTO || o.exchange > TIGR_EXCHANGE_FUSED)
            return fail(TIGR_EINVAL, "run: unknown exchange mode");
        if (o.exchange == TIGR_EXCHANGE_FUSED) {
            if (!p.fq)
                return fail(TIGR_EUNSUPPORTED, "fused exchange needs the queue/dense frontier relax (4 | K, FRONTIER_AUTO/QUEUE)");
            const FusedPeers* fp = nullptr;
            TIGR_TRY(fused_setup(o.comm, p.args.val, p.args.stamp, p.args.ctl, ws.peers, s, &fp));
            p.fa.peers = fp;
            p.fused = true;
        }
        if (o.exchange != TIGR_EXCHANGE_DENSE && !ws.xlist.p)
            TIGR_TRY(ws.xlist.alloc(sizeof(uint2) * (n ? n : 1), s));
        p.xa = ExchangeArgs{o.comm, o.exchange, algo, n, p.args.val, (uint32_t*)p.args.prev, p.args.stamp,
                            ws.xlist.as<uint2>(), p.args.ctl};
    }
    int per_thread = 1;
    if (RelaxFn mlp = relax_mlp_kernel(algo, vg->layout, (int)vg->unit, front, p.bsp, o.collect_stats != 0, &per_thread))
        p.relax = mlp;
    else
        per_thread = 1;
    const uint64_t per_block = (uint64_t)kRelaxThreads * per_thread;
    p.grid = (unsigned)(((uint64_t)(vg->hi - vg->lo) + per_block - 1) / per_block);
    if (p.fq) p.grid = vg->hi > vg->lo ? relax_fq_grid(p.fq) : 0;  // persistent
    const uint32_t max_iters = o.max_iters ? o.max_iters : (n + 1 > n ? n + 1 : n);

    cudaEvent_t t0 = ws.ev[0], t1 = ws.ev[1];
    TIGR_CK(cudaEventRecord(t0, s));
    const tigr_graph* gg = vg->g;
    if (p.fq && p.fa.settled) TIGR_CK(cudaMemsetAsync(p.fa.settled, 0, sizeof(uint32_t) * ((size_t)n / 32 + 1), s));
    k_init<<<grid_for((n & 3u) ? n : n / 4), kBlock, 0, s>>>(algo, n, source, p.args.val, p.args.stamp, p.args.ctl, max_iters,
                                          gg->reordered ? gg->perm_cid.as<uint32_t>() : nullptr,
                                          gg->reordered ? gg->perm_order.as<uint32_t>() : nullptr,
                                          p.fq ? p.fa.settled : nullptr);
    TIGR_CKL("init");
    if (p.bsp || p.comm)
        TIGR_CK(cudaMemcpyAsync((void*)p.args.prev, p.args.val, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s));
    if (p.fq) TIGR_TRY(compact_launch(vg, p.args.ctl, 0, s));  // iteration 1's queue
    if (p.fused) TIGR_TRY(fused_barrier(p.c, s));  // every replica initialised before any remote update

    int kpi = 0;
    uint32_t launches = 0, sparse_exchanges = 0;
    double ms_relax = 0.0, ms_ex = 0.0;
    // NCCL inside a conditional body graph is not relied on: multi-GPU runs use the host loop
    const bool use_graph = o.use_graph && !o.time_kernels && !p.comm;
    if (use_graph) {
        GraphKey key{algo, vg->layout * 16 + (int)vg->unit,
                     p.fq ? 16 + p.fa.mode * 4 + (int)p.fa.dense_div * 16 + (p.fa.settled ? 1 << 30 : 0) : front,
                     p.bsp ? 1 : 0, o.collect_stats ? 1 : 0, p.comm ? 1 : 0, vg->lo, vg->hi,
                     p.fq ? (const void*)p.fq : (const void*)p.relax};
        auto itg = ws.graphs.find(key);
        if (itg == ws.graphs.end()) {
            CachedGraph cg;
            TIGR_CK(cudaStreamCreateWithFlags(&cg.stream, cudaStreamNonBlocking));
            cudaGraph_t g;
            TIGR_CK(cudaGraphCreate(&g, 0));
            cudaGraphConditionalHandle h;
            TIGR_CK(cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault));
            cudaGraphNodeParams cp = {};
            cp.type = cudaGraphNodeTypeConditional;
            cp.conditional.handle = h;
            cp.conditional.type = cudaGraphCondTypeWhile;
            cp.conditional.size = 1;
            cudaGraphNode_t node;
            TIGR_CK(cudaGraphAddNode(&node, g, nullptr, 0, &cp));
            cudaGraph_t body = cp.conditional.phGraph_out[0];
            TIGR_CK(cudaStreamBeginCaptureToGraph(cg.stream, body, nullptr, nullptr, 0,
                                                  cudaStreamCaptureModeThreadLocal));
            tigr_status bst = enqueue_body(p, cg.stream, h, 1, &cg.kernels_per_iter);
            cudaGraph_t captured = nullptr;
            cudaError_t ce = cudaStreamEndCapture(cg.stream, &captured);
            if (bst != TIGR_OK) { cudaGraphDestroy(g); return bst; }
            if (ce != cudaSuccess) { cudaGraphDestroy(g); return cuda_fail(ce, "graph capture", __FILE__, __LINE__); }
            ce = cudaGraphInstantiate(&cg.exec, g, 0);
            cudaGraphDestroy(g);
            if (ce != cudaSuccess) return cuda_fail(ce, "graph instantiate", __FILE__, __LINE__);
            itg = ws.graphs.emplace(key, cg).first;
        }
        CachedGraph& cg = itg->second;
        kpi = cg.kernels_per_iter;
        TIGR_CK(cudaEventRecord(ws.ev[2], s));
        TIGR_CK(cudaStreamWaitEvent(cg.stream, ws.ev[2], 0));
        TIGR_CK(cudaGraphLaunch(cg.exec, cg.stream));
        TIGR_CK(cudaEventRecord(ws.ev[3], cg.stream));
        TIGR_CK(cudaStreamWaitEvent(s, ws.ev[3], 0));
    } else {
        // Host loop (multi-GPU, time_kernels, use_graph = 0).  Iterations are enqueued in batches
        // and the control block is read back once per batch: every kernel of an iteration body
        // returns at once when ctl->cont is already 0, so the iterations enqueued past the fixed
        // point are no-ops (a dense exchange's all-reduce then merges identical replicas).  The
        // dense exchange decides nothing on the host, so it batches 4 iterations per round trip;
        // the sparse and fused exchanges and per-launch timing need the host every iteration.
        const bool dense_x = p.comm && !p.fused && o.exchange == TIGR_EXCHANGE_DENSE;
        const int batch = (dense_x && !o.time_kernels) ? 4 : 1;
        for (;;) {
            for (int b = 0; b < batch; ++b) {
                int k = 0;
                TIGR_TRY(enqueue_body(p, s, 0, 0, &k, o.time_kernels ? ws.ev[2] : nullptr,
                                      o.time_kernels ? ws.ev[3] : nullptr, &sparse_exchanges,
                                      o.time_kernels && p.comm ? ws.ev[4] : nullptr));
                count_launch(k);
            }
            TIGR_CK(cudaMemcpyAsync(ws.ctl_host, p.args.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
            TIGR_CK(cudaStreamSynchronize(s));
            if (o.time_kernels && p.grid) {
                float ms = 0.f;
                TIGR_CK(cudaEventElapsedTime(&ms, ws.ev[2], ws.ev[3]));
                ms_relax += ms;
                if (p.comm) {
                    TIGR_CK(cudaEventElapsedTime(&ms, ws.ev[3], ws.ev[4]));
                    ms_ex += ms;
                }
            }
            if (!ws.ctl_host->cont) break;
        }
    }
    TIGR_CK(cudaEventRecord(t1, s));
    TIGR_CK(cudaMemcpyAsync(ws.ctl_host, p.args.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    const Ctl& c = *ws.ctl_host;
    launches = p.grid ? c.it : 0;  // one relax launch per executed iteration
    if (use_graph) {
        count_launch((uint64_t)c.it * kpi);
    }
    if (st) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, t0, t1);
        st->iterations = c.it;
        st->relax_launches = launches;
        st->edges_processed = c.edges;
        st->updates = c.updates;
        st->active_vnodes = c.vnodes;
        st->ms_total = ms;
        st->ms_relax = ms_relax;
        st->queue_iterations = c.queue_iters;
        st->active_nodes = c.nodes;
        st->sparse_exchanges = sparse_exchanges;
        st->ms_exchange = ms_ex;
        st->ms_kernels = ms - ms_ex;
        // SURVEY §8(d) byte model: per processed arc s_e (+4 weight) + 4 (target
        // value), per update 4, per active virtual node 4 (vn_phys), per active node with arcs
        // 12 (value + row pair), per iteration 2 B per node (frontier flags read + cleared)
        if (o.collect_stats) {
            const uint64_t s_e = (algo == TIGR_SSSP || algo == TIGR_SSWP) ? 8 : 4;
            st->bytes_alg = c.edges * (s_e + 4) + c.updates * 4 + c.vnodes * 4 + c.nodes * 12 +
                            (uint64_t)c.it * 2 * n;
        }
    }
    if (c.notconv) return fail(TIGR_ENOTCONV, "max_iters reached before the fixed point");
    return TIGR_OK;
}

tigr_status run_pr(tigr_vgraph* vg, const tigr_run_opts& o, cudaStream_t s, tigr_stats* st) {
    Workspace& ws = vg->ws;
    const uint32_t n = vg->g->n;
    RelaxArgs a = make_args(vg);
    // preferred: the in-degree-ordered accumulator (pr.cu k_relax_pr_cid); a transposed graph
    // runs pull-based PageRank (pr.cu, NEXT-1) and divides by the original graph's
    // out-degrees, which the transpose carries; 4 ∤ K layouts and stats runs use the plain
    // one-vnode-per-thread push (relax.cu k_relax_pr)
    const bool pull = vg->g->transposed;
    if (o.pr_dangling && (vg->g->part_lo != 0 || vg->g->part_hi < n))
        return fail(TIGR_EUNSUPPORTED, "pr_dangling = 1 needs every out-degree: not on a partitioned graph");
    const uint32_t* out_deg = pull ? vg->g->src_deg.as<uint32_t>() : vg->g->deg.as<uint32_t>();
    const bool use_cid = !pull && !o.collect_stats && vg->vec;
    PrCidPlan cp;
    if (use_cid) {
        TIGR_TRY(pr_cid_prepare(vg, s));
        cp = pr_cid_plan(vg);
    }
    // fused apply (pr.cu PrFuse): the relax derives contributions from the previous accumulator;
    // two accumulators alternate; dangling-mass redistribution keeps the separate apply
    const bool fuse = use_cid && !o.pr_dangling && o.pr_iters > 0;
    if (fuse && !ws.acc2.p) TIGR_TRY(ws.acc2.alloc(sizeof(double) * (n ? n : 1), s));
    // pull: sources in out-degree order (pr.cu pr_pull_prepare)
    const bool pull_oid = pull && vg->vec;
    const uint32_t* oid = nullptr;
    if (pull_oid) {
        TIGR_TRY(pr_pull_prepare(vg, s));
        oid = ws.cid.as<uint32_t>();
        a.col = ws.col_pr.as<uint32_t>();
    }
    RelaxFn relax = nullptr;
    uint64_t per_block = kRelaxThreads;
    if (pull) {
        if (!vg->vec || o.collect_stats)
            return fail(TIGR_EUNSUPPORTED, "pull PageRank needs 4 | K and collect_stats = 0");
        int per = 1;
        relax = relax_pr_pull_kernel(vg->layout, (int)vg->unit, &per);
        per_block *= per;
    } else {
        relax = relax_kernel(TIGR_PR, vg->layout, (int)vg->unit, TIGR_FRONTIER_NONE, false, o.collect_stats != 0);
    }
    const unsigned grid = (unsigned)(((uint64_t)(vg->hi - vg->lo) + per_block - 1) / per_block);
    const bool comm = o.comm != nullptr;
    const double base = (1.0 - o.pr_damping) / (double)n;
    cudaEvent_t t0 = ws.ev[0], t1 = ws.ev[1];
    TIGR_CK(cudaEventRecord(t0, s));
    TIGR_CK(cudaMemsetAsync(a.ctl, 0, sizeof(Ctl), s));
    k_pr_init<<<grid_for(n), kBlock, 0, s>>>(n, out_deg, ws.x.as<double>(), ws.contrib.as<double>(),
                                             ws.acc.as<double>(), a.ctl, oid);
    TIGR_CKL("pr init");
    trace(s, "pr: prepare+init");
    double ms_relax = 0.0, ms_ex = 0.0;
    uint32_t launches = 0;
    if (o.time_kernels) {  // 3 events per iteration: relax start / relax end / exchange end
        while (ws.tev.size() < 3 * (size_t)o.pr_iters) {
            cudaEvent_t e;
            TIGR_CK(cudaEventCreate(&e));
            ws.tev.push_back(e);
        }
    }
    for (uint32_t t = 0; t < o.pr_iters; ++t) {
        if (o.time_kernels) TIGR_CK(cudaEventRecord(ws.tev[3 * t], s));
        double* acc_cur = ws.acc.as<double>();
        PrFuse fz;
        if (fuse) {
            acc_cur = (t & 1) ? ws.acc2.as<double>() : ws.acc.as<double>();
            fz.mode = t == 0 ? 1 : 2;
            fz.n_in = ws.n_in;
            fz.prev = (t & 1) ? ws.acc.as<double>() : ws.acc2.as<double>();
            fz.cid = ws.cid.as<uint32_t>();
            fz.base = base;
            fz.damping = o.pr_damping;
            fz.x0 = 1.0 / (double)n;
            fz.probe = dev_knob("TIGR_PR_EXP", 0);  // always 0 in shipped builds
            if (t > 0) TIGR_CK(cudaMemsetAsync(acc_cur, 0, sizeof(double) * ws.n_in, s));
            a.acc = acc_cur;
        }
        if (use_cid && cp.tiles) {
            cp.fn<<<cp.grid, cp.threads, cp.smem, s>>>(a, ws.col_pr.as<uint32_t>(), cp.tiles, fz);
            TIGR_CKL("pr relax (cid)");
            ++launches;
        } else if (grid) {
            relax<<<grid, kRelaxThreads, 0, s>>>(a);
            TIGR_CKL("pr relax");
            ++launches;
        }
        if (o.time_kernels) TIGR_CK(cudaEventRecord(ws.tev[3 * t + 1], s));
        // in accumulator-id order only the first n_in entries are ever written (pr.cu)
        if (comm) TIGR_TRY(comm_allreduce(o.comm, acc_cur, use_cid ? ws.n_in : n, TIGR_PR, s));
        if (o.time_kernels) TIGR_CK(cudaEventRecord(ws.tev[3 * t + 2], s));
        double* dcur = &a.ctl->dsum[t & 1];
        double* dnext = &a.ctl->dsum[(t + 1) & 1];
        if (o.pr_dangling) TIGR_CK(cudaMemsetAsync(dnext, 0, sizeof(double), s));
        if (fuse) {  // x itself only after the last iteration
            if (t + 1 == o.pr_iters) TIGR_TRY(pr_cid_apply(vg, base, o.pr_damping, 0, dcur, dnext, s, acc_cur, false));
            continue;
        }
        if (use_cid) {
            TIGR_TRY(pr_cid_apply(vg, base, o.pr_damping, o.pr_dangling, dcur, dnext, s));
            continue;
        }
        k_pr_apply<<<grid_for(n), kBlock, 0, s>>>(n, out_deg, base, o.pr_damping, o.pr_dangling,
                                                  ws.x.as<double>(), ws.contrib.as<double>(), ws.acc.as<double>(),
                                                  dcur, dnext, oid);
        TIGR_CKL("pr apply");
    }
    TIGR_CK(cudaEventRecord(t1, s));
    trace(s, "pr: 20 iterations");
    TIGR_CK(cudaMemcpyAsync(ws.ctl_host, a.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    if (o.time_kernels) {
        for (uint32_t t = 0; t < o.pr_iters; ++t) {
            float ms = 0.f;
            TIGR_CK(cudaEventElapsedTime(&ms, ws.tev[3 * t], ws.tev[3 * t + 1]));
            ms_relax += ms;
            TIGR_CK(cudaEventElapsedTime(&ms, ws.tev[3 * t + 1], ws.tev[3 * t + 2]));
            ms_ex += ms;
        }
    }
    if (st) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, t0, t1);
        st->iterations = o.pr_iters;
        st->relax_launches = launches;
        st->edges_processed = ws.ctl_host->edges;
        st->updates = 0;
        st->active_vnodes = ws.ctl_host->vnodes;
        st->ms_total = ms;
        st->ms_relax = ms_relax;
        st->ms_exchange = ms_ex;
        st->ms_kernels = ms - ms_ex;
        // SURVEY §8(d) byte model per relax launch: per arc 4 (target) + 16 (RED = read + write
        // of the f64 accumulator), per virtual node 4, per node with arcs its source value: 20
        // with the apply fused in (previous accumulator 8 + cid 4 + row pair 8), else 16
        // (contrib 8 + row pair 8)
        st->bytes_alg = (uint64_t)launches * (vg->m_local * 20 + (uint64_t)(vg->hi - vg->lo) * 4 + vg->n_out * (fuse ? 20 : 16));
    }
    return TIGR_OK;
}

}  // namespace

tigr_status run_device(tigr_vgraph* vg, tigr_algo algo, uint32_t source, const tigr_run_opts& o, void* out,
                       int out_is_device, tigr_stats* st) {
    const tigr_graph* g = vg->g;
    if ((int)algo < TIGR_BFS || (int)algo > TIGR_PR) return fail(TIGR_EINVAL, "run: unknown algorithm");
    if (o.frontier == TIGR_FRONTIER_QUEUE && algo == TIGR_PR)
        return fail(TIGR_EUNSUPPORTED, "run: frontier QUEUE applies to BFS/SSSP/CC/SSWP");
    if ((algo == TIGR_BFS || algo == TIGR_SSSP || algo == TIGR_SSWP) && source >= g->n)
        return fail(TIGR_EINVAL, "run: source >= n");
    if ((algo == TIGR_SSSP || algo == TIGR_SSWP) && !g->weighted)
        return fail(TIGR_EINVAL, "run: SSSP/SSWP need a weighted graph");
    if (algo == TIGR_CC && !g->symmetric)
        return fail(TIGR_EINVAL, "run: CC needs a symmetric graph (build with symmetrize=1)");
    if (algo == TIGR_PR && !(o.pr_damping >= 0.0 && o.pr_damping <= 1.0))
        return fail(TIGR_EINVAL, "run: pr_damping outside [0, 1]");
    if (o.frontier < TIGR_FRONTIER_AUTO || o.frontier > TIGR_FRONTIER_QUEUE)
        return fail(TIGR_EINVAL, "run: unknown frontier mode");
    cudaStream_t s = (cudaStream_t)o.stream;
    if (st) *st = tigr_stats{};
    if (g->n == 0) return TIGR_OK;
    TIGR_TRY(ensure_ws(vg, algo == TIGR_PR, s));
    tigr_status rs = (algo == TIGR_PR) ? run_pr(vg, o, s, st) : run_frontier(vg, algo, source, o, s, st);
    if (rs != TIGR_OK && rs != TIGR_ENOTCONV) return rs;
    const void* res = (algo == TIGR_PR) ? vg->ws.x.p : vg->ws.val.p;
    const size_t bytes = (size_t)g->n * (algo == TIGR_PR ? sizeof(double) : sizeof(uint32_t));
    if (out) {
        TmpBuf tmp;
        if (g->reordered) {  // values back to original ids
            void* dst = out;
            if (!out_is_device) {
                TIGR_TRY(tmp.alloc(bytes, s));
                dst = tmp.p;
            }
            TIGR_TRY(unpermute(g->n, g->perm_cid.as<uint32_t>(), res, dst, algo == TIGR_PR, s));
            res = dst;
        }
        if (res != out)
            TIGR_CK(cudaMemcpyAsync(out, res, bytes, out_is_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaStreamSynchronize(s));
    }
    return rs;
}

// per-vnode edge lists through the relax kernels' walk (layout parity)
tigr_status assignment_device(const tigr_vgraph* vgc, uint32_t* counts, uint32_t* nbr, uint32_t* w,
                              cudaStream_t s) {
    tigr_vgraph* vg = const_cast<tigr_vgraph*>(vgc);
    if (vg->nv == 0) return TIGR_OK;
    RelaxArgs a = make_args(vg);
    a.lo = 0;
    a.hi = (uint32_t)vg->nv;
    AssignFn f = assign_kernel(vg->layout, (int)vg->unit);
    const unsigned grid = (unsigned)((vg->nv + kRelaxThreads - 1) / kRelaxThreads);
    TmpBuf offs;
    TIGR_TRY(offs.alloc(sizeof(uint32_t) * (vg->nv + 1), s));
    f<<<grid, kRelaxThreads, 0, s>>>(a, nullptr, counts, nullptr, nullptr, vg->g->weighted, 0);
    TIGR_CKL("assign count");
    TIGR_TRY(exclusive_scan_u32(counts, vg->nv, SCAN_U32, 1, offs.as<uint32_t>(), s, nullptr));
    f<<<grid, kRelaxThreads, 0, s>>>(a, offs.as<uint32_t>(), counts, nbr, w, vg->g->weighted, 1);
    TIGR_CKL("assign fill");
    return TIGR_OK;
}

// contiguous, family-aligned vnode ranges with ~equal edge counts: rank r owns
// the vnodes of nodes [cut(r), cut(r+1)), cut(r) = first node whose arc prefix reaches r*m/P
void partition_ranges(uint32_t n, const int64_t* rp, const uint32_t* vp, int nranks, uint32_t* lo, uint32_t* hi) {
    const uint64_t m = (uint64_t)rp[n];
    auto cut = [&](int r) -> uint32_t {
        if (r <= 0) return 0;
        if (r >= nranks) return n;
        const int64_t target = (int64_t)((unsigned __int128)m * (unsigned)r / (unsigned)nranks);
        return (uint32_t)(std::lower_bound(rp, rp + n, target) - rp);
    };
    for (int r = 0; r < nranks; ++r) {
        lo[r] = vp[cut(r)];
        hi[r] = vp[cut(r + 1)];
    }
}

// the same rule on the device: one thread per cut, binary search over row_ptr (no D2H of the
// node arrays; only the 2 range bounds come back)
// nodes with out-arcs among [cuts[0], cuts[1]) (cuts on the device, from k_partition)
__global__ void k_count_out(const uint32_t* __restrict__ deg, const uint32_t* __restrict__ cuts,
                            unsigned long long* __restrict__ cnt) {
    const uint32_t lo = cuts[0], hi = cuts[1];
    uint32_t c = 0;
    for (uint32_t v = lo + blockIdx.x * blockDim.x + threadIdx.x; v < hi; v += gridDim.x * blockDim.x) c += deg[v] != 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(cnt, (unsigned long long)c);
}

__global__ void k_partition(const int64_t* __restrict__ rp, const uint32_t* __restrict__ vp, uint32_t n,
                            int nranks, int rank, uint32_t* out) {
    const int c = threadIdx.x;  // 0: cut(rank), 1: cut(rank + 1)
    if (c > 1) return;
    const int r = rank + c;
    uint32_t cut;
    if (r <= 0) cut = 0;
    else if (r >= nranks) cut = n;
    else {
        const uint64_t m = (uint64_t)rp[n];
        const int64_t target = (int64_t)((unsigned __int128)m * (unsigned)r / (unsigned)nranks);
        uint32_t lo = 0, hi = n;  // first index in [0, n) with rp[idx] >= target (lower_bound)
        while (lo < hi) {
            const uint32_t mid = lo + (hi - lo) / 2;
            if (rp[mid] < target) lo = mid + 1; else hi = mid;
        }
        cut = lo;
    }
    out[c] = vp[cut];
    out[2 + c] = cut;
}

tigr_status partition_host(tigr_vgraph* vg, int nranks, int rank) {
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(TIGR_EINVAL, "partition: bad rank/nranks");
    const tigr_graph* g = vg->g;
    cudaStream_t s = vg->vnode_ptr.s;
    TmpBuf out;
    TIGR_TRY(out.alloc(4 * sizeof(uint32_t) + sizeof(unsigned long long), s));
    unsigned long long* cnt = reinterpret_cast<unsigned long long*>(out.as<char>() + 16);
    if (nranks == 1 || g->n == 0) {
        vg->lo = 0;
        vg->hi = (uint32_t)vg->nv;
        const uint32_t full[4] = {0, (uint32_t)vg->nv, 0, g->n};
        TIGR_CK(cudaMemcpyAsync(out.p, full, sizeof(full), cudaMemcpyHostToDevice, s));
    } else {
        k_partition<<<1, 32, 0, s>>>(g->row_ptr.as<int64_t>(), vg->vnode_ptr.as<uint32_t>(), g->n, nranks, rank,
                                     out.as<uint32_t>());
        TIGR_CKL("partition");
    }
    TIGR_CK(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long), s));
    if (g->n) {
        k_count_out<<<grid_for(g->n / 8 + 1), kBlock, 0, s>>>(g->deg.as<uint32_t>(), out.as<uint32_t>() + 2, cnt);
        TIGR_CKL("partition count");
    }
    uint32_t h[4] = {0, 0, 0, 0};
    unsigned long long hn = 0;
    TIGR_CK(cudaMemcpyAsync(h, out.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaMemcpyAsync(&hn, cnt, sizeof(hn), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    vg->lo = h[0];
    vg->hi = h[1];
    vg->n_out = hn;
    // this rank's arcs: row_ptr[cut(rank + 1)] - row_ptr[cut(rank)] (the byte model's arc count)
    int64_t rp[2] = {0, 0};
    TIGR_CK(cudaMemcpyAsync(&rp[0], g->row_ptr.as<int64_t>() + h[2], sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaMemcpyAsync(&rp[1], g->row_ptr.as<int64_t>() + h[3], sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    vg->m_local = (uint64_t)(rp[1] - rp[0]);
    return TIGR_OK;
}

}  // namespace tigr
