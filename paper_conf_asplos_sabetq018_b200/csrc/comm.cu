// comm.cu -- communicators for the multi-GPU mode.
//
// The paper is single-GPU; the build partitions virtual nodes by range over the GPUs of one
// box and keeps a replicated value array that the ranks merge every iteration: elementwise
// MIN (BFS/SSSP/CC), MAX (SSWP) or SUM of the float64 accumulator (PR).  Two exchange shapes
// (exchange.cu decides per iteration): the dense in-place all-reduce of the whole array, or
// the sparse one, where every rank publishes the (node, value) pairs it changed and every rank
// applies all ranks' lists.
//
// Two transports, same operations:
//   * NCCL (one process per GPU, bootstrap over torch.distributed): ncclAllReduce for the
//     dense exchange; ncclAllGather of the list sizes and one grouped ncclBroadcast per rank
//     for the lists.  libnccl is loaded lazily (dlopen) so that single-GPU use needs no NCCL.
//   * thread group (ranks are threads of ONE process, on one GPU or several): a rank publishes
//     the device pointer of its buffer, a host barrier orders the ranks, and the exchange
//     kernels read the peers' buffers directly (same device, or NVLink peer access enabled at
//     init).  This is also what lets the multi-rank protocol run on a single GPU.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <mutex>
#include <string>
#include <vector>

#include "internal.cuh"

namespace tigr {

// ------------------------------------------------------------------------------ thread group
struct LocalGroup {
    int P = 1;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    bool broken = false;
    std::vector<const void*> ptr;  // published device pointers (one per rank)
    std::vector<const void*> ptrk; // published pointer sets (kMaxSet per rank)
    std::vector<uint32_t> cnt;     // published counts
    std::vector<int> dev;          // device of each rank
    std::vector<char> joined;

    // all P ranks arrive before any leaves; a rank that waits longer than the timeout marks
    // the group broken (a peer failed or never called), and every later barrier fails at once
    tigr_status barrier() {
        std::unique_lock<std::mutex> lk(mu);
        if (broken) return fail(TIGR_ENCCL, "thread-group communicator: a rank failed earlier");
        const uint64_t g = gen;
        if (++arrived == P) {
            arrived = 0;
            ++gen;
            cv.notify_all();
            return TIGR_OK;
        }
        const int secs = getenv("TIGR_GROUP_TIMEOUT") ? atoi(getenv("TIGR_GROUP_TIMEOUT")) : 300;
        if (!cv.wait_for(lk, std::chrono::seconds(secs), [&] { return gen != g || broken; }) || broken) {
            broken = true;
            cv.notify_all();
            return fail(TIGR_ENCCL, "thread-group communicator: barrier timed out (a rank did not arrive)");
        }
        return TIGR_OK;
    }
};

namespace {

// ------------------------------------------------------------------------------ NCCL loader
struct NcclApi {
    void* h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*allGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*groupStart)() = nullptr;
    ncclResult_t (*groupEnd)() = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    const char* (*getErrorString)(ncclResult_t) = nullptr;
};

NcclApi g_nccl;
std::once_flag g_nccl_once;

void load_nccl() {
    const char* cands[] = {
        getenv("TIGR_NCCL_LIB"),
        "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/lib/libnccl.so.2",
        "libnccl.so.2",
        "libnccl.so",
    };
    for (const char* c : cands) {
        if (!c || !*c) continue;
        void* h = dlopen(c, RTLD_NOW | RTLD_GLOBAL);
        if (!h) continue;
        g_nccl.h = h;
        g_nccl.getUniqueId = (decltype(g_nccl.getUniqueId))dlsym(h, "ncclGetUniqueId");
        g_nccl.commInitRank = (decltype(g_nccl.commInitRank))dlsym(h, "ncclCommInitRank");
        g_nccl.allReduce = (decltype(g_nccl.allReduce))dlsym(h, "ncclAllReduce");
        g_nccl.allGather = (decltype(g_nccl.allGather))dlsym(h, "ncclAllGather");
        g_nccl.broadcast = (decltype(g_nccl.broadcast))dlsym(h, "ncclBroadcast");
        g_nccl.groupStart = (decltype(g_nccl.groupStart))dlsym(h, "ncclGroupStart");
        g_nccl.groupEnd = (decltype(g_nccl.groupEnd))dlsym(h, "ncclGroupEnd");
        g_nccl.commDestroy = (decltype(g_nccl.commDestroy))dlsym(h, "ncclCommDestroy");
        g_nccl.getErrorString = (decltype(g_nccl.getErrorString))dlsym(h, "ncclGetErrorString");
        if (g_nccl.getUniqueId && g_nccl.commInitRank && g_nccl.allReduce && g_nccl.allGather && g_nccl.broadcast &&
            g_nccl.groupStart && g_nccl.groupEnd && g_nccl.commDestroy)
            return;
        dlclose(h);
        g_nccl = NcclApi();
    }
}

tigr_status nccl_ready() {
    std::call_once(g_nccl_once, load_nccl);
    if (!g_nccl.h) return fail(TIGR_ENCCL, "libnccl.so.2 could not be loaded (set TIGR_NCCL_LIB)");
    return TIGR_OK;
}

tigr_status nccl_check(ncclResult_t r, const char* what) {
    if (r == ncclSuccess) return TIGR_OK;
    std::string msg = std::string(what) + ": " + (g_nccl.getErrorString ? g_nccl.getErrorString(r) : "nccl error");
    return fail(TIGR_ENCCL, msg);
}

// ------------------------------------------------------------------------------ group kernels
constexpr int kMaxGroup = 16;
struct PeerPtrs {
    const void* p[kMaxGroup];
};

// out[i] = op over ranks 0..P-1 (in rank order, so every rank computes the same bits) of in_r[i]
template <class T, int OP>  // OP: 0 min, 1 max, 2 sum
__global__ void k_group_reduce(PeerPtrs in, int P, size_t count, T* __restrict__ out) {
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
        T v = static_cast<const T*>(in.p[0])[i];
        for (int r = 1; r < P; ++r) {
            const T x = static_cast<const T*>(in.p[r])[i];
            if (OP == 0) v = x < v ? x : v;
            else if (OP == 1) v = x > v ? x : v;
            else v = v + x;
        }
        out[i] = v;
    }
}

tigr_status scratch_bytes(tigr_comm* c, size_t bytes, cudaStream_t s) {
    if (c->scratch.bytes >= bytes && c->scratch.p) return TIGR_OK;
    return c->scratch.alloc(bytes + bytes / 4 + 1024, s);
}

}  // namespace

// ------------------------------------------------------------------------------ setup
tigr_status comm_unique_id(uint8_t id[128]) {
    TIGR_TRY(nccl_ready());
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    ncclUniqueId u;
    TIGR_TRY(nccl_check(g_nccl.getUniqueId(&u), "ncclGetUniqueId"));
    memcpy(id, &u, 128);
    return TIGR_OK;
}

tigr_status comm_init(int nranks, int rank, const uint8_t id[128], tigr_comm** out) {
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(TIGR_EINVAL, "comm_init: bad rank/nranks");
    TIGR_TRY(nccl_ready());
    ncclUniqueId u;
    memcpy(&u, id, 128);
    ncclComm_t c = nullptr;
    TIGR_TRY(nccl_check(g_nccl.commInitRank(&c, nranks, u, rank), "ncclCommInitRank"));
    tigr_comm* tc = new tigr_comm();
    tc->nccl = c;
    tc->nranks = nranks;
    tc->rank = rank;
    cudaGetDevice(&tc->device);
    *out = tc;
    return TIGR_OK;
}

tigr_status comm_group_create(int nranks, tigr_comm_group** out) {
    if (nranks < 1 || nranks > kMaxGroup) return fail(TIGR_EINVAL, "comm_group_create: nranks outside [1, 16]");
    auto g = std::make_shared<LocalGroup>();
    g->P = nranks;
    g->ptr.assign(nranks, nullptr);
    g->ptrk.assign((size_t)nranks * 8, nullptr);
    g->cnt.assign(nranks, 0);
    g->dev.assign(nranks, -1);
    g->joined.assign(nranks, 0);
    *out = new tigr_comm_group{g};
    return TIGR_OK;
}

tigr_status comm_init_group(tigr_comm_group* grp, int rank, tigr_comm** out) {
    LocalGroup& g = *grp->g;
    if (rank < 0 || rank >= g.P) return fail(TIGR_EINVAL, "comm_init_group: rank outside [0, nranks)");
    int dev = 0;
    TIGR_CK(cudaGetDevice(&dev));
    {
        std::lock_guard<std::mutex> lk(g.mu);
        if (g.joined[rank]) return fail(TIGR_EINVAL, "comm_init_group: rank already joined");
        g.joined[rank] = 1;
        g.dev[rank] = dev;
    }
    TIGR_TRY(g.barrier());  // every rank's device is known after this
    for (int r = 0; r < g.P; ++r) {
        if (g.dev[r] == dev) continue;
        int can = 0;
        TIGR_CK(cudaDeviceCanAccessPeer(&can, dev, g.dev[r]));
        if (!can) return fail(TIGR_EUNSUPPORTED, "comm_init_group: no peer access between the ranks' GPUs");
        cudaError_t e = cudaDeviceEnablePeerAccess(g.dev[r], 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        else TIGR_CK(e);
    }
    tigr_comm* tc = new tigr_comm();
    tc->local = grp->g;
    tc->nranks = g.P;
    tc->rank = rank;
    tc->device = dev;
    *out = tc;
    return TIGR_OK;
}

void comm_group_free(tigr_comm_group* g) { delete g; }

void comm_free(tigr_comm* c) {
    if (!c) return;
    if (c->nccl && g_nccl.commDestroy) g_nccl.commDestroy((ncclComm_t)c->nccl);
    delete c;
}

// ------------------------------------------------------------------------------ operations
// in-place all-reduce of a replicated array: MIN (BFS/SSSP/CC), MAX (SSWP) of uint32, SUM of
// float64 (PR).  Thread group: every rank reduces all replicas in rank order into scratch (so
// the float64 sums are bit-identical on every rank), then, once no peer still reads, copies back.
tigr_status comm_allreduce(tigr_comm* c, void* buf, size_t count, int algo, cudaStream_t s) {
    if (c->local) {
        LocalGroup& g = *c->local;
        const size_t esz = algo == TIGR_PR ? sizeof(double) : sizeof(uint32_t);
        TIGR_TRY(scratch_bytes(c, count * esz, s));
        g.ptr[c->rank] = buf;
        TIGR_CK(cudaStreamSynchronize(s));
        TIGR_TRY(g.barrier());
        PeerPtrs pp{};
        for (int r = 0; r < g.P; ++r) pp.p[r] = g.ptr[r];
        if (count) {
            const unsigned grid = (unsigned)std::min<size_t>((count + kBlock - 1) / kBlock, 148 * 8);
            if (algo == TIGR_PR)
                k_group_reduce<double, 2><<<grid, kBlock, 0, s>>>(pp, g.P, count, c->scratch.as<double>());
            else if (algo == TIGR_SSWP)
                k_group_reduce<uint32_t, 1><<<grid, kBlock, 0, s>>>(pp, g.P, count, c->scratch.as<uint32_t>());
            else
                k_group_reduce<uint32_t, 0><<<grid, kBlock, 0, s>>>(pp, g.P, count, c->scratch.as<uint32_t>());
            TIGR_CKL("group all-reduce");
        }
        TIGR_CK(cudaStreamSynchronize(s));
        TIGR_TRY(g.barrier());  // every peer has finished reading this rank's buffer
        if (count) TIGR_CK(cudaMemcpyAsync(buf, c->scratch.p, count * esz, cudaMemcpyDeviceToDevice, s));
        return TIGR_OK;
    }
    TIGR_TRY(nccl_ready());
    ncclDataType_t t = ncclUint32;
    ncclRedOp_t op = ncclMin;
    if (algo == TIGR_PR) { t = ncclFloat64; op = ncclSum; }
    else if (algo == TIGR_SSWP) op = ncclMax;
    return nccl_check(g_nccl.allReduce(buf, buf, count, t, op, (ncclComm_t)c->nccl, s), "ncclAllReduce");
}

// every rank's list length: host_counts[r] for r < nranks (synchronises s)
tigr_status comm_allgather_count(tigr_comm* c, const uint32_t* dev_count, uint32_t* host_counts, cudaStream_t s) {
    uint32_t mine = 0;
    if (c->local) {
        LocalGroup& g = *c->local;
        TIGR_CK(cudaMemcpyAsync(&mine, dev_count, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaStreamSynchronize(s));
        g.cnt[c->rank] = mine;
        TIGR_TRY(g.barrier());
        for (int r = 0; r < g.P; ++r) host_counts[r] = g.cnt[r];
        TIGR_TRY(g.barrier());  // slots may be rewritten after this
        return TIGR_OK;
    }
    TIGR_TRY(nccl_ready());
    if (!c->counts.p) TIGR_TRY(c->counts.alloc(sizeof(uint32_t) * c->nranks, s));
    TIGR_TRY(nccl_check(g_nccl.allGather(dev_count, c->counts.p, 1, ncclUint32, (ncclComm_t)c->nccl, s),
                        "ncclAllGather"));
    TIGR_CK(cudaMemcpyAsync(host_counts, c->counts.p, sizeof(uint32_t) * c->nranks, cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

// make every rank's list of 8-byte records readable on this rank: ptrs[r] (device pointers,
// valid on s until comm_release_lists).  NCCL: one grouped broadcast per rank into scratch.
tigr_status comm_share_lists(tigr_comm* c, const void* mine, const uint32_t* counts, const void** ptrs,
                             cudaStream_t s) {
    if (c->local) {
        LocalGroup& g = *c->local;
        g.ptr[c->rank] = mine;
        TIGR_CK(cudaStreamSynchronize(s));  // the list is complete before peers read it
        TIGR_TRY(g.barrier());
        for (int r = 0; r < g.P; ++r) ptrs[r] = g.ptr[r];
        return TIGR_OK;
    }
    TIGR_TRY(nccl_ready());
    size_t total = 0;
    for (int r = 0; r < c->nranks; ++r) total += counts[r];
    TIGR_TRY(scratch_bytes(c, total * 8, s));
    size_t off = 0;
    TIGR_TRY(nccl_check(g_nccl.groupStart(), "ncclGroupStart"));
    for (int r = 0; r < c->nranks; ++r) {
        char* dst = c->scratch.as<char>() + off * 8;
        ptrs[r] = dst;
        if (counts[r]) {
            ncclResult_t e = g_nccl.broadcast(r == c->rank ? mine : nullptr, dst, counts[r], ncclUint64, r,
                                              (ncclComm_t)c->nccl, s);
            if (e != ncclSuccess) { g_nccl.groupEnd(); return nccl_check(e, "ncclBroadcast"); }
        }
        off += counts[r];
    }
    return nccl_check(g_nccl.groupEnd(), "ncclGroupEnd");
}

// every rank's set of k (<= 8) device pointers: all[r * k + i] (thread group only)
tigr_status comm_share_ptrs(tigr_comm* c, const void* const* mine, int k, const void** all) {
    if (!c->local) return fail(TIGR_EUNSUPPORTED, "pointer exchange needs the thread-group communicator");
    if (k < 1 || k > 8) return fail(TIGR_EINVAL, "comm_share_ptrs: 1..8 pointers");
    LocalGroup& g = *c->local;
    for (int i = 0; i < k; ++i) g.ptrk[(size_t)c->rank * 8 + i] = mine[i];
    TIGR_TRY(g.barrier());
    for (int r = 0; r < g.P; ++r)
        for (int i = 0; i < k; ++i) all[r * k + i] = g.ptrk[(size_t)r * 8 + i];
    return g.barrier();  // slots may be rewritten after this
}

// host barrier of the thread group after this rank's stream has drained (no-op for NCCL)
tigr_status comm_sync_barrier(tigr_comm* c, cudaStream_t s) {
    if (!c->local) return TIGR_OK;
    TIGR_CK(cudaStreamSynchronize(s));
    return c->local->barrier();
}

// the lists shared by comm_share_lists are no longer read by this rank's stream
tigr_status comm_release_lists(tigr_comm* c, cudaStream_t s) {
    if (!c->local) return TIGR_OK;
    TIGR_CK(cudaStreamSynchronize(s));
    return c->local->barrier();
}

}  // namespace tigr
