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
#include <fcntl.h>
#include <nccl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "internal.cuh"

namespace tigr {

constexpr int kMaxGroupRanks = 16;

// ------------------------------------------------------------------------------ peer groups
// Ranks that can read each other's device memory: a published pointer of rank r becomes usable
// on every rank after the next barrier.  Two implementations: ranks as threads of one process
// (LocalGroup) and ranks as processes of one node (NodeGroup: POSIX shared memory for slots and
// barrier, CUDA IPC for the device pointers).
struct PeerGroup {
    int P = 1;
    virtual ~PeerGroup() {}
    virtual tigr_status barrier() = 0;
    virtual tigr_status publish(int me, const void* const* ptrs, int k) = 0;
    virtual tigr_status peer(int me, int r, int k, const void** out) = 0;
    virtual void publish_count(int me, uint32_t c) = 0;
    virtual uint32_t count(int r) = 0;
};

static int group_timeout_s() {
    const char* e = getenv("TIGR_GROUP_TIMEOUT");
    return e ? atoi(e) : 300;
}

struct LocalGroup : PeerGroup {
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    bool broken = false;
    std::vector<const void*> ptrk; // published pointer sets (8 per rank)
    std::vector<uint32_t> cnt;     // published counts
    std::vector<int> dev;          // device of each rank
    std::vector<char> joined;

    // all P ranks arrive before any leaves; a rank that waits longer than the timeout marks
    // the group broken (a peer failed or never called), and every later barrier fails at once
    tigr_status barrier() override {
        std::unique_lock<std::mutex> lk(mu);
        if (broken) return fail(TIGR_ENCCL, "thread-group communicator: a rank failed earlier");
        const uint64_t g = gen;
        if (++arrived == P) {
            arrived = 0;
            ++gen;
            cv.notify_all();
            return TIGR_OK;
        }
        if (!cv.wait_for(lk, std::chrono::seconds(group_timeout_s()), [&] { return gen != g || broken; }) ||
            broken) {
            broken = true;
            cv.notify_all();
            return fail(TIGR_ENCCL, "thread-group communicator: barrier timed out (a rank did not arrive)");
        }
        return TIGR_OK;
    }
    tigr_status publish(int me, const void* const* ptrs, int k) override {
        for (int i = 0; i < k; ++i) ptrk[(size_t)me * 8 + i] = ptrs[i];
        return TIGR_OK;
    }
    tigr_status peer(int, int r, int k, const void** out) override {
        for (int i = 0; i < k; ++i) out[i] = ptrk[(size_t)r * 8 + i];
        return TIGR_OK;
    }
    void publish_count(int me, uint32_t c) override { cnt[me] = c; }
    uint32_t count(int r) override { return cnt[r]; }
};

bool cache_base(const void* p, void** base, size_t* off);  // api.cu: allocation containing p

// Ranks as processes of one node.  The shared segment holds a sense-counting barrier and one
// slot per rank; device pointers travel as CUDA IPC handles of their allocation plus an offset
// and are mapped once per (rank, allocation) with cudaIpcOpenMemHandle.
struct NodeShm {
    static constexpr uint32_t kMagic = 0x54494752u;  // "TIGR"
    std::atomic<uint32_t> magic;
    uint32_t P;
    std::atomic<uint32_t> arrived, gen, broken, joined;
    struct Slot {
        int dev;
        uint32_t count;
        cudaIpcMemHandle_t h[8];
        uint64_t off[8];
    } slot[kMaxGroupRanks];
};

extern std::atomic<uint64_t> g_free_epoch;  // api.cu

struct NodeGroup : PeerGroup {
    std::string name;
    NodeShm* shm = nullptr;
    int me = 0;
    bool owner = false;
    std::vector<const void*> mine = std::vector<const void*>(8, nullptr);
    // exporter: one cudaIpcGetMemHandle per allocation (valid until libtigr frees blocks to the
    // driver, g_free_epoch); importer: mappings by handle, at most kMaxOpened, least recently
    // used closed first (a mapping of a block its owner has since freed is never reused --
    // a new allocation has a new handle -- and is closed when it ages out)
    static constexpr size_t kMaxOpened = 256;  // > 3 pointers x 15 peers of one fused run
    std::map<void*, cudaIpcMemHandle_t> exported;
    uint64_t exported_epoch = 0;
    struct Opened { void* p; uint64_t used; };
    std::map<std::string, Opened> opened;  // IPC handle bytes -> mapped base
    uint64_t clock = 0;

    ~NodeGroup() override {
        for (auto& kv : opened) cudaIpcCloseMemHandle(kv.second.p);
        if (shm) munmap(shm, sizeof(NodeShm));
        if (owner) shm_unlink(name.c_str());
    }
    tigr_status barrier() override {
        if (shm->broken.load()) return fail(TIGR_ENCCL, "node communicator: a rank failed earlier");
        const uint32_t g = shm->gen.load(std::memory_order_acquire);
        if (shm->arrived.fetch_add(1, std::memory_order_acq_rel) + 1 == (uint32_t)P) {
            shm->arrived.store(0, std::memory_order_relaxed);
            shm->gen.fetch_add(1, std::memory_order_acq_rel);
            return TIGR_OK;
        }
        const auto t0 = std::chrono::steady_clock::now();
        int spins = 0;
        while (shm->gen.load(std::memory_order_acquire) == g) {
            if (shm->broken.load()) return fail(TIGR_ENCCL, "node communicator: a rank failed earlier");
            if (++spins > 1000) {
                usleep(20);
                if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(group_timeout_s())) {
                    shm->broken.store(1);
                    return fail(TIGR_ENCCL, "node communicator: barrier timed out (a rank did not arrive)");
                }
            }
        }
        return TIGR_OK;
    }
    tigr_status publish(int r, const void* const* ptrs, int k) override {
        const uint64_t epoch = g_free_epoch.load();
        if (epoch != exported_epoch) {
            exported.clear();
            exported_epoch = epoch;
        }
        for (int i = 0; i < k; ++i) {
            mine[i] = ptrs[i];
            void* base = nullptr;
            size_t off = 0;
            if (!cache_base(ptrs[i], &base, &off))
                return fail(TIGR_EINVAL, "node communicator: buffer not allocated by libtigr");
            auto it = exported.find(base);
            if (it == exported.end()) {
                cudaIpcMemHandle_t h;
                TIGR_CK(cudaIpcGetMemHandle(&h, base));
                it = exported.emplace(base, h).first;
            }
            shm->slot[r].h[i] = it->second;
            shm->slot[r].off[i] = off;
        }
        return TIGR_OK;
    }
    tigr_status peer(int self, int r, int k, const void** out) override {
        for (int i = 0; i < k; ++i) {
            if (r == self) { out[i] = mine[i]; continue; }
            const std::string key(reinterpret_cast<const char*>(&shm->slot[r].h[i]), sizeof(cudaIpcMemHandle_t));
            auto it = opened.find(key);
            if (it == opened.end()) {
                if (opened.size() >= kMaxOpened) {  // close the least recently used mapping
                    auto lru = opened.begin();
                    for (auto j = opened.begin(); j != opened.end(); ++j)
                        if (j->second.used < lru->second.used) lru = j;
                    cudaIpcCloseMemHandle(lru->second.p);
                    opened.erase(lru);
                }
                void* p = nullptr;
                TIGR_CK(cudaIpcOpenMemHandle(&p, shm->slot[r].h[i], cudaIpcMemLazyEnablePeerAccess));
                it = opened.emplace(key, Opened{p, 0}).first;
            }
            it->second.used = ++clock;
            out[i] = static_cast<const char*>(it->second.p) + shm->slot[r].off[i];
        }
        return TIGR_OK;
    }
    void publish_count(int r, uint32_t c) override { shm->slot[r].count = c; }
    uint32_t count(int r) override { return shm->slot[r].count; }
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
constexpr int kMaxGroup = kMaxGroupRanks;
struct PeerPtrs {
    const void* p[kMaxGroup];
};

// out[i] = op over ranks 0..P-1 (in rank order, so every rank computes the same bits) of in_r[i],
// for i in [lo, hi)
template <class T, int OP>  // OP: 0 min, 1 max, 2 sum
__global__ void k_group_reduce(PeerPtrs in, int P, size_t lo, size_t hi, T* __restrict__ out) {
    for (size_t i = lo + (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < hi; i += (size_t)gridDim.x * blockDim.x) {
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

// buf[i] = src_r[i] for i in rank r's slice, every r != me (16-byte copies where aligned)
template <class T>
__global__ void k_group_gather(PeerPtrs src, int P, int me, size_t count, T* __restrict__ buf) {
    const int r = blockIdx.y;
    if (r == me) return;
    const size_t lo = count * (size_t)r / (size_t)P, hi = count * (size_t)(r + 1) / (size_t)P;
    const T* __restrict__ s = static_cast<const T*>(src.p[r]);
    for (size_t i = lo + (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < hi; i += (size_t)gridDim.x * blockDim.x)
        buf[i] = s[i];
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

tigr_status comm_init(int nranks, int rank, const uint8_t id[128], int device, tigr_comm** out) {
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(TIGR_EINVAL, "comm_init: bad rank/nranks");
    if (device >= 0) {
        int count = 0;
        TIGR_CK(cudaGetDeviceCount(&count));
        if (device >= count) return fail(TIGR_EINVAL, "comm_init: device ordinal out of range");
        TIGR_CK(cudaSetDevice(device));
    } else if (device != -1) {
        return fail(TIGR_EINVAL, "comm_init: device must be >= 0 or -1 (current)");
    }
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
    g->ptrk.assign((size_t)nranks * 8, nullptr);
    g->cnt.assign(nranks, 0);
    g->dev.assign(nranks, -1);
    g->joined.assign(nranks, 0);
    *out = new tigr_comm_group{g};
    return TIGR_OK;
}

static tigr_status enable_peers(int dev, const std::vector<int>& devs) {
    for (int d : devs) {
        if (d == dev || d < 0) continue;
        int can = 0;
        TIGR_CK(cudaDeviceCanAccessPeer(&can, dev, d));
        if (!can) return fail(TIGR_EUNSUPPORTED, "communicator: no peer access between the ranks' GPUs");
        cudaError_t e = cudaDeviceEnablePeerAccess(d, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        else TIGR_CK(e);
    }
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
    TIGR_TRY(enable_peers(dev, g.dev));
    tigr_comm* tc = new tigr_comm();
    tc->local = grp->g;
    tc->nranks = g.P;
    tc->rank = rank;
    tc->device = dev;
    *out = tc;
    return TIGR_OK;
}

void comm_group_free(tigr_comm_group* g) { delete g; }

// Node communicator: rank 0 creates the shared segment "/tigr_<name>", the others attach to it
// (waiting up to TIGR_GROUP_TIMEOUT seconds for it to appear), every rank records its device,
// and the call returns once all nranks have joined.
tigr_status comm_init_node(const char* name, int nranks, int rank, tigr_comm** out) {
    if (!name || !*name || strlen(name) > 200) return fail(TIGR_EINVAL, "comm_init_node: bad name");
    if (nranks < 1 || nranks > kMaxGroupRanks || rank < 0 || rank >= nranks)
        return fail(TIGR_EINVAL, "comm_init_node: nranks outside [1, 16] or rank outside [0, nranks)");
    int dev = 0;
    TIGR_CK(cudaGetDevice(&dev));
    auto g = std::make_shared<NodeGroup>();
    g->name = std::string("/tigr_") + name;
    g->P = nranks;
    g->me = rank;
    int fd = -1;
    if (rank == 0) {
        shm_unlink(g->name.c_str());  // a stale segment of an earlier job with this name
        fd = shm_open(g->name.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
        if (fd < 0 || ftruncate(fd, sizeof(NodeShm)) != 0) {
            if (fd >= 0) close(fd);
            return fail(TIGR_ENCCL, "comm_init_node: cannot create the shared segment");
        }
        g->owner = true;
    } else {
        const auto t0 = std::chrono::steady_clock::now();
        while ((fd = shm_open(g->name.c_str(), O_RDWR, 0600)) < 0) {
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(group_timeout_s()))
                return fail(TIGR_ENCCL, "comm_init_node: rank 0 never created the shared segment");
            usleep(1000);
        }
    }
    void* m = mmap(nullptr, sizeof(NodeShm), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (m == MAP_FAILED) return fail(TIGR_ENCCL, "comm_init_node: mmap failed");
    g->shm = static_cast<NodeShm*>(m);
    if (rank == 0) {
        g->shm->P = (uint32_t)nranks;
        g->shm->arrived.store(0);
        g->shm->gen.store(0);
        g->shm->broken.store(0);
        g->shm->joined.store(0);
        g->shm->magic.store(NodeShm::kMagic, std::memory_order_release);
    } else {
        const auto t0 = std::chrono::steady_clock::now();
        while (g->shm->magic.load(std::memory_order_acquire) != NodeShm::kMagic) {
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(group_timeout_s()))
                return fail(TIGR_ENCCL, "comm_init_node: the shared segment was never initialised");
            usleep(1000);
        }
        if (g->shm->P != (uint32_t)nranks) return fail(TIGR_EINVAL, "comm_init_node: nranks differs from rank 0's");
    }
    g->shm->slot[rank].dev = dev;
    g->shm->joined.fetch_add(1);
    TIGR_TRY(g->barrier());  // every rank's device is known after this
    std::vector<int> devs(nranks);
    for (int r = 0; r < nranks; ++r) devs[r] = g->shm->slot[r].dev;
    TIGR_TRY(enable_peers(dev, devs));
    tigr_comm* tc = new tigr_comm();
    tc->local = g;
    tc->nranks = nranks;
    tc->rank = rank;
    tc->device = dev;
    *out = tc;
    return TIGR_OK;
}

void comm_free(tigr_comm* c) {
    if (!c) return;
    if (c->nccl && g_nccl.commDestroy) g_nccl.commDestroy((ncclComm_t)c->nccl);
    delete c;
}

// ------------------------------------------------------------------------------ operations
// in-place all-reduce of a replicated array: MIN (BFS/SSSP/CC), MAX (SSWP) of uint32, SUM of
// float64 (PR).  Peer groups run it as a reduce-scatter + all-gather over peer memory (each
// rank moves ~2x its array, as a ring would): rank r reduces slice r of all replicas, in rank
// order, into its scratch (so the float64 sums are bit-identical on every rank); once every
// slice is reduced, every rank copies the other slices from their owners' scratch.
tigr_status comm_allreduce(tigr_comm* c, void* buf, size_t count, int algo, cudaStream_t s) {
    if (c->local) {
        PeerGroup& g = *c->local;
        const int P = g.P, me = c->rank;
        const size_t esz = algo == TIGR_PR ? sizeof(double) : sizeof(uint32_t);
        TIGR_TRY(scratch_bytes(c, count * esz, s));
        const void* mine[2] = {buf, c->scratch.p};
        TIGR_TRY(g.publish(me, mine, 2));
        TIGR_CK(cudaStreamSynchronize(s));
        TIGR_TRY(g.barrier());
        PeerPtrs rep{}, scr{};
        for (int r = 0; r < P; ++r) {
            const void* two[2];
            TIGR_TRY(g.peer(me, r, 2, two));
            rep.p[r] = two[0];
            scr.p[r] = two[1];
        }
        const size_t lo = count * (size_t)me / (size_t)P, hi = count * (size_t)(me + 1) / (size_t)P;
        if (hi > lo) {
            const unsigned grid = (unsigned)std::min<size_t>((hi - lo + kBlock - 1) / kBlock, 148 * 8);
            if (algo == TIGR_PR)
                k_group_reduce<double, 2><<<grid, kBlock, 0, s>>>(rep, P, lo, hi, c->scratch.as<double>());
            else if (algo == TIGR_SSWP)
                k_group_reduce<uint32_t, 1><<<grid, kBlock, 0, s>>>(rep, P, lo, hi, c->scratch.as<uint32_t>());
            else
                k_group_reduce<uint32_t, 0><<<grid, kBlock, 0, s>>>(rep, P, lo, hi, c->scratch.as<uint32_t>());
            TIGR_CKL("group reduce-scatter");
            TIGR_CK(cudaMemcpyAsync(static_cast<char*>(buf) + lo * esz, c->scratch.as<char>() + lo * esz,
                                    (hi - lo) * esz, cudaMemcpyDeviceToDevice, s));
        }
        TIGR_CK(cudaStreamSynchronize(s));
        TIGR_TRY(g.barrier());  // every slice reduced; no peer reads the replicas any more
        if (count && P > 1) {
            const dim3 grid((unsigned)std::min<size_t>((count / P + kBlock) / kBlock, 148 * 4), (unsigned)P);
            if (algo == TIGR_PR) k_group_gather<double><<<grid, kBlock, 0, s>>>(scr, P, me, count, static_cast<double*>(buf));
            else k_group_gather<uint32_t><<<grid, kBlock, 0, s>>>(scr, P, me, count, static_cast<uint32_t*>(buf));
            TIGR_CKL("group all-gather");
        }
        TIGR_CK(cudaStreamSynchronize(s));
        return g.barrier();  // no peer reads this rank's scratch any more
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
        PeerGroup& g = *c->local;
        TIGR_CK(cudaMemcpyAsync(&mine, dev_count, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaStreamSynchronize(s));
        g.publish_count(c->rank, mine);
        TIGR_TRY(g.barrier());
        for (int r = 0; r < g.P; ++r) host_counts[r] = g.count(r);
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
        PeerGroup& g = *c->local;
        TIGR_TRY(g.publish(c->rank, &mine, 1));
        TIGR_CK(cudaStreamSynchronize(s));  // the list is complete before peers read it
        TIGR_TRY(g.barrier());
        for (int r = 0; r < g.P; ++r) TIGR_TRY(g.peer(c->rank, r, 1, &ptrs[r]));
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

// every rank's set of k (<= 8) device pointers: all[r * k + i] (peer groups only)
tigr_status comm_share_ptrs(tigr_comm* c, const void* const* mine, int k, const void** all) {
    if (!c->local) return fail(TIGR_EUNSUPPORTED, "pointer exchange needs a thread-group or node communicator");
    if (k < 1 || k > 8) return fail(TIGR_EINVAL, "comm_share_ptrs: 1..8 pointers");
    PeerGroup& g = *c->local;
    TIGR_TRY(g.publish(c->rank, mine, k));
    TIGR_TRY(g.barrier());
    for (int r = 0; r < g.P; ++r) TIGR_TRY(g.peer(c->rank, r, k, all + r * k));
    return g.barrier();  // slots may be rewritten after this
}

// host barrier of a peer group after this rank's stream has drained (no-op for NCCL)
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
