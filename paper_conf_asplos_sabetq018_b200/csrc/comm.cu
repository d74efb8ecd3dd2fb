// comm.cu -- NCCL communicator for the multi-GPU mode.
//
// The paper is single-GPU; the build partitions virtual nodes by range over the GPUs of one
// box, keeps a replicated value array and reduces it every iteration with an in-place
// ncclAllReduce (MIN for BFS/SSSP/CC, MAX for SSWP, SUM of the float64 accumulator for PR)
// over NVLink 5 / NVSwitch.  libnccl is loaded lazily (dlopen) so that single-GPU use needs no
// NCCL; the torch-bundled NCCL is preferred, then the system one.
#include <dlfcn.h>
#include <nccl.h>

#include <mutex>
#include <string>

#include "internal.cuh"

namespace tigr {
namespace {

struct NcclApi {
    void* h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
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
        g_nccl.commDestroy = (decltype(g_nccl.commDestroy))dlsym(h, "ncclCommDestroy");
        g_nccl.getErrorString = (decltype(g_nccl.getErrorString))dlsym(h, "ncclGetErrorString");
        if (g_nccl.getUniqueId && g_nccl.commInitRank && g_nccl.allReduce && g_nccl.commDestroy) return;
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

}  // namespace

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
    *out = tc;
    return TIGR_OK;
}

void comm_free(tigr_comm* c) {
    if (!c) return;
    if (c->nccl && g_nccl.commDestroy) g_nccl.commDestroy((ncclComm_t)c->nccl);
    delete c;
}

// in-place all-reduce of the replicated value array
tigr_status comm_allreduce(tigr_comm* c, void* buf, size_t count, int algo, cudaStream_t s) {
    TIGR_TRY(nccl_ready());
    ncclDataType_t t = ncclUint32;
    ncclRedOp_t op = ncclMin;
    if (algo == TIGR_PR) { t = ncclFloat64; op = ncclSum; }
    else if (algo == TIGR_SSWP) op = ncclMax;
    return nccl_check(g_nccl.allReduce(buf, buf, count, t, op, (ncclComm_t)c->nccl, s), "ncclAllReduce");
}

}  // namespace tigr
