// api.cu -- the extern "C" boundary of libtigr.so (include/tigr.h).  Argument checking,
// host<->device staging, error state; every compute step runs in the kernels of the other
// translation units.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <mutex>
#include <cstring>
#include <string>

#include "internal.cuh"
#include "vgraph.cuh"

namespace tigr {

std::atomic<uint64_t> g_launches{0};
static thread_local std::string t_err;

void set_error(const std::string& msg) { t_err = msg; }

void trace(cudaStream_t s, const char* what) {
    static const bool on = getenv("TIGR_TRACE") != nullptr;
    if (!on) return;
    static thread_local std::chrono::steady_clock::time_point last = std::chrono::steady_clock::now();
    cudaStreamSynchronize(s);
    const auto now = std::chrono::steady_clock::now();
    int dev = 0;
    cudaGetDevice(&dev);
    cudaMemPool_t pool;
    uint64_t reserved = 0, used = 0;
    if (cudaDeviceGetMemPool(&pool, dev) == cudaSuccess) {
        cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &reserved);
        cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &used);
    }
    fprintf(stderr, "[tigr trace] %-28s %9.3f ms  (pool reserved %.2f GB, used %.2f GB)\n", what,
            std::chrono::duration<double, std::milli>(now - last).count(), reserved / 1e9, used / 1e9);
    last = now;
}

int dev_knob(const char* name, int dflt) {
#ifdef TIGR_DEV_KNOBS
    const char* e = getenv(name);
    return e ? atoi(e) : dflt;
#else
    (void)name;
    return dflt;
#endif
}

tigr_status fail(tigr_status st, const std::string& msg) {
    t_err = msg;
    return st;
}

tigr_status cuda_fail(cudaError_t e, const char* what, const char* file, int line) {
    char buf[512];
    snprintf(buf, sizeof(buf), "%s: %s (%s) at %s:%d", what, cudaGetErrorName(e), cudaGetErrorString(e), file, line);
    t_err = buf;
    return (e == cudaErrorMemoryAllocation) ? TIGR_ENOMEM : TIGR_ECUDA;
}

// ---- caching device allocator ------------------------------------------------------------
// cudaMallocAsync of multi-GB blocks measured 15-100 ms on B200 even with a raised pool
// release threshold, and a graph build allocates ~6 GB of sort buffers; so libtigr keeps its
// own cache of cudaMalloc'ed blocks (2 MiB granularity, best fit within +25%).  A freed block
// records an event on the stream that last used it; reuse from another stream waits on it.
namespace {
// Blocks are keyed by device as well as size: one process may drive several GPUs (the
// thread-group communicator, comm.cu), and a block must only be reused on the device it lives on.
struct CachedBlock {
    void* p;
    size_t size;
    cudaStream_t s;
    cudaEvent_t ev;
    int dev;
};
std::mutex g_cache_mu;
std::multimap<std::pair<int, size_t>, CachedBlock> g_free;  // (device, size) -> block
std::map<void*, std::pair<int, size_t>> g_live;             // live block -> (device, size)
constexpr size_t kGran = 2u << 20;
}  // namespace

// incremented whenever libtigr returns cached blocks to the driver: an address published before
// may then name a different allocation
std::atomic<uint64_t> g_free_epoch{0};

namespace {

void release_cached_locked() {
    g_free_epoch.fetch_add(1);  // device addresses may be handed out again (comm.cu IPC handle cache)
    int cur = 0;
    cudaGetDevice(&cur);
    for (auto& kv : g_free) {
        cudaSetDevice(kv.second.dev);
        cudaFree(kv.second.p);
        if (kv.second.ev) cudaEventDestroy(kv.second.ev);
    }
    cudaSetDevice(cur);
    g_free.clear();
}
}  // namespace

void init_pool() {}

void* cache_alloc(size_t nbytes, cudaStream_t s, cudaError_t* err) {
    const size_t size = ((nbytes ? nbytes : 1) + kGran - 1) / kGran * kGran;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_free.lower_bound({dev, size});
    if (it != g_free.end() && it->first.first == dev && it->first.second <= size + size / 4 + kGran) {
        CachedBlock b = it->second;
        g_free.erase(it);
        if (b.s != s && b.ev) cudaStreamWaitEvent(s, b.ev, 0);
        if (b.ev) cudaEventDestroy(b.ev);
        g_live[b.p] = {dev, b.size};
        *err = cudaSuccess;
        return b.p;
    }
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, size);
    if (e != cudaSuccess) {  // give the cache back to the driver and retry once
        cudaGetLastError();
        cudaDeviceSynchronize();
        release_cached_locked();
        e = cudaMalloc(&p, size);
    }
    *err = e;
    if (e != cudaSuccess) return nullptr;
    g_live[p] = {dev, size};
    return p;
}

void cache_free(void* p, cudaStream_t s) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_live.find(p);
    if (it == g_live.end()) return;
    CachedBlock b{p, it->second.second, s, nullptr, it->second.first};
    g_live.erase(it);
    if (cudaEventCreateWithFlags(&b.ev, cudaEventDisableTiming) == cudaSuccess) cudaEventRecord(b.ev, s);
    else b.ev = nullptr;
    g_free.emplace(std::make_pair(b.dev, b.size), b);
}

// the live libtigr allocation containing p: its base and p's offset in it (CUDA IPC exports
// whole allocations)
bool cache_base(const void* p, void** base, size_t* off) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_live.upper_bound(const_cast<void*>(p));
    if (it == g_live.begin()) return false;
    --it;
    const char* b = static_cast<const char*>(it->first);
    const char* q = static_cast<const char*>(p);
    if (q < b || q >= b + it->second.second) return false;
    *base = it->first;
    *off = (size_t)(q - b);
    return true;
}

void cache_release_all() {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    cudaDeviceSynchronize();
    release_cached_locked();
}

tigr_status DevBuf::alloc(size_t nbytes, cudaStream_t stream) {
    release();
    s = stream;
    cudaError_t e = cudaSuccess;
    p = cache_alloc(nbytes, stream, &e);
    if (!p) return cuda_fail(e, "cudaMalloc", __FILE__, __LINE__);
    bytes = nbytes;
    return TIGR_OK;
}

void DevBuf::release() {
    if (p) cache_free(p, s);
    p = nullptr;
    bytes = 0;
}

tigr_status TmpBuf::alloc(size_t nbytes, cudaStream_t stream) {
    s = stream;
    cudaError_t e = cudaSuccess;
    p = cache_alloc(nbytes, stream, &e);
    if (!p) return cuda_fail(e, "cudaMalloc", __FILE__, __LINE__);
    return TIGR_OK;
}

TmpBuf::~TmpBuf() {
    if (p) cache_free(p, s);
}

// other translation units
tigr_status rmat_range(uint32_t n, uint64_t e0, uint64_t count, double a, double b, double c, uint64_t seed,
                       uint64_t wseed, uint32_t wmin, uint32_t wmax, uint32_t* src, uint32_t* dst, uint32_t* w,
                       cudaStream_t s);
tigr_status graph_from_coo_device(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                  const uint32_t* w, int symmetrize, cudaStream_t s, tigr_graph** out);
tigr_status graph_from_coo_part_device(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                       const uint32_t* w, int symmetrize, uint32_t src_lo, uint32_t src_hi,
                                       cudaStream_t s, tigr_graph** out, const HostArcs* host);
tigr_status coo_source_cuts(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, int symmetrize,
                            int nranks, cudaStream_t s, uint32_t* cuts);
tigr_status graph_from_csr_device(uint32_t n, uint64_t m, const int64_t* rp, const uint32_t* col, const uint32_t* w,
                                  int symmetric_hint, cudaStream_t s, tigr_graph** out);
tigr_status graph_export_csr_device(const tigr_graph* g, int64_t* rp, uint32_t* col, uint32_t* w, cudaStream_t s);
tigr_status expand_arcs(const tigr_graph* g, uint32_t* src, uint32_t* dst, uint32_t* w, cudaStream_t s);
tigr_status graph_transpose_device(const tigr_graph* g, cudaStream_t s, tigr_graph** out);
tigr_status graph_reorder_device(const tigr_graph* g, cudaStream_t s, tigr_graph** out);
tigr_status graph_udt_device(const tigr_graph* g, uint32_t K, uint32_t dumb, uint32_t unit, cudaStream_t s,
                             tigr_graph** out);
tigr_status graph_rmat_device(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed, uint64_t wseed,
                              uint32_t wmin, uint32_t wmax, int weighted, int symmetrize, cudaStream_t s,
                              tigr_graph** out);
tigr_status virtualize_device(const tigr_graph* g, uint32_t K, tigr_layout layout, cudaStream_t s, tigr_vgraph** out);
tigr_status run_device(tigr_vgraph* vg, tigr_algo algo, uint32_t source, const tigr_run_opts& o, void* out,
                       int out_is_device, tigr_stats* st);
tigr_status assignment_device(const tigr_vgraph* vg, uint32_t* counts, uint32_t* nbr, uint32_t* w, cudaStream_t s);
tigr_status partition_host(tigr_vgraph* vg, int nranks, int rank);
void partition_ranges(uint32_t n, const int64_t* rp, const uint32_t* vp, int nranks, uint32_t* lo, uint32_t* hi);
tigr_status comm_unique_id(uint8_t id[128]);
tigr_status comm_init(int nranks, int rank, const uint8_t id[128], int device, tigr_comm** out);
void comm_free(tigr_comm* c);
tigr_status comm_group_create(int nranks, tigr_comm_group** out);
tigr_status comm_init_node(const char* name, int nranks, int rank, tigr_comm** out);
tigr_status comm_init_group(tigr_comm_group* g, int rank, tigr_comm** out);
void comm_group_free(tigr_comm_group* g);

namespace {

tigr_status need_device() {
    int count = 0;
    cudaError_t e = cudaGetDeviceCount(&count);
    if (e != cudaSuccess || count == 0)
        return fail(TIGR_ECUDA, std::string("no CUDA device available (libtigr has no CPU fallback): ") +
                                    cudaGetErrorString(e));
    return TIGR_OK;
}

// stage a host array into a temporary device buffer (or pass a device pointer through)
template <class T>
tigr_status stage(const T* p, uint64_t count, int is_device, cudaStream_t s, TmpBuf& tmp, const T** out) {
    if (!p || is_device) { *out = p; return TIGR_OK; }
    TIGR_TRY(tmp.alloc(sizeof(T) * (count ? count : 1), s));
    if (count) TIGR_CK(cudaMemcpyAsync(tmp.p, p, sizeof(T) * count, cudaMemcpyHostToDevice, s));
    *out = tmp.as<T>();
    return TIGR_OK;
}

}  // namespace
}  // namespace tigr

using namespace tigr;

extern "C" {

void tigr_run_opts_default(tigr_run_opts* o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->max_iters = 0;
    o->pr_iters = 20;
    o->pr_damping = 0.85;
    o->pr_dangling = 0;
    o->schedule = 0;
    o->frontier = TIGR_FRONTIER_AUTO;
    o->use_graph = 1;
    o->exchange = TIGR_EXCHANGE_AUTO;
}

}  // extern "C"

namespace tigr {
namespace {
// the arc-list builds: device arrays are used in place; host arrays get device buffers that the
// build fills chunk by chunk, overlapping the PCIe copies with its arc-list scan (sort.cu)
tigr_status coo_build(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                      int is_device_ptr, int symmetrize, uint32_t lo, uint32_t hi, cudaStream_t s, tigr_graph** out) {
    if (is_device_ptr || m == 0)
        return graph_from_coo_part_device(n, m, src, dst, w, symmetrize, lo, hi, s, out, nullptr);
    TmpBuf ts, td, tw;
    TIGR_TRY(ts.alloc(sizeof(uint32_t) * m, s));
    TIGR_TRY(td.alloc(sizeof(uint32_t) * m, s));
    if (w) TIGR_TRY(tw.alloc(sizeof(uint32_t) * m, s));
    const HostArcs host{src, dst, w};
    return graph_from_coo_part_device(n, m, ts.as<uint32_t>(), td.as<uint32_t>(), w ? tw.as<uint32_t>() : nullptr,
                                      symmetrize, lo, hi, s, out, &host);
}
}  // namespace
}  // namespace tigr

extern "C" {

tigr_status tigr_graph_from_coo(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                                int is_device_ptr, int symmetrize, void* stream, tigr_graph** out) {
    if (!out) return fail(TIGR_EINVAL, "graph_from_coo: out is NULL");
    *out = nullptr;
    if (n == 0) return fail(TIGR_EINVAL, "graph_from_coo: n == 0");
    if (n > 0xFFFFFFFEu) return fail(TIGR_ERANGE, "graph_from_coo: n > 0xFFFFFFFE");
    if (m && (!src || !dst)) return fail(TIGR_EINVAL, "graph_from_coo: src/dst NULL");
    TIGR_TRY(need_device());
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(coo_build(n, m, src, dst, w, is_device_ptr, symmetrize, 0, 0xFFFFFFFFu, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    trace(s, "coo: done");
    return TIGR_OK;
}

tigr_status tigr_graph_from_coo_part(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                     const uint32_t* w, int is_device_ptr, int symmetrize, uint32_t src_lo,
                                     uint32_t src_hi, void* stream, tigr_graph** out) {
    if (!out) return fail(TIGR_EINVAL, "graph_from_coo_part: out is NULL");
    *out = nullptr;
    if (n == 0) return fail(TIGR_EINVAL, "graph_from_coo_part: n == 0");
    if (n > 0xFFFFFFFEu) return fail(TIGR_ERANGE, "graph_from_coo_part: n > 0xFFFFFFFE");
    if (m && (!src || !dst)) return fail(TIGR_EINVAL, "graph_from_coo_part: src/dst NULL");
    if (src_lo > src_hi) return fail(TIGR_EINVAL, "graph_from_coo_part: src_lo > src_hi");
    TIGR_TRY(need_device());
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(coo_build(n, m, src, dst, w, is_device_ptr, symmetrize, src_lo, src_hi, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_coo_source_cuts(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, int is_device_ptr,
                                 int symmetrize, int nranks, void* stream, uint32_t* cuts) {
    if (!cuts || nranks < 1 || n == 0) return fail(TIGR_EINVAL, "coo_source_cuts: bad argument");
    if (m && (!src || !dst)) return fail(TIGR_EINVAL, "coo_source_cuts: src/dst NULL");
    TIGR_TRY(need_device());
    cudaStream_t s = (cudaStream_t)stream;
    TmpBuf ts, td;
    const uint32_t *ds = nullptr, *dd = nullptr;
    TIGR_TRY(stage(src, m, is_device_ptr, s, ts, &ds));
    TIGR_TRY(stage(dst, m, is_device_ptr, s, td, &dd));
    return coo_source_cuts(n, m, ds, dd, symmetrize, nranks, s, cuts);
}

tigr_status tigr_graph_from_csr(uint32_t n, uint64_t m, const int64_t* row_ptr, const uint32_t* col, const uint32_t* w,
                                int is_device_ptr, int symmetric_hint, void* stream, tigr_graph** out) {
    if (!out) return fail(TIGR_EINVAL, "graph_from_csr: out is NULL");
    *out = nullptr;
    if (n == 0) return fail(TIGR_EINVAL, "graph_from_csr: n == 0");
    if (n > 0xFFFFFFFEu) return fail(TIGR_ERANGE, "graph_from_csr: n > 0xFFFFFFFE");
    if (!row_ptr || (m && !col)) return fail(TIGR_EINVAL, "graph_from_csr: NULL array");
    TIGR_TRY(need_device());
    cudaStream_t s = (cudaStream_t)stream;
    TmpBuf tr, tc, tw;
    const int64_t* dr = nullptr;
    const uint32_t *dc = nullptr, *dw = nullptr;
    TIGR_TRY(stage(row_ptr, (uint64_t)n + 1, is_device_ptr, s, tr, &dr));
    TIGR_TRY(stage(col, m, is_device_ptr, s, tc, &dc));
    TIGR_TRY(stage(w, m, is_device_ptr, s, tw, &dw));
    TIGR_TRY(graph_from_csr_device(n, m, dr, dc, dw, symmetric_hint, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_rmat_coo(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed, uint64_t wseed,
                          uint32_t wmin, uint32_t wmax, uint32_t* src, uint32_t* dst, uint32_t* w, void* stream) {
    if (m && (!src || !dst)) return fail(TIGR_EINVAL, "rmat_coo: src/dst NULL");
    TIGR_TRY(need_device());
    return rmat_range(n, 0, m, a, b, c, seed, wseed, wmin, wmax, src, dst, w, (cudaStream_t)stream);
}

tigr_status tigr_graph_rmat(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed, uint64_t wseed,
                            uint32_t wmin, uint32_t wmax, int weighted, int symmetrize, void* stream,
                            tigr_graph** out) {
    if (!out) return fail(TIGR_EINVAL, "graph_rmat: out is NULL");
    *out = nullptr;
    TIGR_TRY(need_device());
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(graph_rmat_device(n, m, a, b, c, seed, wseed, wmin, wmax, weighted, symmetrize, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_graph_info(const tigr_graph* g, uint32_t* n, uint64_t* m, int* weighted, int* symmetric,
                            int* transposed, uint64_t* device_bytes) {
    if (!g) return fail(TIGR_EINVAL, "graph_info: NULL graph");
    if (n) *n = g->n;
    if (m) *m = g->m;
    if (weighted) *weighted = g->weighted;
    if (symmetric) *symmetric = g->symmetric;
    if (transposed) *transposed = g->transposed;
    if (device_bytes) *device_bytes = g->row_ptr.bytes + g->deg.bytes + g->cptr.bytes + g->col.bytes + g->wt.bytes;
    return TIGR_OK;
}

tigr_status tigr_graph_export_coo(const tigr_graph* g, uint32_t* src, uint32_t* dst, uint32_t* w,
                                  int is_device_ptr, void* stream) {
    if (!g) return fail(TIGR_EINVAL, "graph_export_coo: NULL graph");
    cudaStream_t s = (cudaStream_t)stream;
    const size_t bytes = sizeof(uint32_t) * (g->m ? g->m : 1);
    TmpBuf ds, dd, dw;  // the expansion writes all three; unwanted ones go to scratch
    uint32_t* ps = (is_device_ptr && src) ? src : nullptr;
    uint32_t* pd = (is_device_ptr && dst) ? dst : nullptr;
    uint32_t* pw = (is_device_ptr && w) ? w : nullptr;
    if (!ps) { TIGR_TRY(ds.alloc(bytes, s)); ps = ds.as<uint32_t>(); }
    if (!pd) { TIGR_TRY(dd.alloc(bytes, s)); pd = dd.as<uint32_t>(); }
    if (g->weighted && !pw) { TIGR_TRY(dw.alloc(bytes, s)); pw = dw.as<uint32_t>(); }
    TIGR_TRY(expand_arcs(g, ps, pd, g->weighted ? pw : nullptr, s));
    if (!is_device_ptr && g->m) {
        if (src) TIGR_CK(cudaMemcpyAsync(src, ps, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
        if (dst) TIGR_CK(cudaMemcpyAsync(dst, pd, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
        if (w && g->weighted) TIGR_CK(cudaMemcpyAsync(w, pw, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
    }
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_graph_export_csr(const tigr_graph* g, int64_t* row_ptr, uint32_t* col, uint32_t* w,
                                  int is_device_ptr, void* stream) {
    if (!g) return fail(TIGR_EINVAL, "graph_export_csr: NULL graph");
    cudaStream_t s = (cudaStream_t)stream;
    if (is_device_ptr) {
        TIGR_TRY(graph_export_csr_device(g, row_ptr, col, w, s));
        TIGR_CK(cudaStreamSynchronize(s));
        return TIGR_OK;
    }
    TmpBuf dr, dc, dw;
    if (row_ptr) TIGR_TRY(dr.alloc(sizeof(int64_t) * ((size_t)g->n + 1), s));
    if (col) TIGR_TRY(dc.alloc(sizeof(uint32_t) * (g->m ? g->m : 1), s));
    if (w && g->weighted) TIGR_TRY(dw.alloc(sizeof(uint32_t) * (g->m ? g->m : 1), s));
    TIGR_TRY(graph_export_csr_device(g, dr.as<int64_t>(), dc.as<uint32_t>(), dw.as<uint32_t>(), s));
    if (row_ptr) TIGR_CK(cudaMemcpyAsync(row_ptr, dr.p, sizeof(int64_t) * ((size_t)g->n + 1), cudaMemcpyDeviceToHost, s));
    if (col && g->m) TIGR_CK(cudaMemcpyAsync(col, dc.p, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
    if (w && g->weighted && g->m) TIGR_CK(cudaMemcpyAsync(w, dw.p, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

void tigr_graph_free(tigr_graph* g) { delete g; }

tigr_status tigr_graph_udt(const tigr_graph* g, uint32_t K, uint32_t dumb_weight, uint32_t unit_weight, void* stream,
                           tigr_graph** out) {
    if (!g || !out) return fail(TIGR_EINVAL, "graph_udt: NULL argument");
    *out = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(graph_udt_device(g, K, dumb_weight, unit_weight, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_graph_transpose(const tigr_graph* g, void* stream, tigr_graph** out) {
    if (!g || !out) return fail(TIGR_EINVAL, "graph_transpose: NULL argument");
    *out = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(graph_transpose_device(g, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_graph_reorder(const tigr_graph* g, void* stream, tigr_graph** out) {
    if (!g || !out) return fail(TIGR_EINVAL, "graph_reorder: NULL argument");
    *out = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    TIGR_TRY(graph_reorder_device(g, s, out));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_graph_permutation(const tigr_graph* g, uint32_t* cid, uint32_t* order, int is_device_ptr,
                                   void* stream) {
    if (!g) return fail(TIGR_EINVAL, "graph_permutation: NULL graph");
    if (!g->reordered) return fail(TIGR_EINVAL, "graph_permutation: graph is not reordered");
    cudaStream_t s = (cudaStream_t)stream;
    const cudaMemcpyKind k = is_device_ptr ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
    if (cid && g->n) TIGR_CK(cudaMemcpyAsync(cid, g->perm_cid.p, sizeof(uint32_t) * g->n, k, s));
    if (order && g->n) TIGR_CK(cudaMemcpyAsync(order, g->perm_order.p, sizeof(uint32_t) * g->n, k, s));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_virtualize(const tigr_graph* g, uint32_t K, tigr_layout layout, void* stream, tigr_vgraph** out) {
    if (!g || !out) return fail(TIGR_EINVAL, "virtualize: NULL argument");
    *out = nullptr;
    return virtualize_device(g, K, layout, (cudaStream_t)stream, out);
}

tigr_status tigr_vgraph_info(const tigr_vgraph* vg, uint64_t* nv, uint64_t* bytes, double* ms_build, uint32_t* lo,
                             uint32_t* hi) {
    if (!vg) return fail(TIGR_EINVAL, "vgraph_info: NULL vgraph");
    if (nv) *nv = vg->nv;
    if (bytes) *bytes = vg->vnode_ptr.bytes + vg->vn_phys.bytes + vg->vinfo.bytes;
    if (ms_build) *ms_build = vg->ms_build;
    if (lo) *lo = vg->lo;
    if (hi) *hi = vg->hi;
    return TIGR_OK;
}

tigr_status tigr_vgraph_pr_profile(tigr_vgraph* vg, void* stream, uint64_t* arcs, uint64_t* global_reds,
                                   uint32_t* hot_slots, uint32_t* n_in) {
    if (!vg) return fail(TIGR_EINVAL, "vgraph_pr_profile: NULL vgraph");
    TIGR_TRY(need_device());
    return tigr::pr_cid_profile(vg, (cudaStream_t)stream, arcs, global_reds, hot_slots, n_in);
}

tigr_status tigr_vgraph_export(const tigr_vgraph* vg, uint32_t* vnode_ptr, uint32_t* vn_phys, int is_device_ptr,
                               void* stream) {
    if (!vg) return fail(TIGR_EINVAL, "vgraph_export: NULL vgraph");
    cudaStream_t s = (cudaStream_t)stream;
    const cudaMemcpyKind k = is_device_ptr ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
    if (vnode_ptr)
        TIGR_CK(cudaMemcpyAsync(vnode_ptr, vg->vnode_ptr.p, sizeof(uint32_t) * ((size_t)vg->g->n + 1), k, s));
    if (vn_phys && vg->nv) TIGR_CK(cudaMemcpyAsync(vn_phys, vg->vn_phys.p, sizeof(uint32_t) * vg->nv, k, s));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_vgraph_assignment(const tigr_vgraph* vg, uint32_t* counts, uint32_t* nbr, uint32_t* w,
                                   int is_device_ptr, void* stream) {
    if (!vg || !counts || !nbr) return fail(TIGR_EINVAL, "vgraph_assignment: NULL argument");
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t m = vg->g->m;
    if (is_device_ptr) {
        TIGR_TRY(assignment_device(vg, counts, nbr, w, s));
        TIGR_CK(cudaStreamSynchronize(s));
        return TIGR_OK;
    }
    TmpBuf dc, dn, dw;
    TIGR_TRY(dc.alloc(sizeof(uint32_t) * (vg->nv ? vg->nv : 1), s));
    TIGR_TRY(dn.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    if (w) TIGR_TRY(dw.alloc(sizeof(uint32_t) * (m ? m : 1), s));
    TIGR_TRY(assignment_device(vg, dc.as<uint32_t>(), dn.as<uint32_t>(), dw.as<uint32_t>(), s));
    if (vg->nv) TIGR_CK(cudaMemcpyAsync(counts, dc.p, sizeof(uint32_t) * vg->nv, cudaMemcpyDeviceToHost, s));
    if (m) TIGR_CK(cudaMemcpyAsync(nbr, dn.p, sizeof(uint32_t) * m, cudaMemcpyDeviceToHost, s));
    if (w && m) TIGR_CK(cudaMemcpyAsync(w, dw.p, sizeof(uint32_t) * m, cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    return TIGR_OK;
}

tigr_status tigr_vgraph_partition(tigr_vgraph* vg, int nranks, int rank) {
    if (!vg) return fail(TIGR_EINVAL, "vgraph_partition: NULL vgraph");
    return partition_host(vg, nranks, rank);
}

void tigr_vgraph_free(tigr_vgraph* vg) { delete vg; }

tigr_status tigr_partition_ranges(uint32_t n, const int64_t* row_ptr, const uint32_t* vnode_ptr, int nranks,
                                  uint32_t* lo, uint32_t* hi) {
    if (!row_ptr || !vnode_ptr || !lo || !hi || nranks < 1) return fail(TIGR_EINVAL, "partition_ranges: bad argument");
    partition_ranges(n, row_ptr, vnode_ptr, nranks, lo, hi);
    return TIGR_OK;
}

tigr_status tigr_run(tigr_vgraph* vg, tigr_algo algo, uint32_t source, const tigr_run_opts* opts, void* out_values,
                     int out_is_device, tigr_stats* stats) {
    if (!vg) return fail(TIGR_EINVAL, "run: NULL vgraph");
    tigr_run_opts o;
    if (opts) o = *opts; else tigr_run_opts_default(&o);
    return run_device(vg, algo, source, o, out_values, out_is_device, stats);
}

tigr_status tigr_comm_unique_id(uint8_t id[128]) {
    if (!id) return fail(TIGR_EINVAL, "comm_unique_id: NULL");
    return comm_unique_id(id);
}

tigr_status tigr_comm_init(int nranks, int rank, const uint8_t id[128], int device, tigr_comm** out) {
    if (!id || !out) return fail(TIGR_EINVAL, "comm_init: NULL");
    *out = nullptr;
    TIGR_TRY(need_device());
    return comm_init(nranks, rank, id, device, out);
}

void tigr_comm_free(tigr_comm* c) { comm_free(c); }

tigr_status tigr_comm_group_create(int nranks, tigr_comm_group** out) {
    if (!out) return fail(TIGR_EINVAL, "comm_group_create: NULL");
    *out = nullptr;
    return comm_group_create(nranks, out);
}

tigr_status tigr_comm_init_group(tigr_comm_group* group, int rank, tigr_comm** out) {
    if (!group || !out) return fail(TIGR_EINVAL, "comm_init_group: NULL");
    *out = nullptr;
    return comm_init_group(group, rank, out);
}

void tigr_comm_group_free(tigr_comm_group* g) { comm_group_free(g); }

tigr_status tigr_comm_init_node(const char* name, int nranks, int rank, tigr_comm** out) {
    if (!out) return fail(TIGR_EINVAL, "comm_init_node: NULL");
    *out = nullptr;
    return comm_init_node(name, nranks, rank, out);
}

const char* tigr_last_error(void) { return t_err.c_str(); }

uint64_t tigr_launch_count(void) { return g_launches.load(); }

void tigr_release_cached_memory(void) { cache_release_all(); }

const char* tigr_version(void) { return "tigr-b200 0.1 (sm_100a)"; }

}  // extern "C"
