// internal.cuh -- shared internals of libtigr (CUDA, sm_100a).  Not part of the ABI.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <memory>
#include <string>

#include "tigr.h"

namespace tigr {

constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kChunk = 4;          // edges per 16-byte chunk (col and weight arrays)
constexpr uint32_t kSpan = 8;           // edges per 32-byte span: every node's segment starts on a
                                        // span and is padded to whole spans (cptr counts spans)
constexpr uint32_t kPad = 0xFFFFFFFFu;  // column value of padding slots
constexpr int kBlock = 256;

// ---- error state (tigr_last_error) -------------------------------------------------------
void set_error(const std::string& msg);
tigr_status fail(tigr_status st, const std::string& msg);
tigr_status cuda_fail(cudaError_t e, const char* what, const char* file, int line);

extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t k = 1) { g_launches.fetch_add(k, std::memory_order_relaxed); }

#define TIGR_CK(call)                                                         \
    do {                                                                      \
        cudaError_t _e = (call);                                              \
        if (_e != cudaSuccess) return ::tigr::cuda_fail(_e, #call, __FILE__, __LINE__); \
    } while (0)

#define TIGR_CKL(what)                                                        \
    do {                                                                      \
        ::tigr::count_launch();                                               \
        cudaError_t _e = cudaGetLastError();                                  \
        if (_e != cudaSuccess) return ::tigr::cuda_fail(_e, what, __FILE__, __LINE__); \
    } while (0)

#define TIGR_TRY(expr)                                                        \
    do {                                                                      \
        tigr_status _s = (expr);                                              \
        if (_s != TIGR_OK) return _s;                                         \
    } while (0)

// Development tracing: with TIGR_TRACE=1 in the environment, trace(s, "phase") synchronises
// the stream and prints the host wall time since the previous trace point (stderr).
void trace(cudaStream_t s, const char* what);

// Development knobs for A/B sweeps (tools/dev/): read from the environment only when the
// library is built with -DTIGR_DEV_KNOBS (TIGR_DEV_KNOBS=1 python tools/native_build.py); the
// shipped build always takes the default, so no environment variable changes a kernel.
int dev_knob(const char* name, int dflt);

inline unsigned grid_for(uint64_t items, int block = kBlock) {
    uint64_t g = (items + block - 1) / block;
    return (unsigned)(g ? g : 1);
}

// ---- device buffers ------------------------------------------------------------------------
// Owning device allocation of a persistent structure.  Stream-ordered (cudaMallocAsync from the
// device's default pool, whose release threshold libtigr raises so that freed blocks stay cached:
// rebuilding a graph every bench step costs no cudaMalloc/cudaFree synchronisation).  Freed on
// the stream it was allocated on; callers synchronise before freeing a handle.
struct DevBuf {
    void* p = nullptr;
    size_t bytes = 0;
    cudaStream_t s = nullptr;
    tigr_status alloc(size_t nbytes, cudaStream_t stream);
    void release();
    ~DevBuf() { release(); }
    template <class T> T* as() const { return static_cast<T*>(p); }
};

void init_pool();  // raise the default pool's release threshold (once per process)

struct TmpBuf {  // cudaMallocAsync / cudaFreeAsync on a stream
    void* p = nullptr;
    cudaStream_t s = nullptr;
    tigr_status alloc(size_t nbytes, cudaStream_t stream);
    ~TmpBuf();
    template <class T> T* as() const { return static_cast<T*>(p); }
};

// Host arrays of an arc list (tigr_graph_from_coo with host pointers): the CSR build copies them
// to its device buffers chunk by chunk, overlapped with the arc-list scan (sort.cu).
struct HostArcs {
    const uint32_t* src;
    const uint32_t* dst;
    const uint32_t* w;
};

// ---- scan (scan.cu) ----------------------------------------------------------------------
// out[i] = sum_{k<i} f(k) for i in [0, count], where f is selected by `kind` over `in`:
enum ScanKind : int {
    SCAN_U32 = 0,        // f(k) = in[k]
    SCAN_CEIL_DIV = 1,   // f(k) = ceil(in[k] / div)
};
tigr_status exclusive_scan_u64(const uint32_t* in, uint64_t count, ScanKind kind, uint32_t div,
                               uint64_t* out, cudaStream_t s);
tigr_status exclusive_scan_u32(const uint32_t* in, uint64_t count, ScanKind kind, uint32_t div,
                               uint32_t* out, cudaStream_t s, uint64_t* total_host);

}  // namespace tigr

// ---- handles -----------------------------------------------------------------------------
struct tigr_graph {
    uint32_t n = 0;
    uint64_t m = 0;          // arcs (after symmetrisation)
    uint64_t nchunks = 0;    // 16-byte chunks per edge array (padded segments; even: 2 per span)
    bool weighted = false;
    bool symmetric = false;
    tigr::DevBuf row_ptr;    // int64[n+1], canonical offsets
    tigr::DevBuf deg;        // uint32[n]
    tigr::DevBuf cptr;       // uint32[n+1], first 32-byte span of each node's segment
    tigr::DevBuf col;        // uint32[4 * nchunks], padded segments, pads = 0xFFFFFFFF
    tigr::DevBuf wt;         // uint32[4 * nchunks] or empty
    // in-degree sketch from the arc-list scan (PageRank accumulator order, pr.cu)
    tigr::DevBuf in_flag;    // uint32[n/32 + 1] bitmap: node has an in-arc
    tigr::DevBuf in_sample;  // uint32[n]: in-arcs among every 16th arc
    bool has_in_sketch = false;
    // transposed graphs (tigr_graph_transpose): arcs reversed; src_deg = out-degrees of the
    // original graph (PageRank pull divides by them)
    bool transposed = false;
    // partitioned builds (tigr_graph_from_coo_part): only sources in [part_lo, part_hi) have arcs
    uint32_t part_lo = 0, part_hi = 0xFFFFFFFFu;
    tigr::DevBuf src_deg;    // uint32[n] (transposed graphs only)
    // reordered graphs (tigr_graph_reorder): node c here is node perm_order[c] of the source
    // graph, perm_cid is the inverse; sources and results are translated at the ABI
    bool reordered = false;
    tigr::DevBuf perm_cid;   // uint32[n]: original id -> id here
    tigr::DevBuf perm_order; // uint32[n]: id here -> original id
};

namespace tigr { struct PeerGroup; struct LocalGroup; }

// A rank's communicator.  Two transports (comm.cu): NCCL (one process per GPU), or a thread
// group (ranks are threads of one process; exchanges read the peers' buffers directly through
// unified addressing / NVLink peer access, synchronised by a host barrier).
struct tigr_comm {
    void* nccl = nullptr;    // ncclComm_t (NCCL transport)
    std::shared_ptr<tigr::PeerGroup> local;   // peer-group transport (thread group or node group)
    int nranks = 1;
    int rank = 0;
    int device = 0;
    tigr::DevBuf scratch;    // exchange staging (grown on demand)
    tigr::DevBuf counts;     // uint32[nranks] (NCCL count all-gather)
};

struct tigr_comm_group {
    std::shared_ptr<tigr::LocalGroup> g;
};

struct tigr_vgraph;  // defined in vgraph.cuh

namespace tigr {
// push PageRank's split of a rank's arcs into hot shared-memory slots and global float64
// reductions (pr.cu; the C-ABI diagnostic tigr_vgraph_pr_profile)
tigr_status pr_cid_profile(tigr_vgraph* vg, cudaStream_t s, uint64_t* arcs, uint64_t* reds, uint32_t* hot,
                           uint32_t* n_in);
}  // namespace tigr
