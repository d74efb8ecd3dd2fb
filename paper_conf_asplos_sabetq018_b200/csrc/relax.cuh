// relax.cuh -- kernel argument block and kernel-pointer dispatch for relax.cu (internal).
#pragma once

#include "internal.cuh"
#include "vgraph.cuh"

namespace tigr {

constexpr int kRelaxThreads = 256;

// Worklist stamps (one byte per node and iteration parity): node v is active in iteration it
// iff stamp[(it & 1) n + v] == stamp_of(it).  Stamp values cycle through 1..255 (0 = never
// stamped), so a stale byte can only match again 510 iterations later -- a spurious activation,
// which is harmless: the node re-pushes a value its targets already hold.  One
// byte instead of four: the per-iteration queue build scans n bytes instead of 4n.
typedef uint8_t stamp_t;
__host__ __device__ __forceinline__ stamp_t stamp_of(uint32_t it) { return (stamp_t)(1u + (it - 1u) % 255u); }

struct RelaxArgs {
    const uint32_t* __restrict__ vn_phys;
    const uint4* __restrict__ vinfo;
    const uint32_t* __restrict__ col;
    const uint32_t* __restrict__ wt;
    uint32_t lo, hi, K, n;
    uint32_t* val;               // values, updated in place with atomics
    const uint32_t* prev;        // BSP snapshot
    stamp_t* stamp;              // stamp_t[2n] worklist stamps (stamp_of)
    double* acc;                 // PR accumulator (RED.ADD.F64 target)
    const double* contrib;       // PR x/deg
    Ctl* ctl;
};

typedef void (*RelaxFn)(RelaxArgs);

struct Ctl;
// fused multi-GPU exchange (exchange.cu): the replicas of every rank of a thread group
constexpr int kMaxPeers = 16;
struct FusedPeers {
    int P, me;
    uint32_t* val[kMaxPeers];
    stamp_t* stamp[kMaxPeers];
    Ctl* ctl[kMaxPeers];
};

// queue-driven frontier relax with dynamic virtual-node mapping (frontier.cu)
struct FqArgs {
    const uint32_t* qv;   // uint32[2][n] queue node ids (slot = iteration parity)
    const uint32_t* qo;   // uint32[2][n] queue-space first virtual node of each entry
    int mode;             // 0 = per iteration (queue if vnodes * dense_div < span), 1 = queue, 2 = dense
    uint32_t dense_div;
    uint32_t* settled;    // BFS / CC: bit v set once v's value is final (nullptr: always test the value)
    const FusedPeers* peers;  // fused exchange: every improvement is also applied to the peers' replicas
    uint32_t run;         // queue tiles per warp run (frontier_kernel.cuh): the search runs once per run
    const uint32_t* cw;   // SSSP / SSWP packed arcs: target | (w - wmin) << idbits (nullptr: col + wt)
    uint32_t idmask, idbits, wmin;
};
typedef void (*FqFn)(RelaxArgs, FqArgs);
// unit 4 or 8 (vgraph.cuh); packed: SSSP / SSWP read FqArgs.cw (target | weight slots)
FqFn relax_fq_kernel(int algo, int layout, int unit, bool bsp, bool stats, bool packed);
unsigned relax_fq_grid(FqFn fn);   // persistent grid: SMs x resident blocks
int relax_fq_threads();
struct Ctl;
tigr_status compact_launch(const tigr_vgraph* vg, Ctl* ctl, int delta, cudaStream_t s);
tigr_status pack_arcs_prepare(tigr_vgraph* vg, cudaStream_t s);  // SSSP / SSWP packed arcs (frontier.cu)
typedef void (*AssignFn)(RelaxArgs, const uint32_t*, uint32_t*, uint32_t*, uint32_t*, int, int);

RelaxFn relax_kernel(int algo, int layout, int unit, int front, bool bsp, bool stats);
// frontier relax with *per_thread virtual nodes per thread (nullptr: use relax_kernel's)
RelaxFn relax_mlp_kernel(int algo, int layout, int unit, int front, bool bsp, bool stats, int* per_thread);
// PageRank push with an in-degree-ordered accumulator (pr.cu)
struct PrFuse {
    int mode = 0;               // 0 read contrib, 1 first iteration (x = x0), 2 from prev
    uint32_t n_in = 0;
    const double* prev = nullptr;  // accumulator of the previous iteration (cid order)
    const uint32_t* cid = nullptr;
    double base = 0.0, damping = 0.0, x0 = 0.0;
    int probe = 0;              // 0; development builds: timing decomposition (pr.cu)
};
struct PrCidPlan {
    void (*fn)(RelaxArgs, const uint32_t*, uint32_t, PrFuse) = nullptr;
    unsigned grid = 0, tiles = 0;
    int threads = 256, per_thread = 4;
    size_t smem = 0;
    uint32_t hot = 0;  // accumulator ids below this are summed in shared memory
};
RelaxFn relax_pr_pull_kernel(int layout, int unit, int* per_thread);   // pull PageRank (pr.cu, NEXT-1)
tigr_status pr_cid_prepare(tigr_vgraph* vg, cudaStream_t s);
PrCidPlan pr_cid_plan(tigr_vgraph* vg);
tigr_status pr_cid_apply(tigr_vgraph* vg, double base, double damping, int dangling, const double* dsum_cur,
                         double* dsum_next, cudaStream_t s, double* acc = nullptr, bool reset = true);
AssignFn assign_kernel(int layout, int unit);

__global__ void k_init(int algo, uint32_t n, uint32_t source, uint32_t* __restrict__ val,
                       stamp_t* __restrict__ stamp, Ctl* ctl, uint32_t max_iters,
                       const uint32_t* __restrict__ cid, const uint32_t* __restrict__ order,
                       uint32_t* __restrict__ settled);
// out[v] = val[cid[v]] (results of a reordered graph in original ids)
tigr_status unpermute(uint32_t n, const uint32_t* cid, const void* val, void* out, bool f64, cudaStream_t s);
__global__ void k_control(Ctl* ctl, cudaGraphConditionalHandle h, int use_handle);
__global__ void k_diff(uint32_t n, const uint32_t* __restrict__ val, uint32_t* __restrict__ prev,
                       stamp_t* __restrict__ stamp, Ctl* ctl);
// multi-GPU merge of the replicated frontier values after a relax (exchange.cu)
struct ExchangeArgs {
    tigr_comm* comm;
    int mode;          // tigr_exchange
    int algo;
    uint32_t n;
    uint32_t* val;
    uint32_t* prev;
    stamp_t* stamp;
    uint2* list;       // uint2[n] records of this rank (sparse mode)
    Ctl* ctl;
};
tigr_status exchange_frontier(const ExchangeArgs& x, cudaStream_t s, bool* sparse_used);
tigr_status fused_setup(tigr_comm* c, uint32_t* val, stamp_t* stamp, Ctl* ctl, DevBuf& peers_buf,
                        cudaStream_t s, const FusedPeers** out);
tigr_status fused_barrier(tigr_comm* c, cudaStream_t s);
tigr_status fused_end_iteration(tigr_comm* c, Ctl* ctl, cudaStream_t s);
// oid (nullable): contrib is stored at oid[v] instead of v (pull PageRank's source order, pr.cu)
__global__ void k_pr_init(uint32_t n, const uint32_t* __restrict__ deg, double* __restrict__ x,
                          double* __restrict__ contrib, double* __restrict__ acc, Ctl* ctl,
                          const uint32_t* __restrict__ oid);
__global__ void k_pr_apply(uint32_t n, const uint32_t* __restrict__ deg, double base, double damping,
                           int dangling, double* __restrict__ x, double* __restrict__ contrib,
                           double* __restrict__ acc, const double* dsum_cur, double* dsum_next,
                           const uint32_t* __restrict__ oid);
tigr_status pr_pull_prepare(tigr_vgraph* vg, cudaStream_t s);  // oid order + remapped in-arcs (pr.cu)

}  // namespace tigr
