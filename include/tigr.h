/*
 * tigr.h -- C ABI of the B200-native Tigr hot path (libtigr.so).
 *
 * Tigr (Nodehi Sabet, Qiu, Zhao, ASPLOS'18; /root/reference/PAPER.md) runs
 * push-style vertex-centric graph analytics over a VIRTUALLY split graph: every
 * node of out-degree d is split into ceil(d/K) virtual nodes (Def. 1-2;
 * §4.1 "Virtual Node Array", L819-901, Fig. 10), whose edges are assigned in a
 * coalesced stride order (§4.4 "Edge-array Coalescing", L1104-1180, Fig. 12,
 * Alg. 3), and all virtual nodes of a family read/write the one value slot of
 * their physical node ("Implicit Value Synchronization", L978-1001).  A relax
 * kernel per algorithm (Alg. 2/3, L1080-1090 / L1161-1172) runs to a fixed point
 * under a worklist (§5).
 *
 * Conventions for every call:
 *  - Returns tigr_status; 0 == TIGR_OK.  Never aborts or exits.  On failure the
 *    message is available from tigr_last_error() (thread-local, valid until the
 *    next call on the same thread) and output handles are left NULL.
 *  - "device" pointers are CUDA device (or managed) pointers on the current
 *    device; "host" pointers are plain host memory (pinned memory is faster).
 *    `is_device_ptr` says which one the caller passes.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    All work is ordered on it; calls that return host-visible results
 *    synchronise it.
 *  - Handles own their device memory and are freed with the matching *_free.
 *    A tigr_vgraph references its tigr_graph: free the vgraph first.
 *  - Vertex ids are uint32 in [0, n); n <= 0xFFFFFFFE (0xFFFFFFFF is "infinity").
 *  - There is no CPU fallback: without a usable CUDA device every call that
 *    needs one returns TIGR_ECUDA.
 */
#ifndef TIGR_H_
#define TIGR_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    TIGR_OK = 0,
    TIGR_EINVAL = -1,      /* bad argument: id >= n, K == 0, source >= n, unweighted SSSP/SSWP, ... */
    TIGR_ENOMEM = -2,      /* device allocation failed */
    TIGR_ECUDA = -3,       /* CUDA runtime / driver error (no device, launch failure, ...) */
    TIGR_ENCCL = -4,       /* NCCL error (multi-GPU) */
    TIGR_ERANGE = -5,      /* size limit: n > 0xFFFFFFFE, edge/vnode counts beyond 32-bit slots */
    TIGR_ENOTCONV = -6,    /* max_iters reached before the fixed point */
    TIGR_EUNSUPPORTED = -7 /* option combination not implemented */
} tigr_status;

/* Algorithms (Table 4; semantics in DESIGN.md "Readings"). */
typedef enum {
    TIGR_BFS = 0,   /* level (hop count) from source; unreached = 0xFFFFFFFF (L718-720) */
    TIGR_SSSP = 1,  /* min weight sum from source; unreached = 0xFFFFFFFF (Fig. 2, Alg. 2/3) */
    TIGR_CC = 2,    /* min vertex id of the weakly connected component (Cor. 1, L688-694);
                       needs a graph built with symmetrize=1 (or symmetric_hint=1) */
    TIGR_SSWP = 3,  /* max over paths of the min edge weight; source = 0xFFFFFFFF,
                       unreached = 0 (Cor. 3, L725-734) */
    TIGR_PR = 4     /* PageRank, float64, fixed iteration count (fn. 7 L1078, Cor. 4 L787-791) */
} tigr_algo;

/* Edge assignment of the virtual nodes of one family. */
typedef enum {
    TIGR_LAYOUT_CONSECUTIVE = 0, /* Fig. 10 / Alg. 2: vnode j owns segment positions [jK, (j+1)K)
                                    (whole units: the same unit rule as STRIDED) */
    TIGR_LAYOUT_STRIDED = 1      /* Fig. 12 / Alg. 3: vnode j owns units j, j+m_v, j+2m_v, ...
                                    (unit = one 32-byte span of 8 edges when 8 | K, one 16-byte
                                    chunk of 4 edges when 4 | K, else 1 edge) */
} tigr_layout;

/* Worklist policy (§5; Table 8). */
typedef enum {
    TIGR_FRONTIER_AUTO = 0,    /* per iteration, on the device: QUEUE while the active nodes own
                                  fewer than 1/2 of the virtual nodes, else DENSE
                                  (16-byte-chunk layouts, i.e. 4 | K; otherwise DENSE) */
    TIGR_FRONTIER_DENSE = 1,   /* per-node active flags; every stored virtual node tests its node's
                                  flag, inactive ones exit early */
    TIGR_FRONTIER_NONE = 2,    /* every vnode every iteration (Table 8 "without worklist") */
    TIGR_FRONTIER_QUEUE = 3    /* queue of active nodes, virtual nodes derived on the fly from the
                                  queue and the degree bound ("dynamic mapping reasoning", §4.1
                                  L962-972): the stored virtual node array is never read.
                                  Needs 4 | K (else EUNSUPPORTED). */
} tigr_frontier;

/* Multi-GPU merge of the replicated frontier values after each relax (SURVEY §8(e), §8(f)
 * NEXT-2; exchange.cu).  PageRank always all-reduces its accumulator (every entry changes). */
typedef enum {
    TIGR_EXCHANGE_AUTO = 0,    /* per iteration: SPARSE while all ranks together changed at most
                                  n/2 nodes, else DENSE (the same verdict on every rank) */
    TIGR_EXCHANGE_DENSE = 1,   /* in-place MIN/MAX all-reduce of all n values; activity = moved */
    TIGR_EXCHANGE_SPARSE = 2,  /* every rank publishes {node, value} of the nodes it changed
                                  (8 bytes each); every rank applies all lists with the relax's
                                  atomic and activates the listed nodes */
    TIGR_EXCHANGE_FUSED = 3    /* no exchange step: the relax kernel applies each improvement to
                                  every peer's replica too (peer atomics, over NVLink between GPUs)
                                  and activates it there; a barrier ends each iteration.
                                  Thread-group communicator and 4 | K only (else EUNSUPPORTED). */
} tigr_exchange;

typedef struct tigr_graph tigr_graph;   /* device CSR; owns its buffers */
typedef struct tigr_vgraph tigr_vgraph; /* virtual node array + per-node info; refs its graph */
typedef struct tigr_comm tigr_comm;     /* a rank's communicator (NCCL, or a thread group) */
typedef struct tigr_comm_group tigr_comm_group; /* ranks that are threads of one process */

typedef struct {
    uint32_t max_iters;   /* frontier algorithms: iteration cap (0 = n + 1); exceeded -> TIGR_ENOTCONV */
    uint32_t pr_iters;    /* PR iterations (default 20, BASELINE config 4) */
    double pr_damping;    /* PR damping d (default 0.85) */
    int pr_dangling;      /* 0 = dangling mass dropped (default), 1 = spread uniformly */
    int schedule;         /* 0 = asynchronous in place ("synchronization relaxation", §5),
                             1 = BSP (each vnode reads its node's value from the previous iteration).
                             PR is always Jacobi. */
    int frontier;         /* tigr_frontier */
    int use_graph;        /* 1 (default) = iteration loop as a CUDA graph with a device-side
                             conditional WHILE node (no host round trip per iteration); 0 = host loop */
    int collect_stats;    /* 1 = count processed edges / updates on the device (slower) */
    int time_kernels;     /* 1 = CUDA-event time every relax launch into tigr_stats.ms_relax (host loop) */
    tigr_comm* comm;      /* NULL = single GPU; else this rank's communicator (see tigr_vgraph_partition) */
    void* stream;         /* cudaStream_t */
    int exchange;         /* tigr_exchange (multi-GPU frontier algorithms; default AUTO) */
    uint32_t frontier_div;/* FRONTIER_AUTO switch point D: an iteration runs from the queue while its
                             active nodes own fewer than 1/D of this rank's virtual nodes, else the
                             dense sweep (0 = default 2) */
} tigr_run_opts;

typedef struct {
    uint32_t iterations;      /* relax iterations executed (frontier algorithms: the last changes nothing) */
    uint32_t relax_launches;  /* relax kernel launches */
    uint64_t edges_processed; /* sum over iterations of the edges of active vnodes (collect_stats) */
    uint64_t updates;         /* successful atomic improvements (collect_stats; not PR) */
    uint64_t active_vnodes;   /* sum over iterations of active vnodes (collect_stats) */
    double ms_total;          /* device time of the whole run (init -> values on device) */
    double ms_relax;          /* device time of the relax launches (time_kernels) */
    double ms_exchange;       /* device time of the multi-GPU exchanges (time_kernels) */
    uint32_t queue_iterations;/* iterations whose relax ran from the active-node queue (FRONTIER_AUTO/QUEUE) */
    uint32_t sparse_exchanges;/* multi-GPU: iterations merged by the sparse (changed-node list) exchange */
    uint64_t active_nodes;    /* sum over iterations of active nodes that own virtual nodes (FRONTIER_AUTO/QUEUE) */
    double ms_kernels;        /* device time of the run outside the multi-GPU exchanges (ms_total - ms_exchange) */
    uint64_t bytes_alg;       /* algorithmic bytes of the relax launches by the SURVEY.md §8(d) byte model
                                 (DESIGN.md §5): PR always; BFS/SSSP/CC/SSWP only with collect_stats
                                 (it needs the processed-arc counts), else 0 */
} tigr_stats;

/* Fill *opts with the defaults above. */
void tigr_run_opts_default(tigr_run_opts* opts);

/* ---------------------------------------------------------------- graphs ---- */

/* Build a device CSR from an arc list (src[e] -> dst[e], weight w[e]); w may be NULL
 * (unweighted graph).  Arcs are grouped by source (Fig. 10a); duplicates
 * and self-loops are kept; the build is STABLE: the arcs of a source keep their input order
 * (arc e before arc f iff e < f), so the device CSR is the canonical one (a stable counting sort
 * by source) and tigr_graph_export_coo returns the arcs in that order.
 * symmetrize=1 appends (dst[e] -> src[e], w[e]) for every arc (weak connectivity, CC).
 * is_device_ptr = 0: src / dst / w are host arrays (pinned memory transfers at the link's rate);
 * the call copies them in chunks and, for a whole unsymmetrised graph of more than one chunk,
 * sorts each chunk on the device as it lands and merges the sorted runs into the rows, so most
 * of the build overlaps the transfer (same CSR as the device-input build).  The call returns
 * after the build completed (the stream is synchronised); the caller's arrays are not retained.
 * Errors: EINVAL (an id >= n, n == 0), ERANGE (n > 0xFFFFFFFE or too many arcs). */
tigr_status tigr_graph_from_coo(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                const uint32_t* w, int is_device_ptr, int symmetrize, void* stream,
                                tigr_graph** out);

/* Multi-GPU partitioned build: like tigr_graph_from_coo but keeps only the arcs
 * whose source lies in [src_lo, src_hi).  The graph still spans all n nodes (others have no
 * arcs), so a virtual split of it covers exactly this rank's virtual nodes and tigr_run with a
 * communicator merges the replicated values with the other ranks.  Every rank must use the
 * same full arc list (the PageRank accumulator order is derived from all arcs' targets).
 * tigr_graph_info's m is the kept arc count.  PageRank with pr_dangling = 1 is not supported
 * on partitioned graphs (dangling detection needs every rank's out-degrees). */
tigr_status tigr_graph_from_coo_part(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                     const uint32_t* w, int is_device_ptr, int symmetrize, uint32_t src_lo,
                                     uint32_t src_hi, void* stream, tigr_graph** out);

/* Source-node cuts for nranks partitions with ~equal arc counts: cuts[0] = 0 <= cuts[1] <= ...
 * <= cuts[nranks] = n (host array of nranks+1 entries); rank r builds [cuts[r], cuts[r+1]).
 * Granularity n/16384 nodes; deterministic for the same arc list. */
tigr_status tigr_coo_source_cuts(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                                 int is_device_ptr, int symmetrize, int nranks, void* stream, uint32_t* cuts);

/* Build from a CSR (row_ptr[n+1] int64, col[m], optional w[m]).  symmetric_hint=1 declares
 * the caller's graph symmetric (required for TIGR_CC).  Errors: EINVAL on a non-monotone
 * row_ptr, row_ptr[0] != 0, row_ptr[n] != m, or col >= n. */
tigr_status tigr_graph_from_csr(uint32_t n, uint64_t m, const int64_t* row_ptr, const uint32_t* col,
                                const uint32_t* w, int is_device_ptr, int symmetric_hint, void* stream,
                                tigr_graph** out);

/* Draw an R-MAT arc list on the device (Philox4x32-10 counter-based; spec in DESIGN.md
 * "Generator spec"; bit-identical to graphgen/) into caller-owned DEVICE buffers
 * src[m], dst[m] and (if non-NULL) w[m] with weights in [wmin, wmax]. */
tigr_status tigr_rmat_coo(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed,
                          uint64_t wseed, uint32_t wmin, uint32_t wmax, uint32_t* src, uint32_t* dst,
                          uint32_t* w, void* stream);

/* tigr_rmat_coo into temporary device memory + tigr_graph_from_coo. weighted=0 -> no weights. */
tigr_status tigr_graph_rmat(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed,
                            uint64_t wseed, uint32_t wmin, uint32_t wmax, int weighted, int symmetrize,
                            void* stream, tigr_graph** out);

/* Sizes and flags of a graph (any pointer may be NULL). */
tigr_status tigr_graph_info(const tigr_graph* g, uint32_t* n, uint64_t* m, int* weighted,
                            int* symmetric, int* transposed, uint64_t* device_bytes);

/* In-CSR (transpose) of g on the device: every arc u->v of g becomes v->u, grouped by v and
 * stable in g's arc order; weights follow their arcs.  The result remembers g's out-degrees,
 * so TIGR_PR run on a virtual split of it is PULL-based PageRank (
 * Thm. 3: pull needs an associative combine + atomics across a family).
 * Errors: ENOMEM, ECUDA. */
tigr_status tigr_graph_transpose(const tigr_graph* g, void* stream, tigr_graph** out);

/* Node relabelling by decreasing in-degree (ties by increasing id): node c of the result is
 * node order[c] of g, with its arcs in g's order and targets relabelled.  The paper's
 * transformations change which thread owns which edges, never the node numbering (§4,
 * L819-1180); this is a locality transformation of the same graph, beside them: the hottest
 * destinations get the smallest ids, so the frontier relax can bound their values in shared
 * memory and their value gathers share cache lines.  The result remembers the
 * permutation: tigr_run on a virtual split of it takes the source as an ORIGINAL id and
 * returns values indexed by ORIGINAL ids (CC labels stay the minimum original id).  Its
 * exported CSR / virtual arrays are in the new numbering.  g may be freed afterwards.
 * Errors: EUNSUPPORTED (transposed, partitioned or already reordered g), ENOMEM, ECUDA. */
tigr_status tigr_graph_reorder(const tigr_graph* g, void* stream, tigr_graph** out);

/* Permutation of a reordered graph: cid[v] = new id of original node v, order[c] = original
 * id of new node c (n entries each; either may be NULL).  EINVAL if g is not reordered. */
tigr_status tigr_graph_permutation(const tigr_graph* g, uint32_t* cid, uint32_t* order, int is_device_ptr,
                                   void* stream);

/* PHYSICAL uniform-degree-tree transformation (UDT, §3.2 Alg. 1): every
 * node v of out-degree d > K keeps <= K arcs and hands the rest to t = ceil((d-K)/(K-1)) new
 * split nodes of out-degree exactly K, numbered n, n+1, ... in order of v and creation (the
 * queue order of Alg. 1).  Arcs to original neighbours keep their weight (unit_weight if g is
 * unweighted); arcs to split nodes get dumb_weight: 0 for SSSP/BFS, 0xFFFFFFFF for SSWP
 * (Cor. 2-3, L695-734).  The result is a weighted graph with n + T nodes; results of the
 * original nodes are its first n values (Thm. 1).  Errors: EINVAL (K < 2), ERANGE. */
tigr_status tigr_graph_udt(const tigr_graph* g, uint32_t K, uint32_t dumb_weight, uint32_t unit_weight,
                           void* stream, tigr_graph** out);

/* Copy the arc list out in CSR order: src[m], dst[m], w[m] (w only if weighted and != NULL);
 * arc e is the e-th arc of the canonical CSR (Fig. 10a), so (src, dst, w) rebuilt by
 * tigr_graph_from_coo gives the same graph.  Buffers are caller-owned, host or device
 * (is_device_ptr), any of them may be NULL.  Errors: EINVAL (NULL graph). */
tigr_status tigr_graph_export_coo(const tigr_graph* g, uint32_t* src, uint32_t* dst, uint32_t* w,
                                  int is_device_ptr, void* stream);

/* Copy the CSR out (row_ptr[n+1], col[m], w[m] if weighted and w != NULL), arcs of a
 * source contiguous in the graph's internal order. */
tigr_status tigr_graph_export_csr(const tigr_graph* g, int64_t* row_ptr, uint32_t* col, uint32_t* w,
                                  int is_device_ptr, void* stream);

void tigr_graph_free(tigr_graph* g);

/* --------------------------------------------------------- virtual split ---- */

/* Virtual split transformation with degree bound K >= 1 (Def. 1-2; K = 0xFFFFFFFF means
 * "no split", the K=inf baseline of Table 2).  Builds on the device: family sizes
 * m_v = ceil(d_v / K) (0 for d_v = 0), vnode_ptr = exclusive scan of m_v, the virtual node
 * array vn_phys[NV] (Fig. 10b physicalNodeId row) and a 16-byte per-node record
 * {edge chunk, degree, first vnode, m_v}.  Errors: EINVAL (K == 0), ERANGE (NV >= 2^32). */
tigr_status tigr_virtualize(const tigr_graph* g, uint32_t K, tigr_layout layout, void* stream,
                            tigr_vgraph** out);

/* nv = number of virtual nodes; bytes = device bytes of the virtual structures;
 * ms_build = device time of the last tigr_virtualize (Table 7 analogue). */
tigr_status tigr_vgraph_info(const tigr_vgraph* vg, uint64_t* nv, uint64_t* bytes, double* ms_build,
                             uint32_t* vnode_lo, uint32_t* vnode_hi);

/* Diagnostic (measurement, not the hot path): how the push PageRank relax of this virtual
 * graph splits its arcs (fn. 7 L1078: one float64 accumulate per arc) between the per-SM
 * shared-memory table of the hot accumulator ids and global float64 reductions.  Prepares the
 * accumulator order if no PageRank ran yet (it is cached with the vgraph), then counts over this
 * rank's vnode range: arcs = its arcs, global_reds = the arcs whose accumulator id is >=
 * hot_slots (one L2 RED each per relax launch), n_in = nodes with in-arcs (the accumulator
 * entries ever written).  Any output may be NULL.  Synchronises the stream.  Errors: EINVAL (NULL
 * vgraph), EUNSUPPORTED (4 does not divide K, or a transposed graph: those run other kernels),
 * ECUDA. */
tigr_status tigr_vgraph_pr_profile(tigr_vgraph* vg, void* stream, uint64_t* arcs, uint64_t* global_reds,
                                   uint32_t* hot_slots, uint32_t* n_in);

/* Copy vnode_ptr[n+1] and vn_phys[NV] out (either may be NULL). */
tigr_status tigr_vgraph_export(const tigr_vgraph* vg, uint32_t* vnode_ptr, uint32_t* vn_phys,
                               int is_device_ptr, void* stream);

/* The edges each virtual node owns, walked with the relax kernels' own index arithmetic:
 * counts[NV] and, grouped by vnode in vnode order (offsets = exclusive scan of counts),
 * nbr[m] and (weighted graphs, if non-NULL) w[m].  For layout parity tests. */
tigr_status tigr_vgraph_assignment(const tigr_vgraph* vg, uint32_t* counts, uint32_t* nbr, uint32_t* w,
                                   int is_device_ptr, void* stream);

/* Restrict this rank's relax work to a contiguous, family-aligned vnode range balanced by
 * edge count (rank r of nranks).  nranks = 1 restores the full range. */
tigr_status tigr_vgraph_partition(tigr_vgraph* vg, int nranks, int rank);

void tigr_vgraph_free(tigr_vgraph* vg);

/* The range rule tigr_vgraph_partition applies, as a pure HOST computation (no device needed):
 * from host row_ptr[n+1] (int64) and vnode_ptr[n+1] (uint32), rank r of nranks owns vnodes
 * [lo[r], hi[r]) = the virtual nodes of nodes [cut(r), cut(r+1)), where cut(r) is the first node
 * whose arc prefix reaches r*m/nranks.  Ranges are contiguous, family-aligned and cover [0, NV). */
tigr_status tigr_partition_ranges(uint32_t n, const int64_t* row_ptr, const uint32_t* vnode_ptr, int nranks,
                                  uint32_t* lo, uint32_t* hi);

/* ------------------------------------------------------------------ runs ---- */

/* Run `algo` from `source` (ignored by CC and PR) to the fixed point (PR: pr_iters
 * iterations) and write n values to out_values: uint32 for BFS/SSSP/CC/SSWP, float64
 * for PR.  opts may be NULL (defaults).  stats may be NULL.
 * Errors: EINVAL (source >= n; SSSP/SSWP on an unweighted graph; CC on a graph not built
 * symmetric), ENOTCONV (max_iters hit; values hold the last iterate), ENCCL. */
tigr_status tigr_run(tigr_vgraph* vg, tigr_algo algo, uint32_t source, const tigr_run_opts* opts,
                     void* out_values, int out_is_device, tigr_stats* stats);

/* ------------------------------------------------------------- multi-GPU ---- */

/* NCCL bootstrap: rank 0 creates the 128-byte id and broadcasts it (e.g. over
 * torch.distributed); every rank then calls tigr_comm_init for its own GPU: `device` is the
 * CUDA device ordinal the rank runs on (it becomes the calling thread's current device), or
 * -1 for the current device.  Errors: EINVAL (bad rank / nranks / device), ENCCL. */
tigr_status tigr_comm_unique_id(uint8_t id[128]);
tigr_status tigr_comm_init(int nranks, int rank, const uint8_t id[128], int device, tigr_comm** out);
void tigr_comm_free(tigr_comm* comm);

/* Thread-group communicator: nranks ranks that are threads of ONE process, each on its own
 * current device (several ranks may share one GPU).  Exchanges read the peers' buffers directly
 * (unified addressing; NVLink peer access is enabled between distinct GPUs at init) and a host
 * barrier orders them; results are identical to the NCCL transport's.  Create the group once,
 * then every rank thread calls tigr_comm_init_group with its rank: the call returns once all
 * ranks have joined.  A rank that does not arrive at a barrier within TIGR_GROUP_TIMEOUT seconds
 * (default 300) fails every rank's run with ENCCL instead of hanging.  The group may be freed
 * after every rank has its tigr_comm (ranks keep the shared state alive).
 * Errors: EINVAL (nranks outside [1, 16], rank outside [0, nranks), rank joined twice),
 * EUNSUPPORTED (two ranks' GPUs without peer access). */
tigr_status tigr_comm_group_create(int nranks, tigr_comm_group** out);
tigr_status tigr_comm_init_group(tigr_comm_group* group, int rank, tigr_comm** out);
void tigr_comm_group_free(tigr_comm_group* group);

/* Node communicator: nranks PROCESSES of one node (normally one per GPU, e.g. under torchrun),
 * without NCCL.  Rank 0 creates the POSIX shared-memory segment "/tigr_<name>" (name: unique per
 * job, <= 200 chars), the other ranks attach to it; it holds a barrier and one slot per rank.
 * Device buffers are shared as CUDA IPC handles (mapped once per peer allocation, NVLink peer
 * access between distinct GPUs), so every exchange mode -- dense, sparse and fused -- reads or
 * updates the peers' replicas directly, exactly as the thread-group communicator does.  Each
 * rank calls it on its own current device; it returns once all ranks have joined.
 * Errors: EINVAL (name, nranks outside [1, 16], rank outside [0, nranks), nranks differs from
 * rank 0's), ENCCL (segment not created / barrier timeout, TIGR_GROUP_TIMEOUT seconds),
 * EUNSUPPORTED (GPUs without peer access).  tigr_comm_free detaches (rank 0 unlinks). */
tigr_status tigr_comm_init_node(const char* name, int nranks, int rank, tigr_comm** out);

/* ----------------------------------------------------------------- misc ---- */

const char* tigr_last_error(void);
/* libtigr caches freed device blocks for reuse (graph rebuilds allocate GBs); return them all
 * to the driver.  Synchronises the device. */
void tigr_release_cached_memory(void);
/* Number of CUDA kernels this library launched in this process (graph-launched ones
 * included, counted per executed node). */
uint64_t tigr_launch_count(void);
const char* tigr_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TIGR_H_ */
