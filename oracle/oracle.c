/*
 * oracle/oracle.c -- CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * `--impl reference` legs may load this library.  The product path
 * (paper_conf_asplos_sabetq018_b200/) never links, imports or calls it, and it
 * shares no code, header, table or helper with the CUDA path.
 *
 * Plain, slow, single-threaded, obviously-correct C.  Every function cites the
 * passage of /root/reference/PAPER.md ("L<line>", section / figure / algorithm)
 * it follows; readings of silent or garbled passages are listed in DESIGN.md
 * ("Readings") and SURVEY.md §8(c).
 *
 * Where the method reaches a result with a plain definition (BFS levels,
 * shortest distances, weakly-connected-component labels, widest-path widths)
 * the oracle is that textbook definition (queue BFS, Dijkstra, union-find,
 * max-heap Dijkstra) -- Thm. 2 (L1030-1045) says the virtual split preserves
 * every push-based result, and these four have unique fixed points.  PageRank
 * is the finite power iteration with the same constants.
 * The virtual split and the edge assignment (Def. 2, Fig. 10, Fig. 12, Alg. 2/3)
 * follow the paper step by step, and or_push_virtual() runs Alg. 2/3 literally,
 * sequentially, to pin Thm. 2 and Table 8's iteration-count equality.
 *
 * Pins: tests/test_oracle.py (brute force, library routines, closed forms,
 * worked examples under tests/golden/).  See DESIGN.md "Oracle pins".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_INF32 0xFFFFFFFFu

/* ------------------------------------------------------------------------- */
/* c2  CSR (Fig. 10a): node array = exclusive prefix sum of the     */
/* out-degree histogram; edge array grouped by source, COO order kept within  */
/* a source (a stable counting sort).                                         */
/* ------------------------------------------------------------------------- */
int or_csr_build(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst,
                 const uint32_t* w, int64_t* row_ptr, uint32_t* col, uint32_t* wt) {
    for (uint64_t e = 0; e < m; ++e)
        if (src[e] >= n || dst[e] >= n) return -1;
    for (uint32_t v = 0; v <= n; ++v) row_ptr[v] = 0;
    for (uint64_t e = 0; e < m; ++e) row_ptr[src[e] + 1] += 1;      /* histogram */
    for (uint32_t v = 0; v < n; ++v) row_ptr[v + 1] += row_ptr[v];  /* scan */
    int64_t* cursor = (int64_t*)malloc(sizeof(int64_t) * (n ? n : 1));
    if (!cursor) return -2;
    for (uint32_t v = 0; v < n; ++v) cursor[v] = row_ptr[v];
    for (uint64_t e = 0; e < m; ++e) {                              /* stable scatter */
        int64_t p = cursor[src[e]]++;
        col[p] = dst[e];
        if (w && wt) wt[p] = w[e];
    }
    free(cursor);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* c3  Virtual split (Def. 1-2; §4.1 virtual node array L877-898,    */
/* Fig. 10b).  A node with out-degree d is split into ceil(d/K)      */
/* virtual nodes (Def. 2(iii): |B| = ceil(|Nv|/K)); reading (i): d = 0 gives  */
/* no virtual node.  vnode_ptr[v] = number of vnodes of nodes < v.            */
/* ------------------------------------------------------------------------- */
uint64_t or_virtual_count(uint32_t n, const int64_t* row_ptr, uint64_t K, uint64_t* vnode_ptr) {
    vnode_ptr[0] = 0;
    for (uint32_t v = 0; v < n; ++v) {
        uint64_t d = (uint64_t)(row_ptr[v + 1] - row_ptr[v]);
        uint64_t family = 0;
        uint64_t left = d;
        while (left > 0) {            /* one split node per (up to) K edges */
            family += 1;
            left = (left > K) ? left - K : 0;
        }
        vnode_ptr[v + 1] = vnode_ptr[v] + family;
    }
    return vnode_ptr[n];
}

/* physicalNodeId row of Fig. 10b: vnode i belongs to node v. */
void or_virtual_emit(uint32_t n, const uint64_t* vnode_ptr, uint32_t* vn_phys) {
    for (uint32_t v = 0; v < n; ++v)
        for (uint64_t i = vnode_ptr[v]; i < vnode_ptr[v + 1]; ++i) vn_phys[i] = v;
}

/* Edge assignment of vnode i, as absolute CSR edge indices (canonical order).
 *  layout 0 = consecutive (Fig. 10 / Alg. 2): vnode j of v owns
 *             segment positions [j*K, min((j+1)*K, d)).
 *  layout 1 = strided (Fig. 12 / Alg. 3): offset j, stride m_v
 *             (number of vnodes in the family, L1134-1136), positions
 *             j, j+m_v, j+2*m_v, ... < d  (reading (ii): t starts at 0).
 *             `chunk` c > 1 generalises the unit from one edge to c adjacent
 *             edges (positions p with (p / c) mod m_v == j) -- the layout the
 *             CUDA path uses for 128-bit loads.
 * Returns the number of edges written to out. */
uint64_t or_vnode_edges(const int64_t* row_ptr, const uint64_t* vnode_ptr, const uint32_t* vn_phys,
                        uint64_t i, uint64_t K, int layout, uint64_t chunk, int64_t* out) {
    uint32_t v = vn_phys[i];
    uint64_t j = i - vnode_ptr[v];
    uint64_t mv = vnode_ptr[v + 1] - vnode_ptr[v];
    uint64_t d = (uint64_t)(row_ptr[v + 1] - row_ptr[v]);
    uint64_t cnt = 0;
    if (layout == 0) {
        for (uint64_t p = j * K; p < d && p < (j + 1) * K; ++p) out[cnt++] = row_ptr[v] + (int64_t)p;
    } else {
        if (chunk == 0) chunk = 1;
        for (uint64_t p = 0; p < d; ++p)
            if ((p / chunk) % mv == j) out[cnt++] = row_ptr[v] + (int64_t)p;
    }
    return cnt;
}

/* ------------------------------------------------------------------------- */
/* c4  BFS: level = minimum hop count (BFS == SSSP with unit weights, L718-   */
/* 720).  Textbook FIFO queue over out-arcs.  Unreached = 0xFFFFFFFF.          */
/* ------------------------------------------------------------------------- */
int or_bfs(uint32_t n, const int64_t* row_ptr, const uint32_t* col, uint32_t source, uint32_t* lvl) {
    if (source >= n) return -1;
    for (uint32_t v = 0; v < n; ++v) lvl[v] = OR_INF32;
    uint32_t* queue = (uint32_t*)malloc(sizeof(uint32_t) * n);
    if (!queue) return -2;
    uint64_t head = 0, tail = 0;
    lvl[source] = 0;
    queue[tail++] = source;
    while (head < tail) {
        uint32_t u = queue[head++];
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            uint32_t v = col[e];
            if (lvl[v] == OR_INF32) { lvl[v] = lvl[u] + 1; queue[tail++] = v; }
        }
    }
    free(queue);
    return 0;
}

/* Binary min-heap of (key, vertex) with lazy deletion (shared by Dijkstra and
 * the widest-path variant, which pushes the negated key). */
typedef struct { uint64_t key; uint32_t v; } or_item;
typedef struct { or_item* a; uint64_t size, cap; } or_heap;

static int heap_push(or_heap* h, uint64_t key, uint32_t v) {
    if (h->size == h->cap) {
        uint64_t nc = h->cap ? h->cap * 2 : 1024;
        or_item* na = (or_item*)realloc(h->a, sizeof(or_item) * nc);
        if (!na) return -1;
        h->a = na; h->cap = nc;
    }
    uint64_t i = h->size++;
    h->a[i].key = key; h->a[i].v = v;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h->a[p].key <= h->a[i].key) break;
        or_item t = h->a[p]; h->a[p] = h->a[i]; h->a[i] = t; i = p;
    }
    return 0;
}

static or_item heap_pop(or_heap* h) {
    or_item top = h->a[0];
    h->a[0] = h->a[--h->size];
    uint64_t i = 0;
    for (;;) {
        uint64_t l = 2 * i + 1, r = l + 1, s = i;
        if (l < h->size && h->a[l].key < h->a[s].key) s = l;
        if (r < h->size && h->a[r].key < h->a[s].key) s = r;
        if (s == i) break;
        or_item t = h->a[s]; h->a[s] = h->a[i]; h->a[i] = t; i = s;
    }
    return top;
}

/* ------------------------------------------------------------------------- */
/* c5  SSSP (Fig. 2; Alg. 2/3): dist[v] = min over paths of the sum  */
/* of weights.  Dijkstra, binary heap, lazy deletion, uint64 accumulation.    */
/* Returns -3 if a finite distance does not fit below 0xFFFFFFFF.             */
/* ------------------------------------------------------------------------- */
int or_sssp(uint32_t n, const int64_t* row_ptr, const uint32_t* col, const uint32_t* wt,
            uint32_t source, uint32_t* dist_out) {
    if (source >= n) return -1;
    uint64_t* dist = (uint64_t*)malloc(sizeof(uint64_t) * n);
    if (!dist) return -2;
    for (uint32_t v = 0; v < n; ++v) dist[v] = UINT64_MAX;
    or_heap h = {0, 0, 0};
    dist[source] = 0;
    if (heap_push(&h, 0, source)) { free(dist); return -2; }
    while (h.size) {
        or_item it = heap_pop(&h);
        if (it.key != dist[it.v]) continue;          /* stale entry */
        uint32_t u = it.v;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            uint64_t alt = dist[u] + wt[e];
            if (alt < dist[col[e]]) {
                dist[col[e]] = alt;
                if (heap_push(&h, alt, col[e])) { free(h.a); free(dist); return -2; }
            }
        }
    }
    int rc = 0;
    for (uint32_t v = 0; v < n; ++v) {
        if (dist[v] == UINT64_MAX) dist_out[v] = OR_INF32;
        else if (dist[v] >= OR_INF32) { dist_out[v] = OR_INF32; rc = -3; }
        else dist_out[v] = (uint32_t)dist[v];
    }
    free(h.a); free(dist);
    return rc;
}

/* ------------------------------------------------------------------------- */
/* c7  SSWP (Cor. 3 L725-734: "minimal edge weight along a path"): width[v] = */
/* max over paths of the min edge weight.  Source = 0xFFFFFFFF (empty path),  */
/* unreachable = 0.  Max-heap Dijkstra (key = 0xFFFFFFFF - width in a min-heap)*/
/* ------------------------------------------------------------------------- */
int or_sswp(uint32_t n, const int64_t* row_ptr, const uint32_t* col, const uint32_t* wt,
            uint32_t source, uint32_t* wid) {
    if (source >= n) return -1;
    for (uint32_t v = 0; v < n; ++v) wid[v] = 0;
    or_heap h = {0, 0, 0};
    wid[source] = OR_INF32;
    if (heap_push(&h, 0, source)) return -2;
    while (h.size) {
        or_item it = heap_pop(&h);
        uint32_t u = it.v;
        if ((uint64_t)(OR_INF32 - wid[u]) != it.key) continue;   /* stale entry */
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            uint32_t alt = wid[u] < wt[e] ? wid[u] : wt[e];
            if (alt > wid[col[e]]) {
                wid[col[e]] = alt;
                if (heap_push(&h, (uint64_t)(OR_INF32 - alt), col[e])) { free(h.a); return -2; }
            }
        }
    }
    free(h.a);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* c6  CC (Cor. 1 L688-694; undirected = both directions L363-365):           */
/* label[v] = min vertex id of v's weakly connected component.  Union-find    */
/* over all arcs (path halving, union by size), then min id per root.         */
/* ------------------------------------------------------------------------- */
static uint32_t uf_find(uint32_t* parent, uint32_t x) {
    while (parent[x] != x) { parent[x] = parent[parent[x]]; x = parent[x]; }
    return x;
}

int or_cc(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, uint32_t* label) {
    uint32_t* parent = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    uint32_t* size = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    uint32_t* minid = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    if (!parent || !size || !minid) { free(parent); free(size); free(minid); return -2; }
    for (uint32_t v = 0; v < n; ++v) { parent[v] = v; size[v] = 1; minid[v] = OR_INF32; }
    for (uint64_t e = 0; e < m; ++e) {
        if (src[e] >= n || dst[e] >= n) { free(parent); free(size); free(minid); return -1; }
        uint32_t a = uf_find(parent, src[e]), b = uf_find(parent, dst[e]);
        if (a == b) continue;
        if (size[a] < size[b]) { uint32_t t = a; a = b; b = t; }
        parent[b] = a; size[a] += size[b];
    }
    for (uint32_t v = 0; v < n; ++v) {
        uint32_t r = uf_find(parent, v);
        if (v < minid[r]) minid[r] = v;
    }
    for (uint32_t v = 0; v < n; ++v) label[v] = minid[uf_find(parent, v)];
    free(parent); free(size); free(minid);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* c8  PageRank, float64 power iteration (fn. 7 L1078; Cor. 4 L787-791;       */
/* config: 20 iterations).  x_0 = 1/n;                                        */
/*   x_{t+1}[v] = (1-d)/n + d * sum_{arcs u->v} x_t[u] / d_u                  */
/* arcs counted with multiplicity; dangling (d_u = 0): dropped (policy 0) or  */
/* their mass spread uniformly (policy 1: + d * D / n, D = sum of dangling x).*/
/* The multiply and add are rounded separately (no FMA), as written.          */
/* ------------------------------------------------------------------------- */
int or_pagerank(uint32_t n, const int64_t* row_ptr, const uint32_t* col, uint32_t iters,
                double damping, int dangling, double* x) {
    if (n == 0) return 0;
    double* contrib = (double*)malloc(sizeof(double) * n);
    double* acc = (double*)malloc(sizeof(double) * n);
    if (!contrib || !acc) { free(contrib); free(acc); return -2; }
    const double base = (1.0 - damping) / (double)n;
    for (uint32_t v = 0; v < n; ++v) x[v] = 1.0 / (double)n;
    for (uint32_t t = 0; t < iters; ++t) {
        double dsum = 0.0;
        for (uint32_t u = 0; u < n; ++u) {
            int64_t du = row_ptr[u + 1] - row_ptr[u];
            contrib[u] = du ? x[u] / (double)du : 0.0;
            if (!du) dsum += x[u];
            acc[u] = 0.0;
        }
        for (uint32_t u = 0; u < n; ++u)
            for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) acc[col[e]] += contrib[u];
        volatile double dterm = dangling ? dsum / (double)n : 0.0;
        for (uint32_t v = 0; v < n; ++v) {
            volatile double a = acc[v] + dterm;
            volatile double prod = damping * a;
            x[v] = base + prod;
        }
    }
    free(contrib); free(acc);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Paper-literal push over the VIRTUAL graph (Alg. 2, Alg. 3        */
/* L1161-1172, worklist + synchronisation relaxation §5), run       */
/* sequentially.  Used only to pin Thm. 2 (L1030-1045: same values as the      */
/* original graph) and Table 8 (L1480-1486: same #iterations, BSP).            */
/*  algo: 0 BFS, 1 SSSP, 2 CC, 3 SSWP.  schedule: 0 async in place, 1 BSP      */
/*  (each vnode reads its node's value from the previous iteration).           */
/*  worklist: 0 = every vnode every iteration (Table 8 "without worklist"),    */
/*  1 = only vnodes of nodes whose value changed in the previous iteration.    */
/* Returns the number of iterations executed (when *converged, the last one   */
/* changed nothing), or a negative error.                                      */
/* ------------------------------------------------------------------------- */
static int improves(int algo, uint32_t alt, uint32_t cur) {
    return (algo == 3) ? (alt > cur) : (alt < cur);
}

int64_t or_push_virtual(uint32_t n, const int64_t* row_ptr, const uint32_t* col, const uint32_t* wt,
                        const uint64_t* vnode_ptr, const uint32_t* vn_phys, uint64_t K, int layout,
                        uint64_t chunk, int algo, uint32_t source, int schedule, int worklist,
                        uint32_t* val, uint64_t max_iters, int* converged) {
    uint64_t nv = vnode_ptr[n];
    uint32_t* prev = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    uint8_t* active = (uint8_t*)malloc(n ? n : 1);
    uint8_t* next = (uint8_t*)malloc(n ? n : 1);
    uint64_t maxd = 0;
    for (uint32_t v = 0; v < n; ++v) {
        uint64_t d = (uint64_t)(row_ptr[v + 1] - row_ptr[v]);
        if (d > maxd) maxd = d;
    }
    int64_t* edges = (int64_t*)malloc(sizeof(int64_t) * (maxd ? maxd : 1));
    if (!prev || !active || !next || !edges) { free(prev); free(active); free(next); free(edges); return -2; }
    /* initial values (§2.1, Fig. 2 initial row) */
    for (uint32_t v = 0; v < n; ++v) {
        if (algo == 2) val[v] = v;
        else if (algo == 3) val[v] = 0;
        else val[v] = OR_INF32;
        active[v] = (algo == 2) ? 1 : 0;
    }
    if (algo != 2) {
        if (source >= n) { free(prev); free(active); free(next); free(edges); return -1; }
        val[source] = (algo == 3) ? OR_INF32 : 0;
        active[source] = 1;
    }
    int64_t it = 0;
    *converged = 0;
    for (;;) {
        if ((uint64_t)it >= max_iters) break;       /* stop early: values after max_iters */
        ++it;
        memcpy(prev, val, sizeof(uint32_t) * n);
        memset(next, 0, n);
        int finished = 1;                                   /* Alg. 2 `finished` */
        for (uint64_t i = 0; i < nv; ++i) {                 /* tid = virtual node */
            uint32_t v = vn_phys[i];                        /* Alg. 2 line 2 */
            if (worklist && !active[v]) continue;
            uint32_t x = schedule ? prev[v] : val[v];       /* Alg. 2 line 3 */
            if (algo != 2 && algo != 3 && x == OR_INF32) continue;   /* not reached yet */
            if (algo == 3 && x == 0) continue;
            uint64_t cnt = or_vnode_edges(row_ptr, vnode_ptr, vn_phys, i, K, layout, chunk, edges);
            for (uint64_t t = 0; t < cnt; ++t) {            /* Alg. 2 line 6 / Alg. 3 line 6 */
                int64_t e = edges[t];
                uint32_t alt;
                if (algo == 0) alt = x + 1;
                else if (algo == 1) {
                    uint64_t s = (uint64_t)x + wt[e];
                    alt = s >= OR_INF32 ? OR_INF32 - 1 : (uint32_t)s;
                } else if (algo == 2) alt = x;
                else alt = x < wt[e] ? x : wt[e];
                uint32_t nb = col[e];
                if (improves(algo, alt, val[nb])) {         /* Alg. 2 line 8-10 */
                    val[nb] = alt;
                    next[nb] = 1;
                    finished = 0;
                }
            }
        }
        memcpy(active, next, n);
        if (finished) { *converged = 1; break; }
    }
    free(prev); free(active); free(next); free(edges);
    return it;
}

/* ------------------------------------------------------------------------- */
/* UDT physical transformation (§3.2 Alg. 1; dumb weights §3.3 Cor. 2-3 */
/* L695-734), run literally with a queue per high-degree node.  Node v with    */
/* d_v > K: q = v's neighbours (in CSR order), remove them from v; while       */
/* |q| > K: new node u gets K neighbours popped from the front, u is pushed;   */
/* finally v gets the <= K remaining entries.  New nodes are numbered n, n+1,  */
/* ... in creation order over v = 0..n-1.  An arc to an original neighbour      */
/* keeps its weight; an arc to a new node gets `dumb`.  Output: arc list        */
/* (src, dst, w) in creation order; returns the new node count n' (or 0 when    */
/* the output buffers are NULL: then *m_out receives the arc count only).      */
/* K >= 2 (K = 1 never terminates: each step removes 1 and adds 1).            */
/* ------------------------------------------------------------------------- */
uint64_t or_udt(uint32_t n, const int64_t* row_ptr, const uint32_t* col, const uint32_t* wt, uint64_t K,
                uint32_t dumb, uint32_t unit_weight, uint32_t* src, uint32_t* dst, uint32_t* w, uint64_t* m_out) {
    if (K < 2) return 0;
    uint64_t next = n, arcs = 0;
    uint64_t maxd = 0;
    for (uint32_t v = 0; v < n; ++v) {
        uint64_t d = (uint64_t)(row_ptr[v + 1] - row_ptr[v]);
        if (d > maxd) maxd = d;
    }
    /* queue of (node id, weight of the arc that will point to it) */
    uint64_t cap = maxd + maxd / (K - 1) + 2;
    uint64_t* qn = (uint64_t*)malloc(sizeof(uint64_t) * cap);
    uint32_t* qw = (uint32_t*)malloc(sizeof(uint32_t) * cap);
    if (!qn || !qw) { free(qn); free(qw); return 0; }
#define OR_EMIT(s_, d_, w_)                              \
    do {                                                 \
        if (src) { src[arcs] = (uint32_t)(s_); dst[arcs] = (uint32_t)(d_); w[arcs] = (w_); } \
        ++arcs;                                          \
    } while (0)
    for (uint32_t v = 0; v < n; ++v) {
        uint64_t d = (uint64_t)(row_ptr[v + 1] - row_ptr[v]);
        if (d <= K) {                                    /* not a high-degree node: unchanged */
            for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) OR_EMIT(v, col[e], wt ? wt[e] : unit_weight);
            continue;
        }
        uint64_t head = 0, tail = 0;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {   /* Alg. 1 lines 3-5 */
            qn[tail] = col[e];
            qw[tail] = wt ? wt[e] : unit_weight;
            ++tail;
        }
        while (tail - head > K) {                                   /* lines 6-10 */
            uint64_t u = next++;
            for (uint64_t i = 0; i < K; ++i, ++head) OR_EMIT(u, qn[head], qw[head]);
            qn[tail] = u;
            qw[tail] = dumb;
            ++tail;
        }
        for (; head < tail; ++head) OR_EMIT(v, qn[head], qw[head]);  /* lines 11-13 */
    }
#undef OR_EMIT
    free(qn); free(qw);
    if (m_out) *m_out = arcs;
    return next;
}
