/* omp_pagerank.c -- a multi-core CPU baseline for the PageRank step (SURVEY.md §8(d) "Optional
 * secondary baseline: an OpenMP pull-PR ... on all N cores, labelled clearly").  Not the oracle
 * (oracle/oracle.c stays the single-thread reference the parity tests use) and not the product:
 * bench.py reports it as `cpu_baseline_multicore`, beside the oracle's single-core number.
 *
 * Same iteration as the paper's PageRank (fn. 7 L1078; damping d, 20 iterations, dangling mass
 * dropped): x_{t+1}[v] = (1-d)/n + d * sum_{u->v} x_t[u] / outdeg(u).  Pull form on an in-CSR
 * built here with atomic counting (arc order inside a row is not fixed, so sums may differ from
 * the oracle in the last bits).
 *
 *   int omp_pagerank(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, int iters,
 *                    double d, int threads, double* x, double* ms_build, double* ms_iters);
 * returns 0 (or -1 on allocation failure); x[n] receives the ranks; threads <= 0 uses all.
 */
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static double now_ms(void) { return omp_get_wtime() * 1e3; }

int omp_pagerank(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, int iters, double d,
                 int threads, double* x, double* ms_build, double* ms_iters) {
    if (threads > 0) omp_set_num_threads(threads);
    double t0 = now_ms();
    uint64_t* rp = calloc((size_t)n + 1, sizeof(uint64_t));
    uint32_t* outdeg = calloc(n ? n : 1, sizeof(uint32_t));
    uint32_t* in_src = malloc((m ? m : 1) * sizeof(uint32_t));
    uint64_t* cur = malloc(((size_t)n + 1) * sizeof(uint64_t));
    double* contrib = malloc((n ? n : 1) * sizeof(double));
    if (!rp || !outdeg || !in_src || !cur || !contrib) {
        free(rp); free(outdeg); free(in_src); free(cur); free(contrib);
        return -1;
    }
#pragma omp parallel for schedule(static)
    for (uint64_t e = 0; e < m; ++e) {
        __atomic_fetch_add(&rp[dst[e] + 1], 1, __ATOMIC_RELAXED);
        __atomic_fetch_add(&outdeg[src[e]], 1u, __ATOMIC_RELAXED);
    }
    for (uint32_t v = 0; v < n; ++v) rp[v + 1] += rp[v];
    memcpy(cur, rp, ((size_t)n + 1) * sizeof(uint64_t));
#pragma omp parallel for schedule(static)
    for (uint64_t e = 0; e < m; ++e) in_src[__atomic_fetch_add(&cur[dst[e]], 1, __ATOMIC_RELAXED)] = src[e];
    double t1 = now_ms();
    const double base = (1.0 - d) / (double)n, x0 = 1.0 / (double)n;
#pragma omp parallel for schedule(static)
    for (uint32_t v = 0; v < n; ++v) {
        x[v] = x0;
        contrib[v] = outdeg[v] ? x0 / (double)outdeg[v] : 0.0;
    }
    for (int it = 0; it < iters; ++it) {
#pragma omp parallel for schedule(dynamic, 4096)
        for (uint32_t v = 0; v < n; ++v) {
            double s = 0.0;
            for (uint64_t e = rp[v]; e < rp[v + 1]; ++e) s += contrib[in_src[e]];
            x[v] = base + d * s;
        }
#pragma omp parallel for schedule(static)
        for (uint32_t v = 0; v < n; ++v) contrib[v] = outdeg[v] ? x[v] / (double)outdeg[v] : 0.0;
    }
    double t2 = now_ms();
    if (ms_build) *ms_build = t1 - t0;
    if (ms_iters) *ms_iters = t2 - t1;
    free(rp); free(outdeg); free(in_src); free(cur); free(contrib);
    return 0;
}

/* Level-synchronous top-down BFS from `source` on all cores (the same secondary baseline, for
 * BFS): out-CSR by atomic counting (untimed), then one parallel sweep of the frontier per level
 * with an atomic compare-and-swap claiming each newly reached vertex.  level[n] receives the
 * levels (0xFFFFFFFF = unreached), exactly the oracle's (BFS levels are unique). */
int omp_bfs(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, uint32_t source, int threads,
            uint32_t* level, double* ms_build, double* ms_run) {
    if (threads > 0) omp_set_num_threads(threads);
    double t0 = now_ms();
    uint64_t* rp = calloc((size_t)n + 1, sizeof(uint64_t));
    uint32_t* adj = malloc((m ? m : 1) * sizeof(uint32_t));
    uint64_t* cur = malloc(((size_t)n + 1) * sizeof(uint64_t));
    uint32_t* fa = malloc((n ? n : 1) * sizeof(uint32_t));
    uint32_t* fb = malloc((n ? n : 1) * sizeof(uint32_t));
    if (!rp || !adj || !cur || !fa || !fb) {
        free(rp); free(adj); free(cur); free(fa); free(fb);
        return -1;
    }
#pragma omp parallel for schedule(static)
    for (uint64_t e = 0; e < m; ++e) __atomic_fetch_add(&rp[src[e] + 1], 1, __ATOMIC_RELAXED);
    for (uint32_t v = 0; v < n; ++v) rp[v + 1] += rp[v];
    memcpy(cur, rp, ((size_t)n + 1) * sizeof(uint64_t));
#pragma omp parallel for schedule(static)
    for (uint64_t e = 0; e < m; ++e) adj[__atomic_fetch_add(&cur[src[e]], 1, __ATOMIC_RELAXED)] = dst[e];
    double t1 = now_ms();
#pragma omp parallel for schedule(static)
    for (uint32_t v = 0; v < n; ++v) level[v] = 0xFFFFFFFFu;
    uint64_t nf = 0, nn = 0;
    if (source < n) { level[source] = 0; fa[nf++] = source; }
    for (uint32_t lv = 1; nf; ++lv) {
        nn = 0;
#pragma omp parallel for schedule(dynamic, 64)
        for (uint64_t i = 0; i < nf; ++i) {
            const uint32_t u = fa[i];
            for (uint64_t e = rp[u]; e < rp[u + 1]; ++e) {
                const uint32_t v = adj[e];
                uint32_t expect = 0xFFFFFFFFu;
                if (level[v] == 0xFFFFFFFFu &&
                    __atomic_compare_exchange_n(&level[v], &expect, lv, 0, __ATOMIC_RELAXED, __ATOMIC_RELAXED))
                    fb[__atomic_fetch_add(&nn, 1, __ATOMIC_RELAXED)] = v;
            }
        }
        uint32_t* t = fa; fa = fb; fb = t;
        nf = nn;
    }
    double t2 = now_ms();
    if (ms_build) *ms_build = t1 - t0;
    if (ms_run) *ms_run = t2 - t1;
    free(rp); free(adj); free(cur); free(fa); free(fb);
    return 0;
}
