/* C-ABI example and test driver: plain C (gcc), only include/tigr.h and libtigr.so.
 *
 *   gcc -std=c11 -Iinclude examples/c_abi_bfs.c -Lpaper_conf_asplos_sabetq018_b200 -ltigr \
 *       -Wl,-rpath,$PWD/paper_conf_asplos_sabetq018_b200 -o build/c_abi_bfs
 *
 * Without a GPU it checks the host-only entry points and that compute calls fail with
 * TIGR_ECUDA (no CPU fallback).  With a GPU it builds the 9-node graph of PAPER.md Fig. 10,
 * splits it with K = 3 (4 virtual nodes: physicalNodeId row 1 2 2 3) and runs BFS from node 1.
 * Exit code 0 = all checks passed. */
#include <stdio.h>
#include <string.h>

#include "tigr.h"

static int fails = 0;
#define CHECK(c)                                                 \
    do {                                                         \
        if (!(c)) {                                              \
            fprintf(stderr, "FAILED %s (line %d): %s\n", #c, __LINE__, tigr_last_error()); \
            ++fails;                                             \
        }                                                        \
    } while (0)

int main(int argc, char** argv) {
    const int expect_gpu = argc > 1 && strcmp(argv[1], "--gpu") == 0;
    printf("%s\n", tigr_version());

    /* host-only: the partition rule on Fig. 10's CSR (row_ptr of nodes 0..8) */
    const int64_t row_ptr[10] = {0, 0, 3, 9, 12, 12, 12, 12, 12, 12};
    const uint32_t vnode_ptr[10] = {0, 0, 1, 3, 4, 4, 4, 4, 4, 4};
    uint32_t lo[2], hi[2];
    CHECK(tigr_partition_ranges(9, row_ptr, vnode_ptr, 2, lo, hi) == TIGR_OK);
    CHECK(lo[0] == 0 && hi[1] == 4 && hi[0] == lo[1]);

    /* Fig. 10 arcs (L903-960): v1 -> 2 5 4, v2 -> 5 4 6 8 7 3, v3 -> 7 6 8 */
    const uint32_t src[12] = {1, 1, 1, 2, 2, 2, 2, 2, 2, 3, 3, 3};
    const uint32_t dst[12] = {2, 5, 4, 5, 4, 6, 8, 7, 3, 7, 6, 8};
    tigr_graph* g = NULL;
    tigr_status st = tigr_graph_from_coo(9, 12, src, dst, NULL, 0, 0, NULL, &g);
    if (!expect_gpu) {
        CHECK(st == TIGR_ECUDA && g == NULL);  /* no device: loud failure, no fallback */
        printf(fails ? "c_abi: FAILED\n" : "c_abi: host checks ok (no GPU)\n");
        return fails != 0;
    }
    CHECK(st == TIGR_OK);
    tigr_vgraph* vg = NULL;
    CHECK(tigr_virtualize(g, 3, TIGR_LAYOUT_STRIDED, NULL, &vg) == TIGR_OK);
    uint64_t nv = 0;
    CHECK(tigr_vgraph_info(vg, &nv, NULL, NULL, NULL, NULL) == TIGR_OK && nv == 4);
    uint32_t phys[4];
    CHECK(tigr_vgraph_export(vg, NULL, phys, 0, NULL) == TIGR_OK);
    CHECK(phys[0] == 1 && phys[1] == 2 && phys[2] == 2 && phys[3] == 3);
    uint32_t lvl[9];
    tigr_run_opts o;
    tigr_run_opts_default(&o);
    tigr_stats stats;
    CHECK(tigr_run(vg, TIGR_BFS, 1, &o, lvl, 0, &stats) == TIGR_OK);
    const uint32_t want[9] = {0xFFFFFFFFu, 0, 1, 2, 1, 1, 2, 2, 2};  /* 1->{2,5,4}; 2->{3,6,7,8} */
    for (int v = 0; v < 9; ++v) CHECK(lvl[v] == want[v]);
    CHECK(tigr_run(vg, TIGR_SSSP, 1, &o, lvl, 0, NULL) == TIGR_EINVAL);  /* unweighted */
    tigr_vgraph_free(vg);
    tigr_graph_free(g);
    printf(fails ? "c_abi: FAILED\n" : "c_abi: GPU checks ok (Fig. 10 graph, BFS levels, %u iterations)\n",
           stats.iterations);
    return fails != 0;
}
