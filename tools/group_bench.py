"""Multi-rank frontier runs on ONE GPU through the thread-group communicator: P ranks (threads)
share cuda:0, so the times are not multi-GPU numbers; they show what each exchange protocol
costs on top of the relax work (dense all-reduce, sparse lists, fused peer updates) at a
BASELINE size.  Every rank's result is checked against the single-rank run.

    python tools/group_bench.py [--config cfg4] [--ranks 2] [--algos bfs,sssp,cc]
"""
import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--algos", default="bfs,sssp,cc")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    rec = graphgen.recipe(args.config)
    n, m, P = rec.n, rec.m, args.ranks
    s0 = torch.cuda.current_stream()
    src = torch.empty(m, dtype=torch.int32, device="cuda")
    dst, w = torch.empty_like(src), torch.empty_like(src)
    tigr.tigr_rmat_coo(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, w, stream=s0)
    torch.cuda.synchronize()
    out = {"config": args.config, "ranks": P, "note": "all ranks share one GPU"}
    for algo in args.algos.split(","):
        sym = algo == "cc"
        g1 = tigr.tigr_graph_from_coo(n, src, dst, None if sym else w, symmetrize=sym, stream=s0)
        vg1 = tigr.tigr_virtualize(g1, 8, "strided", stream=s0)
        ref, st1 = tigr.tigr_run(vg1, algo, rec.source, stream=s0, return_stats=True, use_graph=0)
        res = {"single_rank_ms": st1["ms_total"], "iterations": st1["iterations"]}
        vg1.free(); g1.free()
        for mode in ("dense", "sparse", "fused"):
            group = tigr.tigr_comm_group_create(P)
            times = [[] for _ in range(P)]
            bad = []
            stats = [None] * P

            def worker(r):
                torch.cuda.set_device(0)
                s = torch.cuda.Stream()
                comm = tigr.tigr_comm_init_group(group, r)
                g = tigr.tigr_graph_from_coo(n, src, dst, None if sym else w, symmetrize=sym, stream=s)
                vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
                tigr.tigr_vgraph_partition(vg, P, r)
                o = torch.empty(n, dtype=torch.int32, device="cuda")
                for _ in range(args.reps):
                    t0 = time.perf_counter()
                    _, st = tigr.tigr_run(vg, algo, rec.source, out=o, comm=comm, exchange=mode, stream=s,
                                          return_stats=True)
                    times[r].append((time.perf_counter() - t0) * 1e3)
                    stats[r] = st
                if not np.array_equal(o.cpu().numpy().view(np.uint32), ref):
                    bad.append(r)
                vg.free(); g.free()
                comm.free()

            th = [threading.Thread(target=worker, args=(r,)) for r in range(P)]
            for t in th:
                t.start()
            for t in th:
                t.join()
            group.free()
            res[mode] = {"ms_wall_median": statistics.median(max(t[i] for t in times) for i in range(args.reps)),
                         "iterations": stats[0]["iterations"], "sparse_exchanges": stats[0]["sparse_exchanges"],
                         "matches_single_rank": not bad}
        out[algo] = res
        print(json.dumps({algo: res}), flush=True)


if __name__ == "__main__":
    main()
