"""Frontier-relax probe on cfg4 (R-MAT scale 24): runs BFS/SSSP/SSWP (weighted graph) and CC
(symmetrised graph) once each through the host loop, so that an ncu launch list
(`-k regex:k_relax`) gives one row per iteration.  Without ncu it prints per-algorithm totals
(device ms, iterations, processed arcs, updates).

    python tools/frontier_probe.py [--algos bfs,sssp,...] [--reps 3] [--K 8]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--algos", default="bfs,sssp,sswp,cc")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--K", type=int, default=8)
    ap.add_argument("--layout", default="strided")
    ap.add_argument("--graph", type=int, default=1, help="use_graph option (0: host loop)")
    ap.add_argument("--frontier", type=int, default=0)
    ap.add_argument("--reorder", type=int, default=0, help="run on tigr_graph_reorder(g)")
    args = ap.parse_args()
    rec = graphgen.recipe(args.config)
    s = torch.cuda.current_stream()
    algos = args.algos.split(",")
    out = {}
    g = vg = None
    for algo in algos:
        sym = algo == "cc"
        if g is None or g.sym != sym:
            if vg is not None:
                vg.free(); g.free()
            g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                                     weighted=not sym, symmetrize=sym, stream=s)
            if args.reorder:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                g2 = tigr.tigr_graph_reorder(g, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                print(json.dumps({"reorder_ms": e0.elapsed_time(e1), "sym": sym}), flush=True)
                g.free()
                g = g2
            g.sym = sym
            vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
        res = torch.empty(rec.n, dtype=torch.int32, device="cuda")
        if args.reps == 0:  # one plain run (for ncu launch lists)
            tigr.tigr_run(vg, algo, 0, out=res, stream=s, use_graph=args.graph, frontier=args.frontier)
            torch.cuda.synchronize()
            continue
        _, st = tigr.tigr_run(vg, algo, 0, out=res, stream=s, collect_stats=1, return_stats=True,
                              frontier=args.frontier)
        ts = []
        for _ in range(args.reps):
            _, st2 = tigr.tigr_run(vg, algo, 0, out=res, stream=s, return_stats=True, use_graph=args.graph,
                                   frontier=args.frontier)
            ts.append(st2["ms_total"])
        out[algo] = {"ms": statistics.median(ts), "ms_min": min(ts), "iterations": st["iterations"],
                     "edges_processed": st["edges_processed"], "updates": st["updates"],
                     "nv": vg.info()["nv"]}
        print(json.dumps({algo: out[algo]}), flush=True)


if __name__ == "__main__":
    main()
