"""Tigr ablation on B200 (the structure of PAPER.md Fig. 13, §6.3, and
Table 8): the same engine with the transformation disabled (K = infinity: one
virtual node per node = the original graph), the virtual split with consecutive edge
assignment (Tigr-V, Alg. 2) and with the coalesced stride assignment (Tigr-V+, Alg. 3);
worklist on/off and async/BSP schedules.  Device time per run (CUDA events inside tigr_run),
median of 5, on the paper-shaped synthetic graphs.  Prints one JSON line per measurement.

  python tools/ablation.py [--cfg cfg3] [--algos sssp,sswp,bfs,pr]
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

INF_K = 0xFFFFFFFF


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", default="cfg3")
    ap.add_argument("--algos", default="sssp,sswp,bfs,pr")
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    rec = graphgen.recipe(args.cfg)
    s = torch.cuda.current_stream()
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                             weighted=True, stream=s)
    variants = [("baseline K=inf", INF_K, "strided"), ("Tigr-V K=8 consecutive", 8, "consecutive"),
                ("Tigr-V+ K=8 strided", 8, "strided"), ("Tigr-V+ K=4", 4, "strided"),
                ("Tigr-V+ K=16", 16, "strided"), ("Tigr-V+ K=32", 32, "strided")]
    for algo in args.algos.split(","):
        base_ms = {}
        for name, K, layout in variants:
            vg = tigr.tigr_virtualize(g, K, layout, stream=s)
            modes = [("worklist async", 1, 0)]
            if algo != "pr":
                modes += [("worklist BSP", 1, 1), ("no worklist BSP", 2, 1)]
            for mname, front, sched in modes:
                kw = {} if algo == "pr" else {"frontier": front, "schedule": sched}
                times, st = [], None
                for _ in range(args.reps):
                    _, st = tigr.tigr_run(vg, algo, rec.source, stream=s, return_stats=True, **kw)
                    times.append(st["ms_total"])
                ms = statistics.median(times)
                base_ms.setdefault(mname, ms)
                _, st2 = tigr.tigr_run(vg, algo, rec.source, stream=s, return_stats=True, collect_stats=1, **kw)
                print(json.dumps({"cfg": args.cfg, "algo": algo, "variant": name, "mode": mname, "K": K,
                                  "layout": layout, "nv": vg.info()["nv"], "ms": ms,
                                  "speedup_vs_baseline": base_ms[mname] / ms, "iterations": st["iterations"],
                                  "edges_processed": st2["edges_processed"],
                                  "active_vnodes": st2["active_vnodes"]}), flush=True)
            vg.free()
        # Tigr-UDT (physical transformation, Alg. 1 + dumb weights, Cor. 2-3): no virtual split
        if algo in ("sssp", "sswp", "bfs"):
            for Ku in (8, 32):
                if algo == "bfs":
                    g1 = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed,
                                              weighted=False, stream=s)
                    gu = tigr.tigr_graph_udt(g1, Ku, 0, 1, stream=s)
                    g1.free()
                    run_algo = "sssp"  # BFS = SSSP with unit weights and dumb weight 0
                else:
                    gu = tigr.tigr_graph_udt(g, Ku, 0 if algo == "sssp" else 0xFFFFFFFF, stream=s)
                    run_algo = algo
                vgu = tigr.tigr_virtualize(gu, INF_K, "strided", stream=s)
                for mname, front, sched in (("worklist async", 1, 0), ("worklist BSP", 1, 1)):
                    times = []
                    for _ in range(args.reps):
                        _, st = tigr.tigr_run(vgu, run_algo, rec.source, stream=s, return_stats=True,
                                              frontier=front, schedule=sched)
                        times.append(st["ms_total"])
                    ms = statistics.median(times)
                    print(json.dumps({"cfg": args.cfg, "algo": algo, "variant": f"Tigr-UDT K={Ku}", "mode": mname,
                                      "K": Ku, "layout": "physical", "nodes": gu.info()["n"], "ms": ms,
                                      "speedup_vs_baseline": base_ms[mname] / ms,
                                      "iterations": st["iterations"]}), flush=True)
                vgu.free()
                gu.free()


if __name__ == "__main__":
    main()
