"""A/B of the frontier relax's hot-value filter (development build, TIGR_FQ_HOT words per block).

    TIGR_LIB=build/libtigr_dev.so python tools/dev/hot_ab.py [--hot 0,8192,16384] [--reorder 0]

Every run's values are compared with the filter-off run (bit-exact), and the median device ms of
--reps runs (CUDA-graph loop) is printed per algorithm and setting."""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--algos", default="bfs,sssp,sswp,cc")
    ap.add_argument("--hot", default="0,8192,16384")
    ap.add_argument("--minb", default="")
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--reorder", type=int, default=0)
    ap.add_argument("--graph", type=int, default=1, help="use_graph (0: host loop, for ncu)")
    args = ap.parse_args()
    rec = graphgen.recipe(args.config)
    s = torch.cuda.current_stream()
    g = vg = None
    for algo in args.algos.split(","):
        sym = algo == "cc"
        if g is None or g.sym != sym:
            if vg is not None:
                vg.free(); g.free()
            g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                                     weighted=not sym, symmetrize=sym, stream=s)
            if args.reorder:
                g2 = tigr.tigr_graph_reorder(g, stream=s)
                g.free()
                g = g2
            g.sym = sym
            vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
        ref = None
        for hot in [int(h) for h in args.hot.split(",")]:
            for minb in (args.minb.split(",") if args.minb else [""]):
                os.environ["TIGR_FQ_HOT"] = str(hot)
                if minb:
                    os.environ["TIGR_FQ_HOTMINB"] = minb
                res = torch.empty(rec.n, dtype=torch.int32, device="cuda")
                tigr.tigr_run(vg, algo, 0, out=res, stream=s)
                torch.cuda.synchronize()
                if ref is None:
                    ref = res.clone()
                same = bool(torch.equal(res, ref))
                ts = []
                for _ in range(args.reps):
                    _, st = tigr.tigr_run(vg, algo, 0, out=res, stream=s, return_stats=True, use_graph=args.graph)
                    ts.append(st["ms_total"])
                _, st = tigr.tigr_run(vg, algo, 0, out=res, stream=s, return_stats=True, collect_stats=1)
                print(json.dumps({"algo": algo, "hot": hot, "minb": minb, "reorder": args.reorder,
                                  "ms": round(statistics.median(ts), 4), "ms_min": round(min(ts), 4),
                                  "exact": same, "edges": st["edges_processed"], "updates": st["updates"]}),
                      flush=True)


if __name__ == "__main__":
    main()
