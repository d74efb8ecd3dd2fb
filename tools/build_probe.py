"""CSR-build probe on a BASELINE config (default cfg4): the arc list is drawn on the device once,
then tigr_graph_from_coo runs `--reps` times (device-timed); with `--reps 0` it runs exactly
twice (one warm-up), for an ncu capture of the build kernels of the second build:

    ncu --set full -k regex:'k_onesweep|k_coo_scan|k_place|k_runs' -s <launches of one build> \\
        python tools/build_probe.py --reps 0
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
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--weighted", type=int, default=0)
    ap.add_argument("--sym", type=int, default=0)
    ap.add_argument("--host", type=int, default=0, help="pass the arc list as pinned host arrays")
    args = ap.parse_args()
    rec = graphgen.recipe(args.config)
    s = torch.cuda.current_stream()
    src = torch.empty(rec.m, dtype=torch.int32, device="cuda")
    dst, w = torch.empty_like(src), torch.empty_like(src)
    tigr.tigr_rmat_coo(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, w, stream=s)
    wt = w if args.weighted else None
    if args.host:  # host-input build: the copy-in is part of the timed call
        src, dst = src.cpu().pin_memory(), dst.cpu().pin_memory()
        wt = wt.cpu().pin_memory() if wt is not None else None
    reps = max(args.reps, 2)
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        g = tigr.tigr_graph_from_coo(rec.n, src, dst, wt, symmetrize=bool(args.sym), stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        g.free()
    print(json.dumps({"config": args.config, "weighted": args.weighted, "sym": args.sym, "host": args.host,
                      "build_ms_median": statistics.median(ts[1:]), "build_ms_min": min(ts[1:]), "all": ts}))


if __name__ == "__main__":
    main()
