"""Device time of tigr_graph_transpose and tigr_graph_reorder on cfg4 (development tool)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402

rec = graphgen.recipe(os.environ.get("CFG", "cfg4"))
s = torch.cuda.current_stream()
g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=True, stream=s)
for name, fn in (("transpose", tigr.tigr_graph_transpose), ("reorder", tigr.tigr_graph_reorder)):
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        h = fn(g, stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        h.free()
    print(name, [round(t, 2) for t in ts], flush=True)
