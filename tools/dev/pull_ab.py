"""Pull PageRank on cfg4: relax ms per launch with and without the out-degree source order
(TIGR_PR_PULL_OID=0/1), and the max difference of the two results (development tool)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402

rec = graphgen.recipe("cfg4")
s = torch.cuda.current_stream()
g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False, stream=s)
gt = tigr.tigr_graph_transpose(g, stream=s)
g.free()
res = {}
for rep in range(2):
    for v in ("0", "1"):
        os.environ["TIGR_PR_PULL_OID"] = v
        vg = tigr.tigr_virtualize(gt, 8, "strided", stream=s)
        out = torch.empty(rec.n, dtype=torch.float64, device="cuda")
        best = None
        for _ in range(3):
            _, st = tigr.tigr_run(vg, "pr", 0, out=out, stream=s, time_kernels=1, return_stats=True)
            ms = st["ms_relax"] / max(st["relax_launches"], 1)
            best = ms if best is None else min(best, ms)
        torch.cuda.synchronize()
        res[v] = out.clone()
        print(f"rep={rep} oid={v} relax_ms={best:.4f} total_ms={st['ms_total']:.3f}", flush=True)
        vg.free()
print("max|oid1-oid0| =", float((res["1"] - res["0"]).abs().max()))
