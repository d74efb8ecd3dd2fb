"""A/B of a development knob on the cfg4 PageRank run (default TIGR_PR_CFG): total and relax
ms, max |difference| of the results.  Knobs are read only by the -DTIGR_DEV_KNOBS build:
    TIGR_LIB=build/libtigr_dev.so python tools/dev/pr_env_ab.py [VAR] [v1,v2,...]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402

var = sys.argv[1] if len(sys.argv) > 1 else "TIGR_PR_CFG"
vals = sys.argv[2].split(",") if len(sys.argv) > 2 else ["5", "1"]
rec = graphgen.recipe("cfg4")
s = torch.cuda.current_stream()
g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False, stream=s)
vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
ref = None
for rep in range(2):
    for v in vals:
        os.environ[var] = v
        out = torch.empty(rec.n, dtype=torch.float64, device="cuda")
        tot, rel = [], []
        for _ in range(5):
            _, st = tigr.tigr_run(vg, "pr", 0, out=out, stream=s, return_stats=True)
            tot.append(st["ms_total"])
        for _ in range(2):
            _, st = tigr.tigr_run(vg, "pr", 0, out=out, stream=s, time_kernels=1, return_stats=True)
            rel.append(st["ms_relax"] / max(st["relax_launches"], 1))
        torch.cuda.synchronize()
        if ref is None:
            ref = out.clone()
        print(f"rep={rep} {var}={v} total_ms={sorted(tot)[2]:.3f} relax_ms={min(rel):.4f} "
              f"max|d|={float((out - ref).abs().max()):.2e}", flush=True)
