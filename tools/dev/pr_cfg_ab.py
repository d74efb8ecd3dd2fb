"""A/B of PageRank push relax kernel shapes (TIGR_PR_CFG) on cfg4 in one process: per-launch
relax ms (CUDA events) and max |x - x_ref| against the default shape.  Development tool; the
knob is read only by the -DTIGR_DEV_KNOBS build (TIGR_LIB=build/libtigr_dev.so)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402

cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["5", "0", "1", "6"]
rec = graphgen.recipe(os.environ.get("CFG", "cfg4"))
s = torch.cuda.current_stream()
g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False, stream=s)
vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
ref = None
for rep in range(2):
    for c in cfgs:
        os.environ["TIGR_PR_CFG"] = c
        out = torch.empty(rec.n, dtype=torch.float64, device="cuda")
        best = None
        for _ in range(3):
            _, st = tigr.tigr_run(vg, "pr", 0, out=out, stream=s, time_kernels=1, return_stats=True)
            ms = st["ms_relax"] / max(st["relax_launches"], 1)
            best = ms if best is None else min(best, ms)
        torch.cuda.synchronize()
        if ref is None:
            ref = out.clone()
        err = float((out - ref).abs().max())
        nerr = err * rec.n
        print(f"rep={rep} cfg={c} relax_ms={best:.4f} total_ms={st['ms_total']:.3f} max_abs_vs_cfg{cfgs[0]}={err:.3e} (n*err {nerr:.3e})", flush=True)
