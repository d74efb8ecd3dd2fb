"""Timing probe for config 5 on one B200 + the host oracle (development tool)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_asplos_sabetq018_b200 as tigr  # noqa: E402

rec = graphgen.recipe("cfg5")
t = time.time()
g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, weighted=True)
vg = tigr.tigr_virtualize(g, 8)
torch.cuda.synchronize()
print("gpu build weighted", time.time() - t, vg.info(), torch.cuda.mem_get_info(), flush=True)
for algo in ("bfs", "sssp"):
    t = time.time()
    out, st = tigr.tigr_run(vg, algo, 0, return_stats=True)
    print("gpu", algo, time.time() - t, st["ms_total"], st["iterations"], flush=True)
    np.save(f"/tmp/cfg5_{algo}.npy", out)
del vg, g
t = time.time()
gs = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False, symmetrize=True)
vgs = tigr.tigr_virtualize(gs, 8)
print("gpu build sym", time.time() - t, flush=True)
t = time.time()
out, st = tigr.tigr_run(vgs, "cc", return_stats=True)
print("gpu cc", time.time() - t, st["ms_total"], st["iterations"], flush=True)
np.save("/tmp/cfg5_cc.npy", out)
del vgs, gs
t = time.time()
src, dst, w = graphgen.generate(rec)
print("graphgen", time.time() - t, flush=True)
t = time.time()
o = oracle.csr_build(rec.n, src, dst, w)
print("oracle csr", time.time() - t, flush=True)
t = time.time()
b = oracle.bfs(o, 0)
print("oracle bfs", time.time() - t, np.array_equal(b, np.load("/tmp/cfg5_bfs.npy")), flush=True)
t = time.time()
c = oracle.cc(rec.n, src, dst)
print("oracle cc", time.time() - t, np.array_equal(c, np.load("/tmp/cfg5_cc.npy")), flush=True)
t = time.time()
d = oracle.sssp(o, 0)
print("oracle sssp", time.time() - t, np.array_equal(d, np.load("/tmp/cfg5_sssp.npy")), flush=True)
