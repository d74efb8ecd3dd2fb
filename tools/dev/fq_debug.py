"""Debug: cfg1 parity per (K, layout, frontier, TIGR_FQ_MODE); prints mismatch counts."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import graphgen, oracle
import paper_conf_asplos_sabetq018_b200 as tigr
rec = graphgen.recipe("cfg1")
src, dst, w = graphgen.generate(rec)
o = oracle.csr_build(rec.n, src, dst, w)
want = {"bfs": oracle.bfs(o, 0), "sssp": oracle.sssp(o, 0), "sswp": oracle.sswp(o, 0)}
g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
for K in (8, 16, 32):
    for layout in ("consecutive", "strided"):
        vg = tigr.tigr_virtualize(g, K, layout)
        for fr in (1, 3, 0):
            for sched in (0, 1):
                for ug in (1, 0):
                    row = []
                    for a in ("bfs", "sssp", "sswp"):
                        got = tigr.tigr_run(vg, a, 0, frontier=fr, schedule=sched, use_graph=ug)
                        bad = np.nonzero(got != want[a])[0]
                        row.append(f"{a}:{len(bad)}" + (f"{bad[:3].tolist()} got {got[bad[:3]].tolist()} want {want[a][bad[:3]].tolist()}" if len(bad) else ""))
                    print(K, layout, "fr", fr, "sched", sched, "graph", ug, " ".join(row), flush=True)
