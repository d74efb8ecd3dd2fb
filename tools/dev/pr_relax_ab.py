import sys, json, statistics, torch
sys.path.insert(0, '.')
import graphgen, paper_conf_asplos_sabetq018_b200 as tigr
rec = graphgen.recipe("cfg4")
s = torch.cuda.current_stream()
src = torch.empty(rec.m, dtype=torch.int32, device="cuda"); dst = torch.empty_like(src)
tigr.tigr_rmat_coo(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, 1, 64, src, dst, None, stream=s)
g = tigr.tigr_graph_from_coo(rec.n, src, dst, None, stream=s)
vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
out = torch.empty(rec.n, dtype=torch.float64, device="cuda")
ts, tt = [], []
for i in range(8):
    _, st = tigr.tigr_run(vg, "pr", out=out, stream=s, time_kernels=1, return_stats=True)
    ts.append(st["ms_relax"] / st["relax_launches"])
for i in range(8):  # whole 20-iteration runs without per-launch events
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    tigr.tigr_run(vg, "pr", out=out, stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    tt.append(e0.elapsed_time(e1))
print(json.dumps({"lib": tigr.LIB_PATH[-20:], "relax_ms_per_launch": statistics.median(ts[2:]),
                  "pr_run_ms": statistics.median(tt[2:]), "all": ts}))
