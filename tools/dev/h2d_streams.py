import torch, time
n = 268435456
hs = torch.empty(n, dtype=torch.int32).pin_memory(); hd = torch.empty(n, dtype=torch.int32).pin_memory()
ds = torch.empty(n, dtype=torch.int32, device="cuda"); dd = torch.empty_like(ds)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def one():
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s1)
    with torch.cuda.stream(s1):
        ds.copy_(hs, non_blocking=True); dd.copy_(hd, non_blocking=True)
    e1.record(s1); torch.cuda.synchronize(); return e0.elapsed_time(e1)
def two():
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s1); s2.wait_event(e0)
    with torch.cuda.stream(s1): ds.copy_(hs, non_blocking=True)
    with torch.cuda.stream(s2): dd.copy_(hd, non_blocking=True)
    e2 = torch.cuda.Event(); e2.record(s2); s1.wait_event(e2)
    e1.record(s1); torch.cuda.synchronize(); return e0.elapsed_time(e1)
def chunked(k):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s1); s2.wait_event(e0)
    c = n // k
    for i in range(k):
        with torch.cuda.stream(s1): ds[i*c:(i+1)*c].copy_(hs[i*c:(i+1)*c], non_blocking=True)
        with torch.cuda.stream(s2): dd[i*c:(i+1)*c].copy_(hd[i*c:(i+1)*c], non_blocking=True)
    e2 = torch.cuda.Event(); e2.record(s2); s1.wait_event(e2)
    e1.record(s1); torch.cuda.synchronize(); return e0.elapsed_time(e1)
for f in (one, two, one, two):
    print(f.__name__, min(f() for _ in range(4)))
print("chunked16", min(chunked(16) for _ in range(4)))
