#!/usr/bin/env python3
"""Benchmark of the B200 Tigr hot path (driver contract: one JSON line on rank 0).

Workload (BASELINE.json configs[3]): R-MAT scale 24 (16,777,216 vertices,
268,435,456 arcs, Graph500 a/b/c), PageRank 20 iterations, degree bound K = 8, strided
(coalesced) layout.  One step = the whole hot path over the arc list resident in HBM:
CSR build (a1) -> virtual split + layout (a2-a5) -> init + 20 x (relax -> [all-reduce] ->
apply) (a6-a10).  value = 20 * m / step time (GTEPS, input-normalised; every arc is
processed every iteration).  The other configs are parity-test cases (tests/).

  python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--config cfg4]
Multi-GPU: torchrun --nproc-per-node N bench.py --gpus N ...  (vnode ranges, NCCL all-reduce).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

# Algorithmic bytes of the push relax (fixed before measurement; DESIGN.md
# "Roofline"): per processed arc s_e + s_v (read the target value) -- PageRank: s_e + 2 s_v
# (RED = read + write of acc[dst]); per virtual node 4 (vn_phys); per node with d > 0 the
# source value + its row_ptr pair (s_v + 8).  The PageRank relax runs with the apply fused in
# (pr.cu PrFuse): its source value is derived from the previous accumulator, so per node with
# d > 0 it reads acc_prev[cid[v]] (8) + cid[v] (4) + the row pair (8) instead of contrib (8) +
# the row pair.
S_E = 4


def relax_bytes_pr(m, nv, n_out, fused=True):
    return m * (S_E + 16) + nv * 4 + n_out * ((8 + 4 + 8) if fused else (8 + 8))


def pr_apply_bytes(n):
    return n * 28


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="tigr", choices=["tigr", "reference"])
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--K", type=int, default=8)
    ap.add_argument("--layout", default="strided", choices=["strided", "consecutive"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-extra", action="store_true", help="skip the per-algorithm extras")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no extras, no e2e)")
    ap.add_argument("--no-configs", action="store_true", help="skip the other BASELINE configs (per_config)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "node"],
                    help="N > 1: PageRank exchange over NCCL (default) or the node communicator (CUDA IPC + "
                         "shared memory; torch.distributed on gloo; ranks may share a GPU -- for testing)")
    return ap.parse_args()


# ------------------------------------------------------------------------------------------ clocks
def gpu_uuid(torch, dev):
    try:
        u = str(torch.cuda.get_device_properties(dev).uuid)
        return u if u.startswith("GPU-") else "GPU-" + u
    except Exception:
        return None


class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region: an NVML thread polling every
    10 ms (no process start-up lag, so even a short timed region gets samples); nvidia-smi
    -lms 100 when NVML is unavailable."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index, uuid=None):
        self.index, self.uuid, self.rows, self.proc, self.nvml = index, uuid, [], None, None
        self.stop_flag = threading.Event()

    def start(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            try:
                h = nv.nvmlDeviceGetHandleByUUID(self.uuid) if self.uuid else None
            except nv.NVMLError:
                h = None
            self.h = h if h is not None else nv.nvmlDeviceGetHandleByIndex(self.index)
            self.nvml = nv
            self.max_sm = nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM)
            self.bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                         nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
            self._sample_nvml()
            self.rows.clear()
            self.thread = threading.Thread(target=self._poll_nvml, daemon=True)
            self.thread.start()
            return
        except Exception:
            self.nvml = None
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except OSError:
            self.proc = None

    def _sample_nvml(self):
        nv = self.nvml
        sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
        r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        self.rows.append([str(sm), str(self.max_sm), ""] + ["Active" if r & b else "Not Active" for b in self.bits])

    def _poll_nvml(self):
        while not self.stop_flag.is_set():
            try:
                self._sample_nvml()
            except Exception:
                return
            self.stop_flag.wait(0.01)

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def stop(self):
        src = "nvml 10 ms" if self.nvml else "nvidia-smi 100 ms"
        if self.nvml:
            self.stop_flag.set()
            self.thread.join(timeout=2)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        rows = list(self.rows)
        sms = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        reasons = sorted({self.NAMES[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows), "sampler": src}


# ------------------------------------------------------------------------------------------ reference arm
def cpu_pr_sample(rec, iters, threads_note=True):
    """The oracle as it stands (single-threaded C power iteration) on the same workload:
    host generator -> oracle CSR (untimed) -> `iters` PageRank iterations (timed)."""
    import graphgen
    import oracle

    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = oracle.csr_build(rec.n, src, dst)
    del src, dst
    t0 = time.perf_counter()
    oracle.pagerank(g, iters)
    dt = time.perf_counter() - t0
    return dt, g


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle timed on the box's host cores (rank 0 only)."""
    import graphgen
    import oracle

    if rank != 0:
        return
    rec = graphgen.recipe(args.config)
    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = oracle.csr_build(rec.n, src, dst)
    del src, dst
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.pagerank(g, 1)  # one power iteration per step: a bounded sample of the 20-iteration run
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    t = sum(times) / len(times)
    val = rec.m / t / 1e9
    print(json.dumps({
        "impl": "reference", "metric": metric_name(args), "value": val, "unit": "GTEPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_obj(args, rec),
        "cpu_baseline": {"value": val, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                         "sample": "1 of the 20 PageRank iterations per step on the full cfg4 graph "
                                   "(oracle/oracle.c or_pagerank, single thread)", "host": host_cpu()},
        "e2e": {"value": val, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def host_cpu():
    """'<model>, <N> logical cores' of this host (the oracle uses 1 of them)."""
    model = "unknown CPU"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return f"{model}, {os.cpu_count()} logical cores (oracle on 1)"


def metric_name(args):
    return "GTEPS per algorithm at 1/2/4/8 B200; % of HBM roofline; vs CPU oracle"


def config_obj(args, rec):
    return {"workload": f"{args.config}: R-MAT n={rec.n:,} m={rec.m:,} (a,b,c)=({rec.a},{rec.b},{rec.c}) "
                        f"PageRank 20 iterations, K={args.K}, {args.layout} layout",
            "algorithm": "pagerank", "K": args.K, "layout": args.layout, "n": rec.n, "m": rec.m,
            "parallelism": ("source-range partitioned CSR build per rank (arc-balanced cuts) + "
                            + ("NCCL all-reduce" if args.transport == "nccl" else
                               "peer-memory reduce-scatter/all-gather (node communicator)")
                            + " of the PageRank accumulator each iteration") if args.gpus > 1 else "single GPU",
            "l2": "flushed between steps (512 MiB write outside the timed events); arc list 2.1 GB > L2"}


# ------------------------------------------------------------------------------------------ main arm
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist

    import graphgen
    import paper_conf_asplos_sabetq018_b200 as tigr

    local = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(local)
    comm = None
    if world > 1 and args.transport == "nccl":
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        uid = [tigr.tigr_comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        comm = tigr.tigr_comm_init(world, rank, uid[0])
    elif world > 1:
        dist.init_process_group("gloo")
        comm = tigr.tigr_comm_init_node(job_name("pr"), world, rank)

    def allmax(x):
        """max over ranks of a host float (device tensor for NCCL, host tensor for gloo)."""
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda" if args.transport == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    rec = graphgen.recipe(args.config)
    n, m = rec.n, rec.m
    s = torch.cuda.current_stream()
    # inputs resident in HBM: the arc list, drawn on the device (counter-based; identical on every rank)
    src = torch.empty(m, dtype=torch.int32, device="cuda")
    dst = torch.empty_like(src)
    tigr.tigr_rmat_coo(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, None, stream=s)
    out = torch.empty(n, dtype=torch.float64, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    opts = tigr.tigr_run_opts_default()
    opts.stream = s.cuda_stream
    opts.time_kernels = 1
    if comm is not None:
        opts.comm = comm.ptr.value

    def one_step(src_t, dst_t, out_t, host=False):
        """a1 CSR build -> a2-a5 virtualize -> a6-a10 PageRank; returns per-phase events."""
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ev[0].record(s)
        if comm is None:
            g = tigr.tigr_graph_from_coo(n, src_t, dst_t, None, stream=s)
        else:  # e: each rank sorts only the arcs of its source range (arc-balanced cuts)
            cuts = tigr.tigr_coo_source_cuts(n, src_t, dst_t, world, stream=s)
            g = tigr.tigr_graph_from_coo_part(n, src_t, dst_t, None, src_lo=int(cuts[rank]),
                                              src_hi=int(cuts[rank + 1]), stream=s)
        ev[1].record(s)
        vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
        ev[2].record(s)
        _, st = tigr.tigr_run(vg, "pr", 0, opts=opts, out=out_t, return_stats=True)
        ev[3].record(s)
        vi = vg.info()
        nv = (vi["hi"] - vi["lo"], g.info()["m"])  # this rank's virtual nodes and arcs
        vg.free()
        g.free()
        return ev, st, nv

    # warm-up (W >= 3 by contract)
    for _ in range(max(args.warmup, 0)):
        one_step(src, dst, out)
    torch.cuda.synchronize()

    deg_t = torch.bincount(src, minlength=n)
    n_out = int(torch.count_nonzero(deg_t).item())
    clocks = ClockSampler(local, gpu_uuid(torch, local))
    clocks.start()
    l0 = tigr.tigr_launch_count()
    step_ms, phase, relax_ms, relax_launches, nv = [], [[], [], []], 0.0, 0, 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for _ in range(args.steps):
        flush.fill_(1)  # L2 flush outside the timed events
        ev, st, nv = one_step(src, dst, out)
        torch.cuda.synchronize()
        step_ms.append(ev[0].elapsed_time(ev[3]))
        for i in range(3):
            phase[i].append(ev[i].elapsed_time(ev[i + 1]))
        relax_ms += st["ms_relax"]
        relax_launches += st["relax_launches"]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = tigr.tigr_launch_count() - l0
    clk = clocks.stop()

    t_step = allmax(sum(step_ms) / len(step_ms))
    gteps = 20 * m / (t_step * 1e-3) / 1e9

    # roofline of the dominant kernel (PR relax), live CUDA-event durations from the timed region
    relax_avg_ms = relax_ms / max(relax_launches, 1)
    my_nv, my_m = nv
    bytes_launch = relax_bytes_pr(my_m, my_nv, n_out // world if world > 1 else n_out)
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(peaks_path):
        peak = json.load(open(peaks_path))["hbm_gbs"]
        peak_src = "MEASURED_PEAKS.json hbm_gbs (measured copy)"
    else:
        peak, peak_src = 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"
    achieved = bytes_launch / (relax_avg_ms * 1e-3) / 1e9
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "relax_pr_traffic.json")
    if os.path.exists(tpath):
        traffic = json.load(open(tpath)).get("dram_bytes_per_launch")

    if world > torch.cuda.device_count():
        rec_note = f"{world} ranks share {torch.cuda.device_count()} GPU(s): a protocol test, not a scaling number"
    else:
        rec_note = None
    result = {
        "metric": metric_name(args), "value": gteps, "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_step, "ms_per_step_median": statistics.median(step_ms),
        "ms_per_step_min": min(step_ms), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_obj(args, rec),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic,
                     "kernel": "k_relax_pr_cid (PageRank push relax with the apply fused in, pr.cu)",
                     "algorithmic_bytes_per_launch": bytes_launch, "avg_launch_ms": relax_avg_ms,
                     "peak_source": peak_src, "frac_vs_8000_GBps": achieved / 8000.0},
        "breakdown_ms": {"csr_build": statistics.mean(phase[0]), "virtualize": statistics.mean(phase[1]),
                         "pagerank_20it": statistics.mean(phase[2]), "relax_total": relax_ms / args.steps},
        "algo_gteps": 20 * m / (statistics.mean(phase[2]) * 1e-3) / 1e9,
        "nv": my_nv, "gpu_launches": launches, "clocks": clk,
    }
    if rec_note:
        result["note"] = rec_note

    # e2e through the public API with HOST buffers (pinned), H2D and D2H inside the timed region
    if not args.no_e2e and not args.profile:
        hsrc = src.cpu().pin_memory()
        hdst = dst.cpu().pin_memory()
        hout = torch.empty(n, dtype=torch.float64).pin_memory()
        e2e = []
        for _ in range(max(1, min(args.steps, 5))):
            flush.fill_(1)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            one_step(hsrc, hdst, hout)
            e1.record(s)
            torch.cuda.synchronize()
            e2e.append(e0.elapsed_time(e1))
        te = allmax(sum(e2e) / len(e2e))
        # Pipelined variant: step i+1's arc list is copied in on one copy stream and step i-1's
        # ranks are read back on another while step i computes -- the same public API on
        # device buffers, every step's H2D and D2H inside the timed region (first copy to
        # last readback).
        ksteps = max(2, min(args.steps, 6))
        cs = torch.cuda.Stream()
        rs = torch.cuda.Stream()
        dbuf = [(torch.empty_like(src), torch.empty_like(dst)) for _ in range(2)]
        dres = [torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(2)]
        hres = [torch.empty(n, dtype=torch.float64).pin_memory() for _ in range(2)]
        copied = [torch.cuda.Event() for _ in range(2)]
        freed = [torch.cuda.Event() for _ in range(2)]
        read = [torch.cuda.Event() for _ in range(2)]
        flush.fill_(1)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record(s)
        cs.wait_event(p0)

        def h2d(i):
            b = i % 2
            with torch.cuda.stream(cs):
                if i >= 2:
                    cs.wait_event(freed[b])
                dbuf[b][0].copy_(hsrc, non_blocking=True)
                dbuf[b][1].copy_(hdst, non_blocking=True)
                copied[b].record(cs)

        h2d(0)
        for i in range(ksteps):
            b = i % 2
            if i + 1 < ksteps:
                h2d(i + 1)
            s.wait_event(copied[b])
            if i >= 2:
                s.wait_event(read[b])  # step i-2's ranks have left dres[b]
            one_step(dbuf[b][0], dbuf[b][1], dres[b])
            freed[b].record(s)
            with torch.cuda.stream(rs):  # read the ranks back while the next step computes
                rs.wait_event(freed[b])
                hres[b].copy_(dres[b], non_blocking=True)
                read[b].record(rs)
        s.wait_stream(rs)
        p1.record(s)
        torch.cuda.synchronize()
        tp = allmax(p0.elapsed_time(p1) / ksteps)
        # e2e = the pipelined run (what a user streaming batches gets; every step's H2D and
        # D2H are inside the timed region); the unpipelined one is reported beside it
        result["e2e"] = {"value": 20 * m / (tp * 1e-3) / 1e9, "unit": "GTEPS", "ms_per_step": tp,
                         "steps": ksteps, "h2d_bytes_per_step": 2 * m * 4, "d2h_bytes_per_step": n * 8,
                         "note": "H2D of step i+1 (pinned host arc list) and D2H of step i-1's ranks (to "
                                 "pinned host memory) on two copy streams, overlapped with step i"}
        result["e2e_serial"] = {"value": 20 * m / (te * 1e-3) / 1e9, "unit": "GTEPS", "ms_per_step": te,
                                "h2d_bytes_per_step": 2 * m * 4, "d2h_bytes_per_step": n * 8,
                                "note": "H2D -> step -> D2H with nothing overlapped"}

    if not args.no_extra and not args.profile and world == 1:
        result["per_algo"] = per_algo(tigr, torch, rec, args, s, deg_t.cpu().numpy(), peak)

    if not args.no_extra and not args.profile and world > 1:
        result["per_algo_multi"] = per_algo_multi(tigr, torch, dist, rec, args, s, rank, world, allmax)

    if not args.no_extra and not args.no_configs and not args.profile and world == 1:
        result["per_config"] = per_config(tigr, torch, s, peak)

    if rank == 0 and world == 1 and not args.no_cpu and not args.profile:
        dt, _ = cpu_pr_sample(rec, 2)
        v = 2 * m / dt / 1e9
        result["cpu_baseline"] = {"value": v, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                                  "sample": "2 of the 20 PageRank iterations on the full cfg4 graph "
                                            f"({dt:.1f} s; oracle/oracle.c or_pagerank, single thread)",
                                  "host": host_cpu()}
    if rank == 0:
        print(json.dumps(result), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


_JOB_TOKEN = []


def job_name(tag):
    """A name unique to this job (node communicator shared-memory segment): rank 0 draws a
    random token and broadcasts it, so no rank can attach to a stale segment of another run."""
    import torch.distributed as dist
    if not _JOB_TOKEN:
        import uuid
        tok = [uuid.uuid4().hex[:16] if dist.get_rank() == 0 else None]
        dist.broadcast_object_list(tok, src=0)
        _JOB_TOKEN.append(tok[0])
    return f"bench_{tag}_{_JOB_TOKEN[0]}"


def per_algo_multi(tigr, torch, dist, rec, args, s, rank, world, allmax):
    import graphgen
    """N > 1: BFS / SSSP / CC on the scale-24 graph across the ranks with the FUSED exchange
    (the relax applies each improvement to every peer replica over NVLink; node communicator,
    CUDA IPC) -- the multi-GPU frontier path.  Every rank holds the whole graph and relaxes its
    arc-balanced virtual node range; time = max over ranks of the device time of the run;
    matches_single_gpu: every rank's values equal a one-GPU run of the same graph on its GPU.
    Failures are recorded, not raised, after every rank has reached the same point."""
    n, m = rec.n, rec.m
    res = {"exchange": "fused", "transport": "node (CUDA IPC + shared memory)"}
    # probe first, with a short barrier timeout: if shared memory or CUDA IPC is unavailable
    # here, every rank learns it within seconds and the section is skipped on all of them
    os.environ["TIGR_GROUP_TIMEOUT"] = "30"
    comm, err = None, None
    try:
        comm = tigr.tigr_comm_init_node(job_name("frontier"), world, rank)
        small = graphgen.recipe("cfg1")
        gs = tigr.tigr_graph_rmat(small.n, small.m, small.a, small.b, small.c, small.seed, small.wseed,
                                  stream=s)
        vgs = tigr.tigr_virtualize(gs, args.K, args.layout, stream=s)
        tigr.tigr_vgraph_partition(vgs, world, rank)
        tigr.tigr_run(vgs, "sssp", 0, comm=comm, exchange="fused", stream=s)
        tigr.tigr_run(vgs, "sssp", 0, comm=comm, exchange="sparse", stream=s)
        vgs.free()
        gs.free()
    except Exception as e:
        err = repr(e)
    if allmax(1.0 if err else 0.0) != 0.0:
        res["error"] = err or "a peer rank failed the node-communicator probe"
        return res
    os.environ["TIGR_GROUP_TIMEOUT"] = "120"
    for algo in ("bfs", "sssp", "cc"):
        sym = algo == "cc"
        entry = {}
        try:
            g = tigr.tigr_graph_rmat(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                                     weighted=not sym, symmetrize=sym, stream=s)
            vg1 = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
            ref = torch.empty(n, dtype=torch.int32, device="cuda")
            tigr.tigr_run(vg1, algo, 0, out=ref, stream=s)
            vg1.free()
            vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
            tigr.tigr_vgraph_partition(vg, world, rank)
            out = torch.empty(n, dtype=torch.int32, device="cuda")
            ts = []
            for _ in range(3):
                _, st = tigr.tigr_run(vg, algo, 0, out=out, comm=comm, exchange="fused", stream=s,
                                      return_stats=True)
                ts.append(st["ms_total"])
            torch.cuda.synchronize()
            entry = {"ms_rank": statistics.median(ts), "iterations": st["iterations"],
                     "matches_single_gpu": bool(torch.equal(out, ref))}
            for mode in ("sparse", "dense"):  # the other exchanges, for comparison
                tm = []
                for _ in range(3):
                    _, stm = tigr.tigr_run(vg, algo, 0, out=out, comm=comm, exchange=mode, stream=s,
                                           return_stats=True)
                    tm.append(stm["ms_total"])
                torch.cuda.synchronize()
                entry[f"ms_rank_{mode}"] = statistics.median(tm)
                entry["matches_single_gpu"] = entry["matches_single_gpu"] and bool(torch.equal(out, ref))
            vg.free()
            g.free()
        except Exception as e:
            entry = {"error": repr(e)}
        t = allmax(entry.get("ms_rank", float("inf")))
        for mode in ("sparse", "dense"):
            if f"ms_rank_{mode}" in entry or "error" in entry:
                entry[f"ms_{mode}"] = allmax(entry.pop(f"ms_rank_{mode}", float("inf")))
        ok = allmax(0.0 if entry.get("matches_single_gpu") else 1.0) == 0.0
        m_arcs = 2 * m if sym else m
        res[algo] = {"ms": t, "gteps_arcs": m_arcs / (t * 1e-3) / 1e9 if t != float("inf") else None,
                     "matches_single_gpu_all_ranks": ok, **{k: v for k, v in entry.items() if k != "ms_rank"}}
    comm.free()
    return res


def frontier_bytes(algo, st, n):
    """Algorithmic bytes of one frontier run: per processed arc
    s_e (+4 B weight for SSSP/SSWP) + 4 B target-value read; per successful update 4 B; per
    active virtual node 4 B; per active node with arcs 12 B (value + row pair); per iteration
    2 B per node (frontier flags read + cleared)."""
    s_e = S_E + (4 if algo in ("sssp", "sswp") else 0)
    return (st["edges_processed"] * (s_e + 4) + st["updates"] * 4 + st["active_vnodes"] * 4
            + st["active_nodes"] * 12 + st["iterations"] * 2 * n)


def per_algo(tigr, torch, rec, args, s, deg, peak):
    """Algorithm-only GTEPS for BFS/SSSP/CC/SSWP on the same scale-24 graph (weights 1-64;
    CC on the symmetrised graph), device-timed, on the in-degree-reordered graph
    (tigr_graph_reorder; its one-off cost is reported as reorder_ms, like the virtual split's
    transform time) and, for comparison, in canonical numbering (ms_canonical).
    gteps_input = arcs out of reached vertices (CC: all 2m arcs) / time; gteps_processed =
    arcs of active virtual nodes (collect_stats) / time; roofline_frac = algorithmic bytes /
    relax-kernel time (CUDA events per relax launch) / measured HBM peak."""
    res = {}
    n, m = rec.n, rec.m
    g = vg = None
    for algo in ("bfs", "sssp", "sswp", "cc"):
        sym = algo == "cc"
        if g is None or sym:
            if g is not None:
                vg.free(); g.free(); vgc.free(); gc.free()
            gc = tigr.tigr_graph_rmat(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax,
                                      weighted=not sym, symmetrize=sym, stream=s)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            g = tigr.tigr_graph_reorder(gc, stream=s)
            e1.record(s)
            torch.cuda.synchronize()
            reorder_ms = e0.elapsed_time(e1)
            vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
            vgc = tigr.tigr_virtualize(gc, args.K, args.layout, stream=s)
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        _, st = tigr.tigr_run(vg, algo, 0, out=out, stream=s, collect_stats=1, return_stats=True)
        times, canon, relax = [], [], []
        for _ in range(3):
            _, st2 = tigr.tigr_run(vg, algo, 0, out=out, stream=s, return_stats=True)
            times.append(st2["ms_total"])
            _, st3 = tigr.tigr_run(vgc, algo, 0, out=out, stream=s, return_stats=True)
            canon.append(st3["ms_total"])
            _, st4 = tigr.tigr_run(vg, algo, 0, out=out, stream=s, return_stats=True, time_kernels=1)
            relax.append(st4["ms_relax"])
        t = statistics.median(times)
        t_relax = statistics.median(relax)
        if algo == "cc":
            m_in = 2 * m
        else:
            reached = out.cpu().numpy().view(np.uint32)
            mask = reached != (0 if algo == "sswp" else 0xFFFFFFFF)
            m_in = int(deg[mask].sum())
        nbytes = frontier_bytes(algo, st, n)
        res[algo] = {"ms": t, "ms_relax": t_relax, "ms_canonical": statistics.median(canon), "reorder_ms": reorder_ms,
                     "iterations": st["iterations"], "queue_iterations": st["queue_iterations"],
                     "gteps_input": m_in / (t * 1e-3) / 1e9,
                     "gteps_processed": st["edges_processed"] / (t * 1e-3) / 1e9,
                     "edges_processed": st["edges_processed"], "updates": st["updates"],
                     "algorithmic_bytes": nbytes,
                     "roofline_frac": nbytes / (t_relax * 1e-3) / 1e9 / peak,
                     "roofline_frac_whole_run": nbytes / (t * 1e-3) / 1e9 / peak}
    vg.free(); g.free(); vgc.free(); gc.free()
    # NEXT-1: pull PageRank on the in-CSR (same graph, 20 iterations), relax timed per launch
    g = tigr.tigr_graph_rmat(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False, stream=s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    gt = tigr.tigr_graph_transpose(g, stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    g.free()
    vgt = tigr.tigr_virtualize(gt, args.K, args.layout, stream=s)
    out64 = torch.empty(n, dtype=torch.float64, device="cuda")
    runs = []
    for _ in range(3):
        _, st = tigr.tigr_run(vgt, "pr", 0, out=out64, stream=s, time_kernels=1, return_stats=True)
        runs.append(st)
    best = min(runs, key=lambda d: d["ms_total"])
    relax_ms = best["ms_relax"] / max(best["relax_launches"], 1)
    res["pr_pull"] = {"ms_20it": best["ms_total"], "relax_ms_per_launch": relax_ms,
                      "gteps_20it": 20 * m / (best["ms_total"] * 1e-3) / 1e9,
                      "gteps_relax": m / (relax_ms * 1e-3) / 1e9, "transpose_ms": e0.elapsed_time(e1),
                      "note": "SURVEY NEXT-1: in-CSR via tigr_graph_transpose, warp-segmented family sums"}
    vgt.free()
    gt.free()
    return res


def per_config(tigr, torch, s, peak):
    """GTEPS per algorithm on the other BASELINE configs at one GPU (configs[1], [2], [4]; the
    scale-24 graph is the main line and per_algo): cfg2 BFS + CC, cfg3 SSSP + SSWP at K = 4, 8,
    16, 32, cfg5 BFS / SSSP / CC.  Arc list drawn on the device (tigr_rmat_coo), CSR built from
    it (build_ms), virtual split at K (strided), then per algorithm: one stats run
    (processed arcs), the median of 3 device-timed runs (CUDA-graph loop), and one run with
    per-relax CUDA events; then the median of 3 runs on the in-degree-reordered copy
    (tigr_graph_reorder, its one-off cost in reorder_ms; results in original ids).
    gteps_input = arcs out of reached nodes (CC: all 2m arcs) / time."""
    import graphgen

    plan = {"cfg2": [("bfs", 8), ("cc", 8)],
            "cfg3": [(a, K) for K in (4, 8, 16, 32) for a in ("sssp", "sswp")],
            "cfg5": [("bfs", 8), ("sssp", 8), ("cc", 8)]}
    res = {}
    for cfg, runs in plan.items():
        rec = graphgen.recipe(cfg)
        n, m = rec.n, rec.m
        src = torch.empty(m, dtype=torch.int32, device="cuda")
        dst, w = torch.empty_like(src), torch.empty_like(src)
        tigr.tigr_rmat_coo(n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, w, stream=s)
        deg = torch.bincount(src.long(), minlength=n)
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        entry = {"n": n, "m": m, "source": rec.source}
        graphs = {}
        for algo, K in runs:
            sym = algo == "cc"
            if sym not in graphs:
                for g in graphs.values():
                    g.free()
                graphs.clear()
                # one untimed build first: the block cache then holds buffers of these sizes
                tigr.tigr_graph_from_coo(n, src, dst, None if sym else w, symmetrize=sym, stream=s).free()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                graphs[sym] = tigr.tigr_graph_from_coo(n, src, dst, None if sym else w, symmetrize=sym, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                entry["build_ms_sym" if sym else "build_ms"] = e0.elapsed_time(e1)
                # the in-degree-reordered copy (one-off cost reported like the build)
                e0.record(s)
                graphs[(sym, "r")] = tigr.tigr_graph_reorder(graphs[sym], stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                entry["reorder_ms_sym" if sym else "reorder_ms"] = e0.elapsed_time(e1)
            vg = tigr.tigr_virtualize(graphs[sym], K, "strided", stream=s)
            _, st = tigr.tigr_run(vg, algo, rec.source, out=out, stream=s, collect_stats=1, return_stats=True)
            ts = []
            for _ in range(3):
                _, st2 = tigr.tigr_run(vg, algo, rec.source, out=out, stream=s, return_stats=True)
                ts.append(st2["ms_total"])
            _, st3 = tigr.tigr_run(vg, algo, rec.source, out=out, stream=s, return_stats=True, time_kernels=1)
            t = statistics.median(ts)
            if sym:
                m_in = 2 * m
            else:
                reached = out != (0 if algo == "sswp" else -1)
                m_in = int(deg[reached].sum().item())
            nbytes = frontier_bytes(algo, st, n)
            entry[f"{algo}_K{K}"] = {
                "ms": t, "ms_relax": st3["ms_relax"], "iterations": st["iterations"],
                "gteps_input": m_in / (t * 1e-3) / 1e9,
                "gteps_processed": st["edges_processed"] / (t * 1e-3) / 1e9,
                "roofline_frac": nbytes / (st3["ms_relax"] * 1e-3) / 1e9 / peak if st3["ms_relax"] else None,
                "nv": vg.info()["nv"]}
            vg.free()
            # same run on the reordered graph (values come back in original ids)
            vgr = tigr.tigr_virtualize(graphs[(sym, "r")], K, "strided", stream=s)
            tr = []
            for _ in range(3):
                _, st4 = tigr.tigr_run(vgr, algo, rec.source, out=out, stream=s, return_stats=True)
                tr.append(st4["ms_total"])
            tr_med = statistics.median(tr)
            entry[f"{algo}_K{K}"]["ms_reordered"] = tr_med
            entry[f"{algo}_K{K}"]["gteps_input_reordered"] = m_in / (tr_med * 1e-3) / 1e9
            vgr.free()
        for g in graphs.values():
            g.free()
        del src, dst, w, deg, out
        torch.cuda.synchronize()
        res[cfg] = entry
    return res


if __name__ == "__main__":
    main()
