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

The algorithmic byte model of every relax launch is computed inside libtigr
(tigr_stats.bytes_alg, run.cu), so the roofline fractions here and the library agree.
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

# Paper context (never the target): Tigr-V+ on an NVIDIA Quadro P4000 (Pascal,
# sm_61, CUDA 8), Table 4 runtimes (L1276-1310) and Fig. 13's average SSSP
# speedup over the same engine without the transformation (L1341-1367, L1398-1412).
PAPER_CONTEXT = {
    "gpu": "NVIDIA Quadro P4000 (Pascal GP104, sm_61, ~243 GB/s), CUDA 8.0 (PAPER.md L1244-1249)",
    "table4_tigr_v_plus_ms": {
        "source": "PAPER.md Table 4, L1276-1310 (real graphs; GTEPS = m / t is BASELINE.md's derivation)",
        "sssp_livejournal": {"ms": 62.21, "n": 4.0e6, "m": 69e6, "derived_gteps": 1.11},
        "sswp_livejournal": {"ms": 65.67, "n": 4.0e6, "m": 69e6, "derived_gteps": 1.05},
        "bfs_twitter": {"ms": 178.53, "n": 21e6, "m": 530e6, "derived_gteps": 2.97},
        "sssp_twitter": {"ms": 269.75, "n": 21e6, "m": 530e6, "derived_gteps": 1.96},
        "cc_twitter": {"ms": 573.53, "n": 21e6, "m": 530e6, "derived_gteps": 0.92},
        "pr_twitter": {"ms": 221.49, "n": 21e6, "m": 530e6, "derived_gteps_per_run": 2.39},
    },
    "fig13_sssp_speedup_over_no_transform": {"tigr_v_plus": 2.1, "tigr_v": 1.7, "tigr_udt": 1.2,
                                             "source": "PAPER.md Fig. 13, L1341-1367, L1398-1412"},
    "note": "context only: other GPU, real graphs; this build's own ablation is DESIGN.md §12",
}


def ablation_context():
    """This build's Fig. 13 analogue beside the paper's: cfg3 (LiveJournal-shaped) SSSP speedups
    of the virtual transformations over the untransformed engine, K = 8, from the committed
    ablation run (tools/ablation.py -> profiles/r02e_ablation_cfg3.jsonl)."""
    path = os.path.join(ROOT, "profiles", "r02e_ablation_cfg3.jsonl")
    want = {"Tigr-V+ K=8 strided": "tigr_v_plus", "Tigr-V K=8 consecutive": "tigr_v", "Tigr-UDT K=8": "tigr_udt"}
    out = {}
    try:
        for line in open(path):
            d = json.loads(line)
            if d.get("algo") == "sssp" and d.get("mode") == "worklist async" and d.get("variant") in want:
                out[want[d["variant"]]] = round(d["speedup_vs_baseline"], 2)
    except (OSError, ValueError):
        return None
    out["source"] = "profiles/r02e_ablation_cfg3.jsonl (tools/ablation.py, B200, same engine, cfg3 SSSP, K = 8)"
    return out


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
    ap.add_argument("--no-cfg5-multi", action="store_true", help="N > 1: skip the cfg5 BFS/SSSP/CC/SSWP leg")
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
class pinned_to_one_core:
    """`taskset -c 0` for the timed oracle call (SURVEY.md §8(d) "Oracle timing"): the calling
    thread is pinned to one core (core 0 when the process may use it) and restored after."""

    def __enter__(self):
        self.saved = os.sched_getaffinity(0)
        self.core = 0 if 0 in self.saved else min(self.saved)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.saved)
        return False


def cpu_pr_sample(src, dst, n, iters):
    """The oracle as it stands (single-threaded C power iteration) on the same workload: the
    arc list the GPU used -> oracle CSR (untimed) -> `iters` PageRank iterations (timed, pinned
    to one core)."""
    import oracle

    g = oracle.csr_build(n, src, dst)
    with pinned_to_one_core() as pin:
        t0 = time.perf_counter()
        oracle.pagerank(g, iters)
        dt = time.perf_counter() - t0
    return dt, pin.core


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
    with pinned_to_one_core() as pin:
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
                                   f"(oracle/oracle.c or_pagerank, single thread pinned to core {pin.core})",
                         "host": host_cpu()},
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
def peak_hbm():
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(peaks_path):
        return json.load(open(peaks_path))["hbm_gbs"], "MEASURED_PEAKS.json hbm_gbs (measured copy)"
    return 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"


def gather_ceiling():
    """Measured random 4-byte gather rates (G gathers/s) from tools/micro/gather_ceiling.cu
    (build/libmicro.so, built by build()): uniform indices into a 2 MB, 64 MB (L2-resident) and
    1 GB array.  The frontier relax kernels gather one 4-byte target value per processed arc."""
    import ctypes
    path = os.path.join(ROOT, "build", "libmicro.so")
    if not os.path.exists(path):
        return None
    lib = ctypes.CDLL(path)
    lib.micro_gather.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int, ctypes.POINTER(ctypes.c_double)]
    lib.micro_gather.restype = ctypes.c_int
    out = {"source": "tools/micro/gather_ceiling.cu: uniform random u32 gathers, 8 in flight per thread, "
                     "148 x 8 blocks of 256 threads, best of 5"}
    gathers = 1 << 30
    for name, nbytes in (("l1_2MB", 2 << 20), ("l2_64MB", 64 << 20), ("hbm_1GB", 1 << 30)):
        ms = ctypes.c_double()
        rc = lib.micro_gather(nbytes // 4, gathers, 5, ctypes.byref(ms))
        out[name + "_ggather_s"] = gathers / (ms.value * 1e-3) / 1e9 if rc == 0 else None
    return out


def red_ceiling(n_elems, reds):
    """Best-of-5 ms for `reds` uniform random float64 REDs into an n_elems array
    (tools/micro/gather_ceiling.cu micro_red), or None."""
    import ctypes
    path = os.path.join(ROOT, "build", "libmicro.so")
    if not os.path.exists(path) or n_elems == 0:
        return None
    lib = ctypes.CDLL(path)
    if not hasattr(lib, "micro_red"):
        return None
    lib.micro_red.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int, ctypes.POINTER(ctypes.c_double)]
    lib.micro_red.restype = ctypes.c_int
    ms = ctypes.c_double()
    return ms.value if lib.micro_red(n_elems, reds, 5, ctypes.byref(ms)) == 0 else None


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
        comm = tigr.tigr_comm_init(world, rank, uid[0], device=local)
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
    cuts = None
    if comm is not None:  # each rank sorts only the arcs of its source range (arc-balanced cuts)
        cuts = tigr.tigr_coo_source_cuts(n, src, dst, world, stream=s)

    def one_step(src_t, dst_t, out_t, run_opts=opts):
        """a1 CSR build -> a2-a5 virtualize -> a6-a10 PageRank through the C ABI; returns
        per-phase events.  Host src_t / dst_t / out_t: the library copies the arc list in (in
        chunks, overlapped with its arc-list scan) and the ranks out, inside the call."""
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ev[0].record(s)
        if comm is None:
            g = tigr.tigr_graph_from_coo(n, src_t, dst_t, None, stream=s)
        else:
            g = tigr.tigr_graph_from_coo_part(n, src_t, dst_t, None, src_lo=int(cuts[rank]),
                                              src_hi=int(cuts[rank + 1]), stream=s)
        ev[1].record(s)
        vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
        ev[2].record(s)
        _, st = tigr.tigr_run(vg, "pr", 0, opts=run_opts, out=out_t, return_stats=True)
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

    clocks = ClockSampler(local, gpu_uuid(torch, local))
    clocks.start()
    l0 = tigr.tigr_launch_count()
    step_ms, phase, relax_ms, relax_launches, relax_bytes, nv = [], [[], [], []], 0.0, 0, 0, 0
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
        relax_bytes += st["bytes_alg"]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = tigr.tigr_launch_count() - l0
    clk = clocks.stop()

    t_step = allmax(sum(step_ms) / len(step_ms))
    gteps = 20 * m / (t_step * 1e-3) / 1e9

    # roofline of the dominant kernel (PR relax): the library's algorithmic bytes of the relax
    # launches (tigr_stats.bytes_alg) / their live CUDA-event durations in the timed region
    relax_avg_ms = relax_ms / max(relax_launches, 1)
    bytes_launch = relax_bytes / max(relax_launches, 1)
    peak, peak_src = peak_hbm()
    achieved = bytes_launch / (relax_avg_ms * 1e-3) / 1e9
    # DRAM traffic of one launch from the committed ncu --set full capture: only for the
    # configuration it was captured on (one GPU, cfg4, K = 8, strided)
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "relax_pr_traffic.json")
    if world == 1 and args.config == "cfg4" and args.K == 8 and args.layout == "strided" and os.path.exists(tpath):
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
                     "byte_model": "tigr_stats.bytes_alg: per arc 20 (target 4 + f64 RED read+write 16), per "
                                   "virtual node 4, per node with arcs 20 (SURVEY.md §8(d); DESIGN.md §5)",
                     "peak_source": peak_src, "frac_vs_8000_GBps": achieved / 8000.0},
        "breakdown_ms": {"csr_build": statistics.mean(phase[0]), "virtualize": statistics.mean(phase[1]),
                         "pagerank_20it": statistics.mean(phase[2]), "relax_total": relax_ms / args.steps},
        "algo_gteps": 20 * m / (statistics.mean(phase[2]) * 1e-3) / 1e9,
        "nv": nv[0], "gpu_launches": launches, "clocks": clk,
        "paper_context": dict(PAPER_CONTEXT, fig13_analogue_this_build=ablation_context()),
    }
    if rec_note:
        result["note"] = rec_note

    # e2e through the C ABI with HOST buffers: every step passes the pinned host arc list to
    # tigr_graph_from_coo (the library copies it in, chunk by chunk, overlapped with its
    # arc-list scan) and receives the 20-iteration ranks in a pinned host array from tigr_run
    # (D2H inside the call); the timed region is the whole call sequence, per step.
    if not args.no_e2e and not args.profile:
        hsrc = src.cpu().pin_memory()
        hdst = dst.cpu().pin_memory()
        hout = torch.empty(n, dtype=torch.float64).pin_memory()
        e2e_opts = tigr.tigr_run_opts_default()
        e2e_opts.stream = s.cuda_stream
        if comm is not None:
            e2e_opts.comm = comm.ptr.value
        e2e = []
        one_step(hsrc, hdst, hout, e2e_opts)  # untimed warm-up of the host-input path
        for _ in range(max(3, min(args.steps, 5))):
            flush.fill_(1)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            one_step(hsrc, hdst, hout, e2e_opts)
            e1.record(s)
            torch.cuda.synchronize()
            e2e.append(e0.elapsed_time(e1))
        te = allmax(sum(e2e) / len(e2e))
        result["e2e"] = {"value": 20 * m / (te * 1e-3) / 1e9, "unit": "GTEPS", "ms_per_step": te,
                         "steps": len(e2e), "h2d_bytes_per_step": 2 * m * 4, "d2h_bytes_per_step": n * 8,
                         "path": "C ABI with host buffers: tigr_graph_from_coo(pinned host src/dst) -> "
                                 "tigr_virtualize -> tigr_run(out = pinned host array)",
                         "h2d_bound_ms": None}
        # the PCIe floor of this step: the H2D of the arc list alone (same pinned buffers)
        dbuf = torch.empty_like(src)
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        c0.record(s)
        dbuf.copy_(hsrc, non_blocking=True)
        dbuf.copy_(hdst, non_blocking=True)
        c1.record(s)
        torch.cuda.synchronize()
        result["e2e"]["h2d_bound_ms"] = c0.elapsed_time(c1)
        del dbuf
        # the dependency-chain floor of one serial step: PageRank needs the whole CSR, so after
        # the last arc lands at least the virtualisation, the 20 iterations (device-timed above)
        # and the D2H of the ranks must follow; only the CSR build can hide under the H2D
        c0.record(s)
        hout.copy_(out, non_blocking=True)
        c1.record(s)
        torch.cuda.synchronize()
        d2h_ms = c0.elapsed_time(c1)
        floor = result["e2e"]["h2d_bound_ms"] + statistics.mean(phase[1]) + statistics.mean(phase[2]) + d2h_ms
        result["e2e"]["d2h_ms"] = d2h_ms
        result["e2e"]["chain_floor_ms"] = floor
        result["e2e"]["frac_of_chain_floor"] = floor / te
        # Pipelined variant (context, not the e2e key): the same C-ABI calls with host buffers,
        # issued from two host threads on two streams -- a builder thread runs
        # tigr_graph_from_coo(host arcs) + tigr_virtualize for step i+1 while the main thread
        # runs tigr_run(step i, out = pinned host array).  Every step's H2D and D2H happen inside
        # the library calls, inside the timed region (device events from the builder stream's
        # first op to the run stream's last).  ctypes releases the GIL during each call.
        import queue as _queue
        ksteps = max(3, min(args.steps, 6))
        sb = torch.cuda.Stream()
        houts = [torch.empty(n, dtype=torch.float64).pin_memory() for _ in range(2)]
        q = _queue.Queue(maxsize=1)
        run_opts = tigr.tigr_run_opts_default()
        run_opts.stream = s.cuda_stream
        if comm is not None:
            run_opts.comm = comm.ptr.value
        err = []

        def builder(steps):
            try:
                for _ in range(steps):
                    if comm is None:
                        gb = tigr.tigr_graph_from_coo(n, hsrc, hdst, None, stream=sb)
                    else:
                        gb = tigr.tigr_graph_from_coo_part(n, hsrc, hdst, None, src_lo=int(cuts[rank]),
                                                           src_hi=int(cuts[rank + 1]), stream=sb)
                    q.put((gb, tigr.tigr_virtualize(gb, args.K, args.layout, stream=sb)))
            except Exception as ex:  # noqa: BLE001
                err.append(repr(ex))
                q.put(None)

        def pipeline(steps):
            th = threading.Thread(target=builder, args=(steps,))
            th.start()
            for i in range(steps):
                item = q.get()
                if item is None:
                    break
                gb, vgb = item
                tigr.tigr_run(vgb, "pr", 0, opts=run_opts, out=houts[i % 2])
                vgb.free()
                gb.free()
            th.join()

        pipeline(2)  # warm-up: the block cache then holds two steps' buffers
        flush.fill_(1)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record(sb)
        s.wait_event(p0)
        pipeline(ksteps)
        p1.record(s)
        torch.cuda.synchronize()
        if not err:
            tp = allmax(p0.elapsed_time(p1) / ksteps)
            result["e2e_pipelined"] = {
                "value": 20 * m / (tp * 1e-3) / 1e9, "unit": "GTEPS", "ms_per_step": tp, "steps": ksteps,
                "h2d_bytes_per_step": 2 * m * 4, "d2h_bytes_per_step": n * 8,
                "note": "context, not the e2e key: the e2e call sequence (C ABI, host buffers) from two host "
                        "threads on two streams -- step i+1's tigr_graph_from_coo + tigr_virtualize overlap step "
                        "i's tigr_run"}
        else:
            result["e2e_pipelined"] = {"error": err[0]}
        del houts

    if not args.no_extra and not args.profile and world == 1:
        # the PR relax against its own ceiling: the global float64 reductions one launch issues
        # (arcs missing the shared-memory hot table; tigr_vgraph_pr_profile) per second of the
        # live relax time, over the measured random-RED rate into an array of the accumulator's size
        g = tigr.tigr_graph_from_coo(n, src, dst, None, stream=s)
        vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
        prof = tigr.tigr_vgraph_pr_profile(vg, stream=s)
        vg.free()
        g.free()
        red_ms = red_ceiling(prof["n_in"], 1 << 30)
        ach = prof["global_reds"] / (relax_avg_ms * 1e-3) / 1e9
        ceil = (1 << 30) / (red_ms * 1e-3) / 1e9 if red_ms else None
        result["roofline"]["l2_red"] = {
            "arcs_per_launch": prof["arcs"], "global_reds_per_launch": prof["global_reds"],
            "hot_slots": prof["hot_slots"], "accumulator_entries": prof["n_in"],
            "achieved_gred_s": ach, "ceiling_gred_s": ceil, "frac": (ach / ceil) if ceil else None,
            "ceiling_source": "tools/micro/gather_ceiling.cu micro_red: uniform random float64 REDs into "
                              "n_in doubles, 8 per thread in flight, 148 x 8 blocks of 256, best of 5"}
        peak_g = gather_ceiling()
        result["gather_ceiling"] = peak_g
        result["per_algo"] = per_algo(tigr, torch, rec, args, s, peak, peak_g)

    if not args.no_extra and not args.profile and world > 1:
        result["per_algo_multi"] = {"cfg4": per_algo_multi(tigr, torch, dist, graphgen.recipe("cfg4"), args, s,
                                                           rank, world, allmax, comm)}
        if not args.no_cfg5_multi:
            result["per_algo_multi"]["cfg5"] = per_algo_multi(tigr, torch, dist, graphgen.recipe("cfg5"), args, s,
                                                              rank, world, allmax, comm)

    if not args.no_extra and not args.no_configs and not args.profile and world == 1:
        result["per_config"] = per_config(tigr, torch, s, peak)

    if rank == 0 and world == 1 and not args.no_cpu and not args.profile:
        hs = src.cpu().numpy().view(np.uint32)  # the device-drawn arc list the GPU ran on
        hd = dst.cpu().numpy().view(np.uint32)
        dt, core = cpu_pr_sample(hs, hd, n, 2)
        v = 2 * m / dt / 1e9
        result["cpu_baseline"] = {"value": v, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                                  "sample": "2 of the 20 PageRank iterations on the full cfg4 graph (the device-drawn "
                                            f"arc list), {dt:.1f} s; oracle/oracle.c or_pagerank, single thread "
                                            f"pinned to core {core}",
                                  "host": host_cpu()}
        # SURVEY §8(d)'s optional secondary baseline: OpenMP pull PageRank on all host cores (not
        # the oracle; tools/cpu_baseline/omp_pagerank.c, tested against the oracle in
        # tests/test_cpu_baseline.py).  A bounded sample: 5 of the 20 iterations, in-CSR build untimed.
        try:
            from tools import cpu_baseline
            its = 5
            _, mb, mi = cpu_baseline.omp_pagerank(n, hs, hd, its, 0.85, 0)
            result["cpu_baseline_multicore"] = {
                "value": its * m / (mi * 1e-3) / 1e9, "unit": "GTEPS", "cores": os.cpu_count(),
                "kind": "openmp pull PageRank (tools/cpu_baseline/omp_pagerank.c), not the oracle",
                "sample": f"{its} of the 20 PageRank iterations on the full cfg4 graph, {mi / 1e3:.1f} s "
                          f"(in-CSR build {mb / 1e3:.1f} s, untimed)"}
            lv, bb, br = cpu_baseline.omp_bfs(n, hs, hd, 0, 0)  # the per_algo BFS graph's arcs, source 0
            reach = int(np.bincount(hs, minlength=n)[lv != 0xFFFFFFFF].sum())
            result["cpu_baseline_multicore"]["bfs"] = {
                "gteps_input": reach / (br * 1e-3) / 1e9, "ms": br, "levels": int(lv[lv != 0xFFFFFFFF].max()) + 1,
                "kind": "level-synchronous OpenMP BFS from vertex 0 (out-CSR build untimed)"}
        except (OSError, MemoryError) as e:
            result["cpu_baseline_multicore"] = {"error": str(e)}
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


def frontier_graph(tigr, torch, rec, sym, s):
    """cfg graph for BFS/SSSP/SSWP (weighted) or CC (symmetrised), drawn on the device, plus the
    out-degrees of the drawn arc list (input-normalised GTEPS count the arcs of reached nodes)."""
    src = torch.empty(rec.m, dtype=torch.int32, device="cuda")
    dst, w = torch.empty_like(src), torch.empty_like(src)
    tigr.tigr_rmat_coo(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, src, dst, w,
                       stream=s)
    deg = torch.bincount(src.long(), minlength=rec.n)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, None if sym else w, symmetrize=sym, stream=s)
    del src, dst, w
    torch.cuda.synchronize()
    return g, deg


def input_arcs(algo, out, deg, m):
    """arcs out of reached nodes (CC: all 2m arcs of the symmetrised graph)."""
    if algo == "cc":
        return 2 * m
    reached = out != (0 if algo == "sswp" else -1)
    return int(deg[reached].sum().item())


def per_algo_multi(tigr, torch, dist, rec, args, s, rank, world, allmax, comm):
    """N > 1: BFS / SSSP / SSWP / CC on `rec` (cfg4, and BASELINE configs[4] = cfg5) across the
    ranks.  Every rank holds the whole graph and relaxes its arc-balanced, family-aligned virtual
    node range (tigr_vgraph_partition); after each relax the replicated values are merged by the
    communicator: the dense in-place MIN/MAX all-reduce (NCCL ncclAllReduce; BASELINE configs[4]
    "NCCL min-allreduce"), the sparse exchange of changed nodes, AUTO (per iteration), and --
    through a node communicator (CUDA IPC) -- the fused exchange.  time = max over ranks of the
    device time of the run (median of 3); matches_single_gpu_all_ranks: every rank's values equal
    a one-GPU run of the same graph.  Failures are recorded, not raised, once every rank has
    reached the same point."""
    import graphgen

    n, m = rec.n, rec.m
    res = {"config": rec.name, "n": n, "m": m, "partition": "vnode ranges (tigr_vgraph_partition)",
           "transport": "nccl" if args.transport == "nccl" else "node (CUDA IPC + shared memory)"}
    # fused needs peer memory: the node communicator (probe first, with a short barrier timeout,
    # so a box without shared memory / CUDA IPC skips it on every rank within seconds)
    fcomm = comm if args.transport == "node" else None
    if fcomm is None:
        saved = os.environ.get("TIGR_GROUP_TIMEOUT")
        os.environ["TIGR_GROUP_TIMEOUT"] = "30"
        err = None
        try:
            fcomm = tigr.tigr_comm_init_node(job_name(f"frontier_{rec.name}"), world, rank)
            small = graphgen.recipe("cfg1")
            gs = tigr.tigr_graph_rmat(small.n, small.m, small.a, small.b, small.c, small.seed, small.wseed, stream=s)
            vgs = tigr.tigr_virtualize(gs, args.K, args.layout, stream=s)
            tigr.tigr_vgraph_partition(vgs, world, rank)
            tigr.tigr_run(vgs, "sssp", 0, comm=fcomm, exchange="fused", stream=s)
            vgs.free()
            gs.free()
        except Exception as e:  # noqa: BLE001
            err = repr(e)
        if allmax(1.0 if err else 0.0) != 0.0:
            res["fused_error"] = err or "a peer rank failed the node-communicator probe"
            if fcomm is not None:
                fcomm.free()
            fcomm = None
        if saved is None:
            os.environ.pop("TIGR_GROUP_TIMEOUT", None)
        else:
            os.environ["TIGR_GROUP_TIMEOUT"] = saved
    modes = [("dense", comm), ("sparse", comm), ("auto", comm)] + ([("fused", fcomm)] if fcomm is not None else [])
    for algo in ("bfs", "sssp", "sswp", "cc"):
        sym = algo == "cc"
        entry = {}
        try:
            g, deg = frontier_graph(tigr, torch, rec, sym, s)
            vg1 = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
            ref = torch.empty(n, dtype=torch.int32, device="cuda")
            _, st1 = tigr.tigr_run(vg1, algo, rec.source, out=ref, stream=s, return_stats=True)
            vg1.free()
            entry["ms_single_gpu"] = st1["ms_total"]
            entry["m_input"] = input_arcs(algo, ref, deg, m)
            vg = tigr.tigr_virtualize(g, args.K, args.layout, stream=s)
            tigr.tigr_vgraph_partition(vg, world, rank)
            out = torch.empty(n, dtype=torch.int32, device="cuda")
            ok = True
            for mode, c in modes:
                ts = []
                for _ in range(3):
                    _, st = tigr.tigr_run(vg, algo, rec.source, out=out, comm=c, exchange=mode, stream=s,
                                          return_stats=True)
                    ts.append(st["ms_total"])
                torch.cuda.synchronize()
                entry[f"ms_rank_{mode}"] = statistics.median(ts)
                entry[f"iterations_{mode}"] = st["iterations"]
                ok = ok and bool(torch.equal(out, ref))
            entry["matches_single_gpu"] = ok
            vg.free()
            g.free()
            del deg
        except Exception as e:  # noqa: BLE001
            entry = {"error": repr(e)}
        row = {"matches_single_gpu_all_ranks": allmax(0.0 if entry.get("matches_single_gpu") else 1.0) == 0.0}
        m_in = allmax(float(entry.get("m_input", 0)))
        for mode, _ in modes:
            t = allmax(entry.get(f"ms_rank_{mode}", float("inf")))
            row[mode] = {"ms": t, "iterations": entry.get(f"iterations_{mode}"),
                         "gteps_input": m_in / (t * 1e-3) / 1e9 if t != float("inf") else None}
        if "ms_single_gpu" in entry:
            row["ms_single_gpu_rank"] = entry["ms_single_gpu"]
        if "error" in entry:
            row["error"] = entry["error"]
        res[algo] = row
        torch.cuda.synchronize()
    if fcomm is not None and fcomm is not comm:
        fcomm.free()
    return res


def per_algo(tigr, torch, rec, args, s, peak, gceil):
    """Algorithm-only GTEPS for BFS/SSSP/SSWP/CC on the same scale-24 graph (weights 1-64; CC on
    the symmetrised graph), device-timed, in canonical numbering (the main numbers) and, beside
    them, on the in-degree-reordered copy (tigr_graph_reorder; its one-off cost is reorder_ms).
    gteps_input = arcs out of reached vertices (CC: all 2m arcs) / time; gteps_processed = arcs
    of active virtual nodes (collect_stats) / time; roofline_frac = the library's algorithmic
    bytes (tigr_stats.bytes_alg) / relax-kernel time (CUDA events per relax
    launch) / measured HBM peak; gather_frac_l2 = processed arcs per second of relax time / the
    measured L2 random-gather ceiling (each processed arc gathers one 4-byte target value)."""
    res = {}
    n, m = rec.n, rec.m
    ceil_l2 = (gceil or {}).get("l2_64MB_ggather_s")

    def measure(vg, algo, deg):
        out = torch.empty(n, dtype=torch.int32, device="cuda")
        _, st = tigr.tigr_run(vg, algo, 0, out=out, stream=s, collect_stats=1, return_stats=True)
        times, relax = [], []
        for _ in range(3):
            _, st2 = tigr.tigr_run(vg, algo, 0, out=out, stream=s, return_stats=True)
            times.append(st2["ms_total"])
            _, st4 = tigr.tigr_run(vg, algo, 0, out=out, stream=s, return_stats=True, time_kernels=1)
            relax.append(st4["ms_relax"])
        t, t_relax = statistics.median(times), statistics.median(relax)
        m_in = input_arcs(algo, out, deg, m)
        r = {"ms": t, "ms_relax": t_relax, "iterations": st["iterations"],
             "queue_iterations": st["queue_iterations"], "gteps_input": m_in / (t * 1e-3) / 1e9,
             "gteps_processed": st["edges_processed"] / (t * 1e-3) / 1e9,
             "edges_processed": st["edges_processed"], "updates": st["updates"],
             "algorithmic_bytes": st["bytes_alg"],
             "roofline_frac": st["bytes_alg"] / (t_relax * 1e-3) / 1e9 / peak,
             "roofline_frac_whole_run": st["bytes_alg"] / (t * 1e-3) / 1e9 / peak}
        if ceil_l2:
            r["gather_frac_l2"] = st["edges_processed"] / (t_relax * 1e-3) / 1e9 / ceil_l2
            # L1 sector accesses per processed arc by the kernel's access pattern:
            # one target gather (BFS/CC: the settled-bit test, level reads it does not skip
            # uncounted) + one access per 8-arc span of each streamed array (col; SSSP/SSWP +wt)
            unit = 8 if args.K % 8 == 0 else (4 if args.K % 4 == 0 else 1)
            acc = 1.0 + (2.0 if algo in ("sssp", "sswp") else 1.0) / unit
            r["l1_accesses_per_arc_model"] = acc
            r["l1_access_frac_l2"] = r["gather_frac_l2"] * acc
        return r

    for algo in ("bfs", "sssp", "sswp", "cc"):
        sym = algo == "cc"
        gc, deg = frontier_graph(tigr, torch, rec, sym, s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        gr = tigr.tigr_graph_reorder(gc, stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        vgc = tigr.tigr_virtualize(gc, args.K, args.layout, stream=s)
        vgr = tigr.tigr_virtualize(gr, args.K, args.layout, stream=s)
        res[algo] = measure(vgc, algo, deg)
        res[algo]["reordered"] = measure(vgr, algo, deg)
        res[algo]["reordered"]["reorder_ms"] = e0.elapsed_time(e1)
        vgc.free()
        vgr.free()
        gc.free()
        gr.free()
        del deg
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
            nbytes = st["bytes_alg"]  # the library's byte model (collect_stats run)
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
