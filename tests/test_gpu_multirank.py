"""Multi-rank runs on real kernels (§8(f) NEXT-2), on one GPU.

The ranks are threads of this process joined in a thread-group communicator
(tigr_comm_group_create / tigr_comm_init_group): every rank owns a contiguous, family-aligned
virtual node range (tigr_vgraph_partition) or a source range of the arc list
(tigr_graph_from_coo_part), relaxes only its own virtual nodes against its replica, and the
replicas are merged every iteration -- dense all-reduce, or the sparse exchange of changed
nodes.  Every rank must return the oracle's values: bit-exact for BFS/SSSP/SSWP/CC, PageRank
within 1e-6 and bit-identical across ranks (the group reduces in rank order).  The NCCL
transport runs the same protocol; with one GPU it is covered at one rank
(test_exchange_modes_single_rank_nccl)."""
import threading

import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tigr():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_asplos_sabetq018_b200 as t
    return t


def _graph(name):
    if name == "cfg1":
        rec = graphgen.recipe("cfg1")
        src, dst, w = graphgen.generate(rec)
        return rec.n, src, dst, w
    # scale 16 R-MAT (Graph500 parameters): deeper frontiers, lists of thousands of nodes
    n, m = 1 << 16, 1 << 20
    src, dst, w = graphgen.rmat(n, m, 0.57, 0.19, 0.19, 11, 12, 1, 64)
    return n, src, dst, w


_WANT = {}


def _want(name):
    if name not in _WANT:
        n, src, dst, w = _graph(name)
        o = oracle.csr_build(n, src, dst, w)
        _WANT[name] = {"bfs": oracle.bfs(o, 0), "sssp": oracle.sssp(o, 0), "sswp": oracle.sswp(o, 0),
                       "cc": oracle.cc(n, src, dst), "pr": oracle.pagerank(o, 20)}
    return _WANT[name]


def _run_group(tigr, P, body):
    """body(rank, comm, stream) on P threads (all on cuda:0); returns the per-rank results."""
    group = tigr.tigr_comm_group_create(P)
    out, errs = [None] * P, []

    def worker(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            comm = tigr.tigr_comm_init_group(group, r)
            out[r] = body(r, comm, s)
            torch.cuda.synchronize()
            comm.free()
        except Exception as e:  # pragma: no cover - reported below
            errs.append((r, repr(e)))

    th = [threading.Thread(target=worker, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    group.free()
    assert not errs, errs
    return out


def _check(want, res, algos=("bfs", "sssp", "sswp", "cc", "pr")):
    for rank, got in enumerate(res):
        for a in algos:
            if a == "pr":
                assert np.abs(got[a] - want[a]).max() <= 1e-6, (rank, a)
                assert np.array_equal(got[a], res[0][a]), ("pr replicas differ", rank)
            else:
                assert np.array_equal(got[a], want[a]), (rank, a)


@pytest.mark.parametrize("graph", ["cfg1", "s16"])
@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("exchange", ["dense", "sparse", "auto", "fused"])
def test_group_vnode_partition(tigr, graph, P, exchange):
    """Full graph on every rank, virtual node range per rank (tigr_vgraph_partition)."""
    n, src, dst, w = _graph(graph)
    want = _want(graph)

    def body(r, comm, s):
        g = tigr.tigr_graph_from_coo(n, src, dst, w, stream=s)
        gs = tigr.tigr_graph_from_coo(n, src, dst, None, symmetrize=True, stream=s)
        vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
        vgs = tigr.tigr_virtualize(gs, 8, "strided", stream=s)
        tigr.tigr_vgraph_partition(vg, P, r)
        tigr.tigr_vgraph_partition(vgs, P, r)
        res, stats = {}, {}
        for a in ("bfs", "sssp", "sswp"):
            res[a], stats[a] = tigr.tigr_run(vg, a, 0, comm=comm, exchange=exchange, stream=s, return_stats=True)
        res["cc"], stats["cc"] = tigr.tigr_run(vgs, "cc", comm=comm, exchange=exchange, stream=s, return_stats=True)
        res["pr"] = tigr.tigr_run(vg, "pr", comm=comm, stream=s)
        res["stats"] = stats
        return res

    res = _run_group(tigr, P, body)
    _check(want, res)
    for r in res:
        for a, st in r["stats"].items():
            assert st["iterations"] == res[0]["stats"][a]["iterations"]  # same termination on every rank
            if exchange in ("dense", "fused"):
                assert st["sparse_exchanges"] == 0
            elif exchange == "sparse":
                assert st["sparse_exchanges"] == st["iterations"], (a, st)


@pytest.mark.parametrize("P", [2, 4])
def test_group_source_partition_bsp_and_queue(tigr, P):
    """Arc-balanced source ranges (tigr_graph_from_coo_part): each rank holds only its arcs;
    BSP schedule and the queue frontier go through the same exchange."""
    n, src, dst, w = _graph("s16")
    want = _want("s16")
    cuts = tigr.tigr_coo_source_cuts(n, src, dst, P)
    cuts_sym = tigr.tigr_coo_source_cuts(n, src, dst, P, symmetrize=True)

    def body(r, comm, s):
        g = tigr.tigr_graph_from_coo_part(n, src, dst, w, src_lo=int(cuts[r]), src_hi=int(cuts[r + 1]), stream=s)
        gs = tigr.tigr_graph_from_coo_part(n, src, dst, None, symmetrize=True, src_lo=int(cuts_sym[r]),
                                           src_hi=int(cuts_sym[r + 1]), stream=s)
        vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
        vgs = tigr.tigr_virtualize(gs, 8, "strided", stream=s)
        res = {}
        for a in ("bfs", "sssp", "sswp"):
            res[a] = tigr.tigr_run(vg, a, 0, comm=comm, exchange="sparse", schedule=1, stream=s)
            q = tigr.tigr_run(vg, a, 0, comm=comm, exchange="auto", frontier=tigr.TIGR_FRONTIER_QUEUE, stream=s)
            assert np.array_equal(q, res[a]), a
            for sched in (0, 1):  # fused exchange, asynchronous and BSP
                fz = tigr.tigr_run(vg, a, 0, comm=comm, exchange="fused", schedule=sched, stream=s)
                assert np.array_equal(fz, res[a]), (a, sched)
        res["cc"] = tigr.tigr_run(vgs, "cc", comm=comm, exchange="sparse", stream=s)
        assert np.array_equal(tigr.tigr_run(vgs, "cc", comm=comm, exchange="fused", stream=s), res["cc"])
        res["pr"] = tigr.tigr_run(vg, "pr", comm=comm, stream=s)
        return res

    _check(want, _run_group(tigr, P, body))


def test_group_consecutive_layout_and_odd_K(tigr):
    """K = 3 (per-edge units) and the consecutive layout through the exchange."""
    n, src, dst, w = _graph("cfg1")
    want = _want("cfg1")

    def body(r, comm, s):
        out = {}
        for K, layout in ((3, "consecutive"), (5, "strided")):
            g = tigr.tigr_graph_from_coo(n, src, dst, w, stream=s)
            vg = tigr.tigr_virtualize(g, K, layout, stream=s)
            tigr.tigr_vgraph_partition(vg, 3, r)
            for a in ("bfs", "sssp", "sswp"):
                got = tigr.tigr_run(vg, a, 0, comm=comm, exchange="sparse", stream=s)
                assert np.array_equal(got, want[a]), (K, layout, a)
            with pytest.raises(tigr.TigrError) as e:  # fused needs the 16-byte-chunk relax (4 | K)
                tigr.tigr_run(vg, "bfs", 0, comm=comm, exchange="fused", stream=s)
            assert e.value.status == tigr.TIGR_EUNSUPPORTED
            out[K] = True
        return out

    _run_group(tigr, 3, body)


def test_group_errors(tigr):
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_comm_group_create(0)
    assert e.value.status == tigr.TIGR_EINVAL
    with pytest.raises(tigr.TigrError):
        tigr.tigr_comm_group_create(17)
    g = tigr.tigr_comm_group_create(1)
    with pytest.raises(tigr.TigrError):
        tigr.tigr_comm_init_group(g, 1)
    c = tigr.tigr_comm_init_group(g, 0)  # a one-rank group needs no peer
    with pytest.raises(tigr.TigrError):
        tigr.tigr_comm_init_group(g, 0)  # joined twice
    n, src, dst, w = _graph("cfg1")
    vg = tigr.tigr_virtualize(tigr.tigr_graph_from_coo(n, src, dst, w), 8)
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_run(vg, "bfs", 0, comm=c, exchange=7)
    assert e.value.status == tigr.TIGR_EINVAL
    assert np.array_equal(tigr.tigr_run(vg, "bfs", 0, comm=c, exchange="sparse"), _want("cfg1")["bfs"])
    c.free()
    g.free()


@pytest.mark.parametrize("exchange", ["dense", "sparse", "auto"])
def test_exchange_modes_single_rank_nccl(tigr, exchange):
    """The NCCL transport's sparse path (count all-gather, grouped broadcast, apply) at one rank."""
    n, src, dst, w = _graph("s16")
    want = _want("s16")
    comm = tigr.tigr_comm_init(1, 0, tigr.tigr_comm_unique_id())
    g = tigr.tigr_graph_from_coo(n, src, dst, w)
    gs = tigr.tigr_graph_from_coo(n, src, dst, None, symmetrize=True)
    vg = tigr.tigr_virtualize(g, 8)
    vgs = tigr.tigr_virtualize(gs, 8)
    for a in ("bfs", "sssp", "sswp"):
        got, st = tigr.tigr_run(vg, a, 0, comm=comm, exchange=exchange, return_stats=True)
        assert np.array_equal(got, want[a]), a
        if exchange == "sparse":
            assert st["sparse_exchanges"] == st["iterations"]
    assert np.array_equal(tigr.tigr_run(vgs, "cc", comm=comm, exchange=exchange), want["cc"])
    with pytest.raises(tigr.TigrError) as e:  # fused needs peer pointers: thread group only
        tigr.tigr_run(vg, "bfs", 0, comm=comm, exchange="fused")
    assert e.value.status == tigr.TIGR_EUNSUPPORTED
    comm.free()


@pytest.mark.slow
@pytest.mark.parametrize("exchange", ["sparse", "auto", "fused"])
def test_group_cfg2_full(tigr, exchange):
    """Config 2 at full size (R-MAT scale 20: 16.8 M arcs, 33.6 M symmetrised) on 4 ranks:
    BFS and CC bit-exact on every rank, plus SSSP through the source-range build."""
    rec = graphgen.recipe("cfg2")
    src, dst, w = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst, w)
    want = {"bfs": oracle.bfs(o, 0), "sssp": oracle.sssp(o, 0), "cc": oracle.cc(rec.n, src, dst)}
    P = 4
    cuts = tigr.tigr_coo_source_cuts(rec.n, src, dst, P)

    def body(r, comm, s):
        g = tigr.tigr_graph_from_coo(rec.n, src, dst, w, stream=s)
        vg = tigr.tigr_virtualize(g, 8, "strided", stream=s)
        tigr.tigr_vgraph_partition(vg, P, r)
        gs = tigr.tigr_graph_from_coo(rec.n, src, dst, None, symmetrize=True, stream=s)
        vgs = tigr.tigr_virtualize(gs, 8, "strided", stream=s)
        tigr.tigr_vgraph_partition(vgs, P, r)
        gp = tigr.tigr_graph_from_coo_part(rec.n, src, dst, w, src_lo=int(cuts[r]), src_hi=int(cuts[r + 1]),
                                           stream=s)
        vgp = tigr.tigr_virtualize(gp, 8, "strided", stream=s)
        return {"bfs": tigr.tigr_run(vg, "bfs", 0, comm=comm, exchange=exchange, stream=s),
                "cc": tigr.tigr_run(vgs, "cc", comm=comm, exchange=exchange, stream=s),
                "sssp": tigr.tigr_run(vgp, "sssp", 0, comm=comm, exchange=exchange, stream=s)}

    res = _run_group(tigr, P, body)
    for rank, got in enumerate(res):
        for a in ("bfs", "sssp", "cc"):
            assert np.array_equal(got[a], want[a]), (rank, a)


# ------------------------------------------------------------------------------ node communicator
def _node_worker(name, P, r, exchange, q):
    import os
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    try:
        import torch as t
        import paper_conf_asplos_sabetq018_b200 as tg
        t.cuda.set_device(0)
        n, src, dst, w = _graph("s16")
        comm = tg.tigr_comm_init_node(name, P, r)
        g = tg.tigr_graph_from_coo(n, src, dst, w)
        gs = tg.tigr_graph_from_coo(n, src, dst, None, symmetrize=True)
        vg = tg.tigr_virtualize(g, 8, "strided")
        vgs = tg.tigr_virtualize(gs, 8, "strided")
        tg.tigr_vgraph_partition(vg, P, r)
        tg.tigr_vgraph_partition(vgs, P, r)
        out = {a: tg.tigr_run(vg, a, 0, comm=comm, exchange=exchange) for a in ("bfs", "sssp", "sswp")}
        out["cc"] = tg.tigr_run(vgs, "cc", comm=comm, exchange=exchange)
        out["pr"] = tg.tigr_run(vg, "pr", comm=comm)
        t.cuda.synchronize()
        comm.free()
        q.put((r, out, None))
    except Exception as e:  # pragma: no cover - reported by the parent
        q.put((r, None, repr(e)))


@pytest.mark.parametrize("exchange", ["dense", "sparse", "fused"])
def test_node_communicator_processes(tigr, exchange):
    """Ranks as separate PROCESSES (both on cuda:0): shared-memory barrier + CUDA IPC buffers,
    no NCCL -- every exchange mode through real cross-process peer mappings."""
    import os
    import torch.multiprocessing as mp

    P = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    name = f"pytest_{os.getpid()}_{exchange}"
    procs = [ctx.Process(target=_node_worker, args=(name, P, r, exchange, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(P)]
    for p in procs:
        p.join(timeout=120)
    errs = [(r, e) for r, _, e in res if e]
    assert not errs, errs
    _check(_want("s16"), [out for _, out, _ in sorted(res, key=lambda x: x[0])])


def test_node_communicator_errors_and_single_rank(tigr):
    import os
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_comm_init_node("", 2, 0)
    assert e.value.status == tigr.TIGR_EINVAL
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_comm_init_node("x", 17, 0)
    assert e.value.status == tigr.TIGR_EINVAL
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_comm_init_node("x", 2, 2)
    assert e.value.status == tigr.TIGR_EINVAL
    c = tigr.tigr_comm_init_node(f"pytest1_{os.getpid()}", 1, 0)  # one rank: no peer, no wait
    n, src, dst, w = _graph("cfg1")
    vg = tigr.tigr_virtualize(tigr.tigr_graph_from_coo(n, src, dst, w), 8)
    for ex in ("dense", "sparse", "fused", "auto"):
        assert np.array_equal(tigr.tigr_run(vg, "sssp", 0, comm=c, exchange=ex), _want("cfg1")["sssp"]), ex
    assert np.abs(tigr.tigr_run(vg, "pr", comm=c) - _want("cfg1")["pr"]).max() <= 1e-6
    c.free()


# ------------------------------------------------------------------------------ NCCL, one GPU per rank
def _nccl_worker(uid, P, r, q):
    """rank r of P on cuda:r, NCCL communicator bootstrapped from the parent's unique id"""
    import os
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    try:
        import torch as t
        import paper_conf_asplos_sabetq018_b200 as tg
        t.cuda.set_device(r)
        comm = tg.tigr_comm_init(P, r, uid, device=r)
        n, src, dst, w = _graph("s16")
        g = tg.tigr_graph_from_coo(n, src, dst, w)
        gs = tg.tigr_graph_from_coo(n, src, dst, None, symmetrize=True)
        vg = tg.tigr_virtualize(g, 8, "strided")
        vgs = tg.tigr_virtualize(gs, 8, "strided")
        tg.tigr_vgraph_partition(vg, P, r)
        tg.tigr_vgraph_partition(vgs, P, r)
        # the source-range partitioned build too (each rank sorts only its own arcs)
        cuts = tg.tigr_coo_source_cuts(n, src, dst, P)
        gp = tg.tigr_graph_from_coo_part(n, src, dst, w, src_lo=int(cuts[r]), src_hi=int(cuts[r + 1]))
        vgp = tg.tigr_virtualize(gp, 8, "strided")
        out = {}
        for ex in ("dense", "sparse", "auto"):
            for a in ("bfs", "sssp", "sswp"):
                out[f"{a}_{ex}"] = tg.tigr_run(vg, a, 0, comm=comm, exchange=ex)
                out[f"{a}_{ex}_bsp"] = tg.tigr_run(vg, a, 0, comm=comm, exchange=ex, schedule=1)
            out[f"cc_{ex}"] = tg.tigr_run(vgs, "cc", comm=comm, exchange=ex)
            out[f"sssp_{ex}_part"] = tg.tigr_run(vgp, "sssp", 0, comm=comm, exchange=ex)
        out["pr"] = tg.tigr_run(vg, "pr", comm=comm)
        out["pr_part"] = tg.tigr_run(vgp, "pr", comm=comm)
        t.cuda.synchronize()
        comm.free()
        q.put((r, out, None))
    except Exception as e:  # pragma: no cover - reported by the parent
        q.put((r, None, repr(e)))


def test_nccl_one_process_per_gpu(tigr):
    """The NCCL transport with one process per GPU (the bench's N > 1 launch shape): 2-4 ranks,
    vnode-range and source-range partitions, dense / sparse / auto exchanges, both schedules.
    Every rank must return the oracle's values (PageRank within 1e-6 and bit-identical across
    ranks: NCCL sums every replica in the same order).  Skips below two GPUs -- one GPU cannot
    host two NCCL ranks."""
    import torch.multiprocessing as mp

    ngpu = torch.cuda.device_count()
    if ngpu < 2:
        pytest.skip(f"{ngpu} GPU visible: NCCL ranks need one GPU each")
    P = min(ngpu, 4)
    uid = tigr.tigr_comm_unique_id()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_nccl_worker, args=(uid, P, r, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = [q.get(timeout=900) for _ in range(P)]
    for p in procs:
        p.join(timeout=120)
    errs = [(r, e) for r, _, e in res if e]
    assert not errs, errs
    want = _want("s16")
    outs = [out for _, out, _ in sorted(res, key=lambda x: x[0])]
    for rank, out in enumerate(outs):
        for key, got in out.items():
            a = key.split("_")[0]
            if a == "pr":
                assert np.abs(got - want["pr"]).max() <= 1e-6, (rank, key)
                assert np.array_equal(got, outs[0][key]), (rank, key)  # identical across ranks
            else:
                assert np.array_equal(got, want[a]), (rank, key)


def _node_gpu_worker(name, P, r, q):
    """node communicator, rank r on cuda:r (distinct GPUs: CUDA IPC over NVLink)"""
    import os
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    try:
        import torch as t
        import paper_conf_asplos_sabetq018_b200 as tg
        t.cuda.set_device(r)
        n, src, dst, w = _graph("s16")
        comm = tg.tigr_comm_init_node(name, P, r)
        g = tg.tigr_graph_from_coo(n, src, dst, w)
        vg = tg.tigr_virtualize(g, 8, "strided")
        tg.tigr_vgraph_partition(vg, P, r)
        out = {f"{a}_{ex}": tg.tigr_run(vg, a, 0, comm=comm, exchange=ex)
               for ex in ("fused", "dense") for a in ("bfs", "sssp", "sswp")}
        t.cuda.synchronize()
        comm.free()
        q.put((r, out, None))
    except Exception as e:  # pragma: no cover
        q.put((r, None, repr(e)))


def test_node_communicator_distinct_gpus(tigr):
    """The fused exchange across distinct GPUs: every improvement is applied to the peer GPUs'
    replicas with system-scope atomics over NVLink (frontier_kernel.cuh push_peers).  Skips
    below two GPUs."""
    import os
    import torch.multiprocessing as mp

    ngpu = torch.cuda.device_count()
    if ngpu < 2:
        pytest.skip(f"{ngpu} GPU visible: needs two GPUs")
    P = min(ngpu, 4)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    name = f"pytest_gpus_{os.getpid()}"
    procs = [ctx.Process(target=_node_gpu_worker, args=(name, P, r, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = [q.get(timeout=900) for _ in range(P)]
    for p in procs:
        p.join(timeout=120)
    errs = [(r, e) for r, _, e in res if e]
    assert not errs, errs
    want = _want("s16")
    for r, out, _ in res:
        for key, got in out.items():
            assert np.array_equal(got, want[key.split("_")[0]]), (r, key)
