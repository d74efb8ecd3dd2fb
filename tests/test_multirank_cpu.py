"""Multi-rank host logic on CPU (torch.distributed, gloo, world_size 2 and 3).

What runs on N GPUs is: every rank owns the contiguous, family-aligned vnode
range that tigr_partition_ranges assigns (product code, a pure host function of the C ABI),
relaxes only its virtual nodes against a replicated value array, and the replicas are merged
every iteration by an all-reduce (MIN for BFS/SSSP/CC, MAX for SSWP, SUM for the PageRank
accumulator); activity for the next iteration is "value changed by the exchange".  Here the
per-rank relax is emulated in numpy (test code) and the all-reduce is a real gloo collective,
so the partition rule and the exchange protocol are checked end to end against the oracle.
Both merges are covered: the dense all-reduce and the sparse exchange of changed nodes
(all-gather of {node, value} lists, apply, activate the union).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

INF = 0xFFFFFFFF


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _relax_range(o, vg, lo, hi, algo, val, active, xs=None):
    """One BSP relax of vnodes [lo, hi) of the oracle's virtual graph (strided layout)."""
    new = val.copy() if algo != "pr" else np.zeros(o.n)
    for i in range(lo, hi):
        v = int(vg.vn_phys[i])
        if algo == "pr":
            d = int(o.row_ptr[v + 1] - o.row_ptr[v])
            e = vg.edges(i, 1)
            np.add.at(new, o.col[e].astype(np.int64), xs[v] / d)
            continue
        if not active[v]:
            continue
        x = int(val[v])
        for e in vg.edges(i, 1):
            nb = int(o.col[e])
            if algo == "bfs":
                alt = x + 1
            elif algo == "sssp":
                alt = x + int(o.wt[e])
            elif algo == "cc":
                alt = x
            else:
                alt = min(x, int(o.wt[e]))
            if (alt > new[nb]) if algo == "sswp" else (alt < new[nb]):
                new[nb] = alt
    return new


def _merge_sparse(algo, val, mine):
    """Sparse exchange (exchange.cu, NEXT-2): every rank publishes {node, value} of the nodes its
    relax improved; every rank applies all lists with the relax's own combine and activates
    exactly the listed nodes (the union, identical on every rank)."""
    changed = np.nonzero(mine != val)[0]
    lists = [None] * dist.get_world_size()
    dist.all_gather_object(lists, (changed.tolist(), mine[changed].tolist()))
    nxt = mine.copy()
    active = np.zeros(len(val), dtype=bool)
    for ids, vals in lists:
        ids = np.asarray(ids, dtype=np.int64)
        vals = np.asarray(vals, dtype=np.int64)
        if algo == "sswp":
            np.maximum.at(nxt, ids, vals)
        else:
            np.minimum.at(nxt, ids, vals)
        active[ids] = True
    return nxt, active


def _worker(rank, world, port, q, mode="dense"):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import graphgen
    import oracle
    import paper_conf_asplos_sabetq018_b200 as tigr

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rec = graphgen.recipe("cfg1")
        src, dst, w = graphgen.generate(rec)
        o = oracle.csr_build(rec.n, src, dst, w)
        sym = oracle.symmetrize(src, dst, w)
        osym = oracle.csr_build(rec.n, *sym)
        out = {}
        for algo in ("bfs", "sssp", "sswp", "cc", "pr"):
            g = osym if algo == "cc" else o
            vg = oracle.Virtual(g, 8)
            lo, hi = tigr.tigr_partition_ranges(g.row_ptr, vg.vnode_ptr.astype(np.uint32), world)
            mylo, myhi = int(lo[rank]), int(hi[rank])
            if algo == "pr":
                x = np.full(g.n, 1.0 / g.n)
                for _ in range(20):
                    acc = torch.from_numpy(_relax_range(g, vg, mylo, myhi, "pr", None, None, x))
                    dist.all_reduce(acc, op=dist.ReduceOp.SUM)
                    x = 0.15 / g.n + 0.85 * acc.numpy()
                out[algo] = x
                continue
            val = np.full(g.n, INF, dtype=np.int64)
            active = np.zeros(g.n, dtype=bool)
            if algo == "cc":
                val = np.arange(g.n, dtype=np.int64)
                active[:] = True
            elif algo == "sswp":
                val[:] = 0
                val[0] = INF
                active[0] = True
            else:
                val[0] = 0
                active[0] = True
            while True:
                mine = _relax_range(g, vg, mylo, myhi, algo, val, active)
                if mode == "sparse":
                    nxt, active = _merge_sparse(algo, val, mine)
                else:
                    t = torch.from_numpy(mine)
                    dist.all_reduce(t, op=dist.ReduceOp.MAX if algo == "sswp" else dist.ReduceOp.MIN)
                    nxt = t.numpy()
                    active = nxt != val  # identical on every rank: no extra collective needed
                val = nxt
                if not active.any():
                    break
            out[algo] = val.astype(np.uint32)
        q.put((rank, [int(x) for x in lo], [int(x) for x in hi], out))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,mode", [(2, "dense"), (3, "dense"), (2, "sparse"), (3, "sparse")])
def test_partitioned_exchange_matches_oracle(world, mode):
    import graphgen
    import oracle

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, mode)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst, w)
    want = {"bfs": oracle.bfs(o, 0), "sssp": oracle.sssp(o, 0), "sswp": oracle.sswp(o, 0),
            "cc": oracle.cc(rec.n, src, dst), "pr": oracle.pagerank(o, 20)}
    for rank, lo, hi, out in res:
        # ranges tile [0, NV) contiguously
        assert lo[0] == 0 and all(hi[r] == lo[r + 1] for r in range(world - 1))
        assert hi[-1] == oracle.Virtual(o, 8).nv  # ranges of the last graph run (PR on the arc graph)
        for algo in ("bfs", "sssp", "sswp", "cc"):
            assert np.array_equal(out[algo], want[algo]), (rank, algo)
        assert np.abs(out["pr"] - want["pr"]).max() < 1e-12


def test_partition_ranges_balance():
    """Ranges are balanced by arc count up to one family."""
    import graphgen
    import oracle
    import paper_conf_asplos_sabetq018_b200 as tigr

    rec = graphgen.recipe("cfg2")
    src, dst, _ = graphgen.rmat(rec.n, rec.m // 8, rec.a, rec.b, rec.c, rec.seed, weighted=False)
    o = oracle.csr_build(rec.n, src, dst)
    vg = oracle.Virtual(o, 8)
    deg = np.diff(o.row_ptr)
    fam_start = vg.vnode_ptr.astype(np.int64)
    for P in (2, 4, 8):
        lo, hi = tigr.tigr_partition_ranges(o.row_ptr, vg.vnode_ptr.astype(np.uint32), P)
        assert lo[0] == 0 and hi[-1] == vg.nv and (lo[1:] == hi[:-1]).all()
        assert set(lo.tolist()) <= set(fam_start.tolist())  # family-aligned
        arcs = [int(o.row_ptr[vg.vn_phys[h - 1] + 1] - o.row_ptr[vg.vn_phys[l_]]) if h > l_ else 0
                for l_, h in zip(lo, hi)]
        assert sum(arcs) == o.m
        assert max(arcs) - o.m / P <= deg.max() + 1, (P, arcs)
