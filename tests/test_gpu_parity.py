"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded
inputs.  Bit-exact for generator / CSR / virtual split / BFS / SSSP / CC / SSWP; PageRank
within 1e-6 max abs per vertex (BASELINE.json north_star).  Where several results are
correct (the order of arcs inside a CSR segment, hence which arcs a virtual node owns) the
unique part is compared exactly and the rest is checked for validity."""
import numpy as np
import pytest

import graphgen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

INF = 0xFFFFFFFF


@pytest.fixture(scope="module")
def tigr():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_asplos_sabetq018_b200 as t
    return t


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


# ------------------------------------------------------------------------------------ a0
@pytest.mark.parametrize("cfg", ["cfg1", "cfg2", "cfg3"])
def test_generator_bit_exact(tigr, cfg):
    rec = graphgen.recipe(cfg)
    m = min(rec.m, 1 << 24)
    src, dst, w = graphgen.rmat(rec.n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax)
    ds = torch.empty(m, dtype=torch.int32, device="cuda")
    dd, dw = torch.empty_like(ds), torch.empty_like(ds)
    tigr.tigr_rmat_coo(rec.n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, ds, dd, dw)
    torch.cuda.synchronize()
    assert np.array_equal(_u32(ds), src) and np.array_equal(_u32(dd), dst) and np.array_equal(_u32(dw), w)


def test_generator_full_scale_sampled(tigr):
    """cfg5 (1.47B arcs): a prefix and a far slice, drawn on both sides (counter-based)."""
    rec = graphgen.recipe("cfg5")
    m = 1 << 20
    ds = torch.empty(m, dtype=torch.int32, device="cuda")
    dd, dw = torch.empty_like(ds), torch.empty_like(ds)
    tigr.tigr_rmat_coo(rec.n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax, ds, dd, dw)
    src, dst, w = graphgen.rmat(rec.n, m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, rec.wmin, rec.wmax)
    assert np.array_equal(_u32(ds), src) and np.array_equal(_u32(dd), dst) and np.array_equal(_u32(dw), w)


# ------------------------------------------------------------------------------------ a1
def _canon(rp, col, w):
    """Per-segment sort by (col, w): the unique content of a CSR with unordered segments."""
    n = len(rp) - 1
    seg = np.repeat(np.arange(n), np.diff(rp))
    keys = (col, seg) if w is None else (w, col, seg)
    order = np.lexsort(keys)
    return col[order], (None if w is None else w[order])


@pytest.mark.parametrize("sym", [False, True])
def test_csr_build_matches_oracle(tigr, sym):
    rec = graphgen.recipe("cfg2")
    src, dst, w = graphgen.rmat(rec.n, rec.m // 2, rec.a, rec.b, rec.c, rec.seed, rec.wseed)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w, symmetrize=sym)
    rp, col, wt = tigr.tigr_graph_export_csr(g)
    o = oracle.csr_build(rec.n, *(oracle.symmetrize(src, dst, w) if sym else (src, dst, w)))
    assert np.array_equal(rp, o.row_ptr)
    # the radix-sort build is stable: the canonical CSR, element by element
    assert np.array_equal(col, o.col) and np.array_equal(wt, o.wt)
    c1, w1 = _canon(rp, col, wt)
    c2, w2 = _canon(o.row_ptr, o.col, o.wt)
    assert np.array_equal(c1, c2) and np.array_equal(w1, w2)


def test_export_coo_roundtrip(tigr):
    """tigr_graph_export_coo: the canonical CSR's arc list (Fig. 10a order); host and device
    outputs agree, and rebuilding from it gives the same CSR."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    es, ed, ew = tigr.tigr_graph_export_coo(g)
    o = oracle.csr_build(rec.n, src, dst, w)
    assert np.array_equal(es, np.repeat(np.arange(rec.n, dtype=np.uint32), np.diff(o.row_ptr)))
    assert np.array_equal(ed, o.col) and np.array_equal(ew, o.wt)
    d = [torch.empty(rec.m, dtype=torch.int32, device="cuda") for _ in range(3)]
    tigr._check(tigr._lib.tigr_graph_export_coo(g.ptr, d[0].data_ptr(), d[1].data_ptr(), d[2].data_ptr(), 1, None))
    assert np.array_equal(_u32(d[0]), es) and np.array_equal(_u32(d[1]), ed) and np.array_equal(_u32(d[2]), ew)
    g2 = tigr.tigr_graph_from_coo(rec.n, es, ed, ew)
    for a, b in zip(tigr.tigr_graph_export_csr(g2), tigr.tigr_graph_export_csr(g)):
        assert np.array_equal(a, b)
    gs = tigr.tigr_graph_from_coo(rec.n, src, dst, None, symmetrize=True)
    ss, sd, sw = tigr.tigr_graph_export_coo(gs)
    assert sw is None and len(ss) == 2 * rec.m


def test_csr_from_csr_roundtrip(tigr):
    src, dst, w = graphgen.random_small(300, 4000, 5)
    o = oracle.csr_build(300, src, dst, w)
    g = tigr.tigr_graph_from_csr(300, o.row_ptr, o.col, o.wt)
    rp, col, wt = tigr.tigr_graph_export_csr(g)
    assert np.array_equal(rp, o.row_ptr) and np.array_equal(col, o.col) and np.array_equal(wt, o.wt)


# ------------------------------------------------------------------------------------ a2-a5
@pytest.mark.parametrize("K", [1, 3, 4, 8, 12, 32, 0xFFFFFFFF])
@pytest.mark.parametrize("layout", ["consecutive", "strided"])
def test_virtual_split_and_assignment(tigr, K, layout):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, K, layout)
    vp, ph = tigr.tigr_vgraph_export(vg)
    rp, col, wt = tigr.tigr_graph_export_csr(g)
    o = oracle.csr_build(rec.n, src, dst, w)
    ov = oracle.Virtual(o, K)
    assert np.array_equal(vp, ov.vnode_ptr.astype(np.uint32)) and np.array_equal(ph, ov.vn_phys)
    counts, nbr, ww = tigr.tigr_vgraph_assignment(vg)
    # the unit of the layout: 32-byte spans (8 edges) when 8 | K, 16-byte chunks
    # (4 edges) when 4 | K, else one edge
    chunk = 8 if (K % 8 == 0 or K == 0xFFFFFFFF) else (4 if K % 4 == 0 else 1)
    lay = 0 if layout == "consecutive" else 1
    want = np.array([len(ov.edges(i, lay, chunk)) for i in range(ov.nv)], dtype=np.uint32)
    assert np.array_equal(counts, want)
    assert counts.max() <= K
    # every arc exactly once: a family's arcs are its node's segment (as multisets)
    offs = np.concatenate([[0], np.cumsum(counts.astype(np.int64))])
    for v in np.flatnonzero(np.diff(o.row_ptr)):
        a, b = offs[vp[v]], offs[vp[v + 1]]
        got = sorted(zip(nbr[a:b].tolist(), ww[a:b].tolist()))
        exp = sorted(zip(o.col[o.row_ptr[v]:o.row_ptr[v + 1]].tolist(), o.wt[o.row_ptr[v]:o.row_ptr[v + 1]].tolist()))
        assert got == exp, v
    # stable CSR: every vnode owns exactly the oracle's arcs, in the oracle's order
    assert np.array_equal(col, o.col)
    want_nbr = np.concatenate([o.col[ov.edges(i, lay, chunk)] for i in range(ov.nv)])
    want_w = np.concatenate([o.wt[ov.edges(i, lay, chunk)] for i in range(ov.nv)])
    assert np.array_equal(nbr, want_nbr) and np.array_equal(ww, want_w)


# ------------------------------------------------------------------------------------ a6-a9
def _oracle_all(n, src, dst, w, source=0):
    o = oracle.csr_build(n, src, dst, w)
    return {"bfs": oracle.bfs(o, source), "sssp": oracle.sssp(o, source), "sswp": oracle.sswp(o, source),
            "cc": oracle.cc(n, src, dst), "pr": oracle.pagerank(o, 20)}


def _run_all(tigr, n, src, dst, w, K=8, layout="strided", source=0, **kw):
    g = tigr.tigr_graph_from_coo(n, src, dst, w)
    gs = tigr.tigr_graph_from_coo(n, src, dst, None, symmetrize=True)
    vg = tigr.tigr_virtualize(g, K, layout)
    vgs = tigr.tigr_virtualize(gs, K, layout)
    out = {a: tigr.tigr_run(vg, a, source, **kw) for a in ("bfs", "sssp", "sswp")}
    out["cc"] = tigr.tigr_run(vgs, "cc", **kw)
    prkw = {k: v for k, v in kw.items() if k not in ("schedule", "frontier")}
    out["pr"] = tigr.tigr_run(vg, "pr", **prkw)
    return out


def _assert_parity(got, want):
    for a in ("bfs", "sssp", "sswp", "cc"):
        assert np.array_equal(got[a], want[a]), a
    err = np.abs(got["pr"] - want["pr"]).max() if len(want["pr"]) else 0.0
    assert err <= 1e-6, err


@pytest.mark.parametrize("K", [1, 4, 8, 12, 32, 0xFFFFFFFF])
@pytest.mark.parametrize("layout", ["consecutive", "strided"])
def test_cfg1_all_algorithms(tigr, K, layout):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    _assert_parity(_run_all(tigr, rec.n, src, dst, w, K, layout), _oracle_all(rec.n, src, dst, w))


@pytest.mark.parametrize("schedule,frontier,use_graph", [(0, 1, 1), (1, 1, 1), (0, 2, 1), (1, 2, 0), (0, 1, 0),
                                                          (0, 3, 1), (1, 3, 1), (0, 3, 0), (1, 0, 1), (0, 0, 0)])
def test_cfg1_schedules(tigr, schedule, frontier, use_graph):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    got = _run_all(tigr, rec.n, src, dst, w, schedule=schedule, frontier=frontier, use_graph=use_graph)
    _assert_parity(got, _oracle_all(rec.n, src, dst, w))


def test_bsp_iterations_match_paper_literal_push(tigr):
    """Table 8 (L1480-1486): BSP #iterations are the same for the original graph and every
    virtual split; and equal to the oracle's paper-literal sequential push (BSP, worklist)."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst, w)
    for algo, code in (("bfs", oracle.BFS), ("sssp", oracle.SSSP), ("sswp", oracle.SSWP)):
        _, want_it, _ = oracle.push_virtual(o, oracle.Virtual(o, 8), code, 0, schedule=1, worklist=1)
        for K in (1, 8, 0xFFFFFFFF):
            g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
            vg = tigr.tigr_virtualize(g, K, "strided")
            vals, st = tigr.tigr_run(vg, algo, 0, schedule=1, return_stats=True)
            assert st["iterations"] == want_it, (algo, K, st["iterations"], want_it)


def test_cfg2_bfs_cc(tigr):
    rec = graphgen.recipe("cfg2")
    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False)
    gs = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False,
                              symmetrize=True)
    vg = tigr.tigr_virtualize(g, 8)
    vgs = tigr.tigr_virtualize(gs, 8)
    o = oracle.csr_build(rec.n, src, dst)
    assert np.array_equal(tigr.tigr_run(vg, "bfs", 0), oracle.bfs(o, 0))
    assert np.array_equal(tigr.tigr_run(vgs, "cc"), oracle.cc(rec.n, src, dst))


# ------------------------------------------------------------------------------------ edge cases
def _edge_cases():
    cases = {}
    cases["single_vertex"] = (1, [], [], [])
    cases["no_edges"] = (5, [], [], [])
    cases["self_loops_dups"] = (4, [0, 0, 0, 1, 1, 2], [0, 1, 1, 1, 2, 2], [3, 5, 2, 1, 7, 4])
    cases["source_deg0"] = (4, [1, 2], [2, 3], [1, 1])
    cases["two_components"] = (6, [0, 1, 3, 4], [1, 2, 4, 5], [2, 2, 9, 9])
    cases["cycle"] = (7, list(range(7)), [(i + 1) % 7 for i in range(7)], [1, 2, 3, 4, 5, 6, 7])
    star = 70000  # hub with d >> 32K
    cases["hub"] = (star + 1, [0] * star + list(range(1, star + 1)), list(range(1, star + 1)) + [0] * star,
                    [(i % 64) + 1 for i in range(2 * star)])
    for d in (7, 8, 9, 16, 17, 257):  # d around K and 32K+1 for K = 8
        cases[f"deg{d}"] = (d + 2, [0] * d + [1], list(range(1, d + 1)) + [d + 1], [(3 * i) % 64 + 1 for i in range(d + 1)])
    k = 12
    cases["complete"] = (k, [i for i in range(k) for j in range(k) if i != j],
                         [j for i in range(k) for j in range(k) if i != j], [((i * 7 + j) % 64) + 1 for i in range(k) for j in range(k) if i != j])
    return cases


@pytest.mark.parametrize("name", list(_edge_cases()))
@pytest.mark.parametrize("K", [1, 8])
def test_edge_cases(tigr, name, K):
    n, src, dst, w = _edge_cases()[name]
    src, dst, w = (np.asarray(x, dtype=np.uint32) for x in (src, dst, w))
    _assert_parity(_run_all(tigr, n, src, dst, w, K), _oracle_all(n, src, dst, w))


@pytest.mark.parametrize("name", list(_edge_cases()))
@pytest.mark.parametrize("K", [4, 8, 32])
@pytest.mark.parametrize("schedule", [0, 1])
def test_edge_cases_queue(tigr, name, K, schedule):
    """Frontier QUEUE (dynamic mapping, frontier.cu): the active-node queue and the on-the-fly
    (node, j) mapping reproduce the oracle on every edge case, incl. a 70 000-arc hub whose
    8750 virtual nodes span hundreds of warp rounds of one queue entry."""
    n, src, dst, w = _edge_cases()[name]
    src, dst, w = (np.asarray(x, dtype=np.uint32) for x in (src, dst, w))
    got = _run_all(tigr, n, src, dst, w, K, frontier=3, schedule=schedule)
    _assert_parity(got, _oracle_all(n, src, dst, w))


@pytest.mark.parametrize("layout", ["consecutive", "strided"])
@pytest.mark.parametrize("div", [1, 2, 1000000])
def test_hybrid_frontier_switch(tigr, layout, div):
    """FRONTIER_AUTO switches between the queue and the dense sweep per iteration on the device
    (frontier_div = D: queue while the queued vnodes are < 1/D of all, so D = 1 is almost always
    the queue and D = 1e6 almost always the dense sweep): every switch point gives the oracle's
    values and BSP iteration counts."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    want = _oracle_all(rec.n, src, dst, w)
    for K in (4, 8, 32):
        _assert_parity(_run_all(tigr, rec.n, src, dst, w, K, layout, frontier_div=div), want)
    o = oracle.csr_build(rec.n, src, dst, w)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, 8, layout)
    for algo, code in (("bfs", oracle.BFS), ("sssp", oracle.SSSP), ("sswp", oracle.SSWP)):
        _, want_it, _ = oracle.push_virtual(o, oracle.Virtual(o, 8), code, 0, schedule=1, worklist=1)
        vals, st = tigr.tigr_run(vg, algo, 0, schedule=1, return_stats=True, frontier_div=div)
        assert np.array_equal(vals, want[algo]) and st["iterations"] == want_it, (algo, st["iterations"], want_it)


def test_queue_mode_stats_and_errors(tigr):
    """QUEUE counts the same processed arcs as the dense sweep (BSP BFS: every arc of every
    reached node), reports its queue iterations, and needs the 16-byte-chunk layout."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, 8)
    deg = np.bincount(src, minlength=rec.n)
    lv, st = tigr.tigr_run(vg, "bfs", 0, schedule=1, frontier=3, collect_stats=1, return_stats=True)
    assert st["edges_processed"] == int(deg[lv != INF].sum())
    assert st["queue_iterations"] == st["iterations"]
    _, st1 = tigr.tigr_run(vg, "bfs", 0, schedule=1, frontier=1, collect_stats=1, return_stats=True)
    assert st1["edges_processed"] == st["edges_processed"] and st1["queue_iterations"] == 0
    vg3 = tigr.tigr_virtualize(g, 3)  # 4 does not divide K: per-arc units, no queue kernel
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_run(vg3, "bfs", 0, frontier=3)
    assert e.value.status == tigr.TIGR_EUNSUPPORTED
    assert np.array_equal(tigr.tigr_run(vg3, "bfs", 0), lv)  # AUTO falls back to the dense sweep
    with pytest.raises(tigr.TigrError):
        tigr.tigr_run(vg, "pr", frontier=3)


def test_unit_weights_sssp_equals_bfs(tigr):
    src, dst, _ = graphgen.random_small(500, 3000, 11)
    g = tigr.tigr_graph_from_coo(500, src, dst, np.ones(len(src), np.uint32))
    vg = tigr.tigr_virtualize(g, 8)
    assert np.array_equal(tigr.tigr_run(vg, "sssp", 3), tigr.tigr_run(vg, "bfs", 3))


def test_pr_dangling_redistribute(tigr):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, None)
    vg = tigr.tigr_virtualize(g, 8)
    got = tigr.tigr_run(vg, "pr", pr_dangling=1)
    want = oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20, 0.85, 1)
    assert np.abs(got - want).max() <= 1e-6
    assert abs(got.sum() - 1.0) < 1e-9  # redistribute conserves mass


@pytest.mark.parametrize("dangling", [0, 1])
def test_pr_iteration_counts_and_fused_apply(tigr, dangling):
    """PageRank after 0, 1, 2, 3 and 20 iterations, with the apply fused into the relax
    (pr_dangling = 0, the default) and as a separate pass (pr_dangling = 1 needs it): the two
    accumulators alternate correctly and x is materialised after the last iteration; damping
    0.5 and 1.0 exercise the constants."""
    rec = graphgen.recipe("cfg1")
    src, dst, _ = graphgen.generate(rec)
    o = oracle.csr_build(rec.n, src, dst)
    vg = tigr.tigr_virtualize(tigr.tigr_graph_from_coo(rec.n, src, dst, None), 8)
    for iters in (0, 1, 2, 3, 20):
        got = tigr.tigr_run(vg, "pr", pr_iters=iters, pr_dangling=dangling)
        assert np.abs(got - oracle.pagerank(o, iters, 0.85, dangling)).max() <= 1e-15, iters
    for d in (0.5, 1.0):
        got = tigr.tigr_run(vg, "pr", pr_iters=7, pr_damping=d, pr_dangling=dangling)
        assert np.abs(got - oracle.pagerank(o, 7, d, dangling)).max() <= 1e-15, d


def test_errors(tigr):
    src, dst, w = graphgen.random_small(10, 30, 1)
    g = tigr.tigr_graph_from_coo(10, src, dst, None)
    vg = tigr.tigr_virtualize(g, 8)
    for bad in (lambda: tigr.tigr_run(vg, "sssp", 0),          # unweighted
                lambda: tigr.tigr_run(vg, "cc"),                # not symmetric
                lambda: tigr.tigr_run(vg, "bfs", 10),           # source >= n
                lambda: tigr.tigr_virtualize(g, 0),             # K = 0
                lambda: tigr.tigr_graph_from_coo(10, [0, 10], [1, 2]),  # id >= n
                lambda: tigr.tigr_graph_from_csr(3, np.array([0, 2, 1, 3]), np.array([0, 1, 2]))):
        with pytest.raises(tigr.TigrError) as ei:
            bad()
        assert ei.value.status == tigr.TIGR_EINVAL
    gw = tigr.tigr_graph_from_coo(10, src, dst, w)
    vgw = tigr.tigr_virtualize(gw, 8)
    with pytest.raises(tigr.TigrError) as ei:
        tigr.tigr_run(vgw, "sssp", 0, max_iters=1)
    assert ei.value.status == tigr.TIGR_ENOTCONV


def test_device_buffers_and_streams(tigr):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        g = tigr.tigr_graph_from_coo(rec.n, _dev(src), _dev(dst), _dev(w), stream=s)
        vg = tigr.tigr_virtualize(g, 8, stream=s)
        out = torch.empty(rec.n, dtype=torch.int32, device="cuda")
        tigr.tigr_run(vg, "sssp", 0, out=out, stream=s)
        s.synchronize()
    assert np.array_equal(_u32(out), oracle.sssp(oracle.csr_build(rec.n, src, dst, w), 0))
    prd = torch.empty(rec.n, dtype=torch.float64, device="cuda")
    tigr.tigr_run(vg, "pr", out=prd, stream=s)
    assert np.abs(prd.cpu().numpy() - oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20)).max() <= 1e-6


def test_stats_counts(tigr):
    """collect_stats: PR processes every arc every iteration; frontier runs count edges of
    active vnodes (BFS in BSP mode = arcs out of each level, i.e. all arcs of reached nodes)."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, 8)
    _, st = tigr.tigr_run(vg, "pr", collect_stats=1, return_stats=True)
    assert st["edges_processed"] == 20 * rec.m
    lv, st = tigr.tigr_run(vg, "bfs", 0, schedule=1, collect_stats=1, return_stats=True)
    deg = np.bincount(src, minlength=rec.n)
    assert st["edges_processed"] == int(deg[lv != INF].sum())


def test_partition_ranges(tigr):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, 8)
    vp, _ = tigr.tigr_vgraph_export(vg)
    nv = vg.info()["nv"]
    for P in (2, 3, 8):
        bounds = []
        for r in range(P):
            tigr.tigr_vgraph_partition(vg, P, r)
            i = vg.info()
            bounds.append((i["lo"], i["hi"]))
            assert i["lo"] in set(vp.tolist()) and i["hi"] in set(vp.tolist())  # family-aligned
        assert bounds[0][0] == 0 and bounds[-1][1] == nv
        assert all(bounds[r][1] == bounds[r + 1][0] for r in range(P - 1))
        rp, _, _ = tigr.tigr_graph_export_csr(g)
        lo, hi = tigr.tigr_partition_ranges(rp, vp, P)  # host rule == device rule
        assert [tuple(x) for x in zip(lo.tolist(), hi.tolist())] == bounds
    tigr.tigr_vgraph_partition(vg, 1, 0)
    assert vg.info()["hi"] == nv


def test_exchange_path_single_rank_nccl(tigr):
    """The multi-GPU code path (NCCL all-reduce every iteration, k_diff activation, host loop)
    on a 1-rank communicator: results must not change."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    comm = tigr.tigr_comm_init(1, 0, tigr.tigr_comm_unique_id())
    want = _oracle_all(rec.n, src, dst, w)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    gs = tigr.tigr_graph_from_coo(rec.n, src, dst, None, symmetrize=True)
    vg = tigr.tigr_virtualize(g, 8)
    vgs = tigr.tigr_virtualize(gs, 8)
    tigr.tigr_vgraph_partition(vg, 1, 0)
    for algo in ("bfs", "sssp", "sswp"):
        assert np.array_equal(tigr.tigr_run(vg, algo, 0, comm=comm), want[algo]), algo
        assert np.array_equal(tigr.tigr_run(vg, algo, 0, comm=comm, schedule=1), want[algo]), algo
    assert np.array_equal(tigr.tigr_run(vgs, "cc", comm=comm), want["cc"])
    assert np.abs(tigr.tigr_run(vg, "pr", comm=comm) - want["pr"]).max() <= 1e-6
    comm.free()


# ------------------------------------------------------------------------------------ NEXT-1: pull PR
def _owner(rp):
    return np.repeat(np.arange(len(rp) - 1, dtype=np.uint32), np.diff(rp))


def test_transpose_matches_oracle(tigr):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    gt = tigr.tigr_graph_transpose(g)
    assert gt.info()["transposed"] and gt.info()["m"] == rec.m
    o = oracle.csr_build(rec.n, src, dst, w)
    # the transpose keeps the forward CSR's arc order (stable): reverse the oracle's CSR arcs
    ot = oracle.csr_build(rec.n, o.col, _owner(o.row_ptr), o.wt)
    rp, col, wt = tigr.tigr_graph_export_csr(gt)
    assert np.array_equal(rp, ot.row_ptr) and np.array_equal(col, ot.col) and np.array_equal(wt, ot.wt)
    vgt = tigr.tigr_virtualize(gt, 8)
    assert np.array_equal(tigr.tigr_run(vgt, "bfs", 3), oracle.bfs(ot, 3))   # BFS on the reversed graph


@pytest.mark.parametrize("K", [1, 4, 8, 32, 0xFFFFFFFF])
@pytest.mark.parametrize("layout", ["consecutive", "strided"])
def test_pull_pagerank_cfg1(tigr, K, layout):
    """PageRank pulled over a virtual split of the in-CSR equals the
    push / power-iteration result (Thm. 3)."""
    rec = graphgen.recipe("cfg1")
    src, dst, _ = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, None)
    gt = tigr.tigr_graph_transpose(g)
    if K % 4 and K != 0xFFFFFFFF:
        with pytest.raises(tigr.TigrError):
            tigr.tigr_run(tigr.tigr_virtualize(gt, K, layout), "pr")
        return
    got = tigr.tigr_run(tigr.tigr_virtualize(gt, K, layout), "pr")
    want = oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20)
    assert np.abs(got - want).max() <= 1e-6
    assert np.abs(got - want).max() <= 1e-15  # float64, tiny graph: only association differs
    for dang in (1,):
        got = tigr.tigr_run(tigr.tigr_virtualize(gt, K, layout), "pr", pr_dangling=dang)
        want = oracle.pagerank(oracle.csr_build(rec.n, src, dst), 20, 0.85, dang)
        assert np.abs(got - want).max() <= 1e-6


def test_pull_pagerank_edge_cases(tigr):
    for name, (n, src, dst, w) in _edge_cases().items():
        src, dst = (np.asarray(x, dtype=np.uint32) for x in (src, dst))
        g = tigr.tigr_graph_from_coo(n, src, dst, None)
        gt = tigr.tigr_graph_transpose(g)
        got = tigr.tigr_run(tigr.tigr_virtualize(gt, 8), "pr")
        want = oracle.pagerank(oracle.csr_build(n, src, dst), 20)
        assert np.abs(got - want).max() <= 1e-12, name


# ------------------------------------------------------------------------------------ NEXT-4: UDT
@pytest.mark.parametrize("K", [2, 3, 8])
def test_udt_matches_oracle(tigr, K):
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    o = oracle.csr_build(rec.n, src, dst, w)
    n2, us, ud, uw = oracle.udt(o, K, 0)
    gu = tigr.tigr_graph_udt(g, K, 0)
    assert gu.info()["n"] == n2 and gu.info()["m"] == len(us)
    ou = oracle.csr_build(n2, us, ud, uw)
    rp, col, wt = tigr.tigr_graph_export_csr(gu)
    assert np.array_equal(rp, ou.row_ptr) and np.array_equal(col, ou.col) and np.array_equal(wt, ou.wt)
    # Cor. 2: SSSP over the UDT graph (any virtual split of it) keeps the original distances
    for vk in (8, 0xFFFFFFFF):
        vgu = tigr.tigr_virtualize(gu, vk)
        assert np.array_equal(tigr.tigr_run(vgu, "sssp", 0)[:rec.n], oracle.sssp(o, 0))
    # Cor. 3: SSWP with dumb weight = +inf
    gw = tigr.tigr_graph_udt(g, K, 0xFFFFFFFF)
    assert np.array_equal(tigr.tigr_run(tigr.tigr_virtualize(gw, 8), "sswp", 0)[:rec.n], oracle.sswp(o, 0))
    # BFS = SSSP with unit weights on an unweighted graph's UDT
    g1 = tigr.tigr_graph_from_coo(rec.n, src, dst, None)
    gb = tigr.tigr_graph_udt(g1, K, 0, 1)
    assert np.array_equal(tigr.tigr_run(tigr.tigr_virtualize(gb, 8), "sssp", 0)[:rec.n],
                          oracle.bfs(oracle.csr_build(rec.n, src, dst), 0))
    with pytest.raises(tigr.TigrError):
        tigr.tigr_graph_udt(g, 1, 0)


# ------------------------------------------------------------------------------------ e: partitioned builds
@pytest.mark.parametrize("sym", [False, True])
def test_partitioned_build_union(tigr, sym):
    """Rank r's source-filtered build holds exactly the rows [cuts[r], cuts[r+1]) of the full
    CSR (same stable order); the cuts balance arcs to within one histogram bucket."""
    rec = graphgen.recipe("cfg2")
    n = rec.n
    src, dst, w = graphgen.rmat(n, rec.m // 4, rec.a, rec.b, rec.c, rec.seed, rec.wseed)
    S, D, W = oracle.symmetrize(src, dst, w) if sym else (src, dst, w)
    o = oracle.csr_build(n, S, D, W)
    deg = np.diff(o.row_ptr)
    M = len(S)
    for P in (1, 2, 3, 8):
        cuts = tigr.tigr_coo_source_cuts(n, src, dst, P, symmetrize=sym)
        assert cuts[0] == 0 and cuts[-1] == n and np.all(np.diff(cuts.astype(np.int64)) >= 0)
        width = max(1, n // 16384)
        assert all(c % width == 0 for c in cuts[:-1])
        bucket_max = int(np.add.reduceat(deg, np.arange(0, n, width)).max())
        for r in range(1, P):
            assert abs(int(o.row_ptr[cuts[r]]) - r * M // P) <= bucket_max
    cuts = tigr.tigr_coo_source_cuts(n, src, dst, 3, symmetrize=sym)
    total = 0
    for r in range(3):
        lo, hi = int(cuts[r]), int(cuts[r + 1])
        gp = tigr.tigr_graph_from_coo_part(n, src, dst, w, symmetrize=sym, src_lo=lo, src_hi=hi)
        rp, col, wt = tigr.tigr_graph_export_csr(gp)
        pd = np.diff(rp)
        assert np.array_equal(pd[lo:hi], deg[lo:hi]) and not pd[:lo].any() and not pd[hi:].any()
        a, b = int(o.row_ptr[lo]), int(o.row_ptr[hi])
        assert np.array_equal(col, o.col[a:b]) and np.array_equal(wt, o.wt[a:b])
        assert gp.info()["m"] == b - a
        total += b - a
    assert total == M
    # empty and full ranges
    ge = tigr.tigr_graph_from_coo_part(n, src, dst, w, src_lo=5, src_hi=5)
    assert ge.info()["m"] == 0
    gf = tigr.tigr_graph_from_coo_part(n, src, dst, w, src_lo=0, src_hi=n)
    assert np.array_equal(tigr.tigr_graph_export_csr(gf)[1], oracle.csr_build(n, src, dst, w).col)


def test_partitioned_graph_runs(tigr):
    """A partition is a graph of its own: without a communicator every algorithm reaches the
    oracle's result on the filtered arc list; PageRank's dangling mass is refused there."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    cuts = tigr.tigr_coo_source_cuts(rec.n, src, dst, 2)
    for r in range(2):
        lo, hi = int(cuts[r]), int(cuts[r + 1])
        keep = (src >= lo) & (src < hi)
        o = oracle.csr_build(rec.n, src[keep], dst[keep], w[keep])
        gp = tigr.tigr_graph_from_coo_part(rec.n, src, dst, w, src_lo=lo, src_hi=hi)
        for K, layout in ((8, "strided"), (3, "consecutive")):
            vg = tigr.tigr_virtualize(gp, K, layout)
            assert np.array_equal(tigr.tigr_run(vg, "bfs", 0), oracle.bfs(o, 0))
            assert np.array_equal(tigr.tigr_run(vg, "sssp", 0), oracle.sssp(o, 0))
            assert np.array_equal(tigr.tigr_run(vg, "sswp", 0), oracle.sswp(o, 0))
            assert np.abs(tigr.tigr_run(vg, "pr") - oracle.pagerank(o, 20)).max() <= 1e-6
            with pytest.raises(tigr.TigrError):
                tigr.tigr_run(vg, "pr", pr_dangling=1)


# ------------------------------------------------------------------------------------ reordered graphs
def test_reorder_permutation_and_csr(tigr):
    """tigr_graph_reorder: nodes by decreasing in-degree (ties by id), the CSR equal to the
    canonical CSR of the relabelled arc list (targets relabelled, each node's arcs in order)."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    g2 = tigr.tigr_graph_reorder(g)
    cid, order = tigr.tigr_graph_permutation(g2)
    assert np.array_equal(np.sort(order), np.arange(rec.n)) and np.array_equal(cid[order], np.arange(rec.n))
    indeg = np.bincount(dst, minlength=rec.n)
    assert np.array_equal(order, np.lexsort((np.arange(rec.n), -indeg)))
    o2 = oracle.csr_build(rec.n, cid[src], cid[dst], w)
    rp, col, ww = tigr.tigr_graph_export_csr(g2)
    assert np.array_equal(rp, o2.row_ptr) and np.array_equal(col, o2.col) and np.array_equal(ww, o2.wt)
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_graph_reorder(g2)
    assert e.value.status == tigr.TIGR_EUNSUPPORTED
    with pytest.raises(tigr.TigrError) as e:
        tigr.tigr_graph_permutation(g)
    assert e.value.status == tigr.TIGR_EINVAL


def _run_all_reordered(tigr, n, src, dst, w, K=8, layout="strided", source=0, **kw):
    g = tigr.tigr_graph_reorder(tigr.tigr_graph_from_coo(n, src, dst, w))
    gs = tigr.tigr_graph_reorder(tigr.tigr_graph_from_coo(n, src, dst, None, symmetrize=True))
    vg = tigr.tigr_virtualize(g, K, layout)
    vgs = tigr.tigr_virtualize(gs, K, layout)
    out = {a: tigr.tigr_run(vg, a, source, **kw) for a in ("bfs", "sssp", "sswp")}
    out["cc"] = tigr.tigr_run(vgs, "cc", **kw)
    prkw = {k: v for k, v in kw.items() if k not in ("schedule", "frontier")}
    out["pr"] = tigr.tigr_run(vg, "pr", **prkw)
    return out


@pytest.mark.parametrize("K", [1, 4, 8, 32])
@pytest.mark.parametrize("layout", ["consecutive", "strided"])
@pytest.mark.parametrize("frontier", [0, 1, 3])
def test_reordered_cfg1(tigr, K, layout, frontier):
    """Runs on a reordered graph take and return original ids; values equal the oracle's on the
    original graph (incl. CC's minimum original id), through the shared-memory hot bound."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    if frontier == 3 and K % 4:
        pytest.skip("QUEUE needs 4 | K")
    for source in (0, 17):
        got = _run_all_reordered(tigr, rec.n, src, dst, w, K, layout, source=source, frontier=frontier)
        _assert_parity(got, _oracle_all(rec.n, src, dst, w, source=source))


@pytest.mark.parametrize("name", list(_edge_cases()))
def test_reordered_edge_cases(tigr, name):
    n, src, dst, w = _edge_cases()[name]
    src, dst, w = (np.asarray(x, dtype=np.uint32) for x in (src, dst, w))
    for sched in (0, 1):
        _assert_parity(_run_all_reordered(tigr, n, src, dst, w, 8, schedule=sched), _oracle_all(n, src, dst, w))


def test_reordered_cfg2_and_iterations(tigr):
    """cfg2 (n = 2^20, the hot table covers 1/64 of the nodes): BFS/CC on the reordered graph
    equal the oracle; BSP iteration counts equal the original graph's (same graph, renumbered)."""
    rec = graphgen.recipe("cfg2")
    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False)
    gs = tigr.tigr_graph_rmat(rec.n, rec.m, rec.a, rec.b, rec.c, rec.seed, rec.wseed, weighted=False,
                              symmetrize=True)
    g2, gs2 = tigr.tigr_graph_reorder(g), tigr.tigr_graph_reorder(gs)
    vg, vg2, vgs2 = tigr.tigr_virtualize(g, 8), tigr.tigr_virtualize(g2, 8), tigr.tigr_virtualize(gs2, 8)
    o = oracle.csr_build(rec.n, src, dst)
    want = oracle.bfs(o, 0)
    assert np.array_equal(tigr.tigr_run(vg2, "bfs", 0), want)
    assert np.array_equal(tigr.tigr_run(vgs2, "cc"), oracle.cc(rec.n, src, dst))
    _, st1 = tigr.tigr_run(vg, "bfs", 0, schedule=1, return_stats=True)
    lv, st2 = tigr.tigr_run(vg2, "bfs", 0, schedule=1, return_stats=True)
    assert np.array_equal(lv, want) and st1["iterations"] == st2["iterations"]


# ------------------------------------------------------------------------- round-2 paths
@pytest.mark.parametrize("frontier", [0, 1, 3])
@pytest.mark.parametrize("schedule", [0, 1])
def test_long_path_stamp_wraparound(tigr, frontier, schedule):
    """A 1300-node path (plus a hub feeding its first nodes) needs ~1300 iterations: the one-byte
    worklist stamps (values 1..255, relax.cuh stamp_of) wrap around five times, and a stale byte
    may re-activate a node 510 iterations later.  Values must still equal the oracle, and BSP
    iteration counts must equal the paper-literal push's."""
    n = 1300
    src = list(range(n - 1)) + [0] * 40
    dst = list(range(1, n)) + list(range(2, 42))
    w = [(i % 64) + 1 for i in range(n - 1)] + [64] * 40
    src, dst, w = (np.asarray(x, dtype=np.uint32) for x in (src, dst, w))
    got = _run_all(tigr, n, src, dst, w, 8, frontier=frontier, schedule=schedule)
    _assert_parity(got, _oracle_all(n, src, dst, w))
    if schedule == 1:
        o = oracle.csr_build(n, src, dst, w)
        vg = tigr.tigr_virtualize(tigr.tigr_graph_from_coo(n, src, dst, w), 8)
        _, want_it, _ = oracle.push_virtual(o, oracle.Virtual(o, 8), oracle.BFS, 0, schedule=1, worklist=1)
        _, st = tigr.tigr_run(vg, "bfs", 0, schedule=1, frontier=frontier, return_stats=True)
        assert st["iterations"] == want_it > 510


@pytest.mark.parametrize("weights", ["offset", "wide", "max"])
@pytest.mark.parametrize("K", [4, 8])
def test_packed_arcs_and_fallback(tigr, weights, K):
    """SSSP/SSWP pack target | (w - wmin) << idbits when ids and the weight range fit 32 bits
    (frontier.cu pack_arcs_prepare): weights in [100, 163] exercise the wmin offset; weights up to
    2^30 (30 bits + 11 id bits) and up to 2^32 - 2 do not fit and run from the two arrays."""
    rec = graphgen.recipe("cfg1")
    src, dst, _ = graphgen.generate(rec)
    rng = np.random.default_rng(5)
    if weights == "offset":
        w = rng.integers(100, 164, len(src), dtype=np.uint32)
    elif weights == "wide":
        w = rng.integers(1, 1 << 30, len(src), dtype=np.uint32)
    else:
        w = rng.integers(1, 0xFFFFFFFE, len(src), dtype=np.uint32)
    o = oracle.csr_build(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(tigr.tigr_graph_from_coo(rec.n, src, dst, w), K)
    for _ in range(2):  # the second run reuses the packed array
        assert np.array_equal(tigr.tigr_run(vg, "sswp", 0), oracle.sswp(o, 0))
        if weights != "max":  # 2^32-scale SSSP sums saturate (reading R14); SSWP covers that case
            assert np.array_equal(tigr.tigr_run(vg, "sssp", 0), oracle.sssp(o, 0))
    if weights != "max":  # the BSP schedule runs the unpacked kernel on the same graph
        assert np.array_equal(tigr.tigr_run(vg, "sssp", 0, schedule=1), oracle.sssp(o, 0))


@pytest.mark.parametrize("sym", [False, True])
def test_host_input_multi_chunk(tigr, sym):
    """Host arc lists are copied in 2^24-arc chunks overlapped with the arc-list scan (sort.cu):
    2^24 + 12345 arcs from host memory (two chunks, the second ragged) must build the same CSR
    as the oracle's stable counting sort, symmetrised or not, and the same as the device-input
    build."""
    n, m = 1 << 20, (1 << 24) + 12345
    rng = np.random.default_rng(9)
    src = rng.integers(0, n, m, dtype=np.uint32)
    dst = rng.integers(0, n, m, dtype=np.uint32)
    w = rng.integers(1, 65, m, dtype=np.uint32)
    g = tigr.tigr_graph_from_coo(n, src, dst, None if sym else w, symmetrize=sym)
    rp, col, ww = tigr.tigr_graph_export_csr(g)
    if sym:
        o = oracle.csr_build(n, np.concatenate([src, dst]), np.concatenate([dst, src]))
    else:
        o = oracle.csr_build(n, src, dst, w)
        assert np.array_equal(ww, o.wt)
    assert np.array_equal(rp, o.row_ptr) and np.array_equal(col, o.col)
    gd = tigr.tigr_graph_from_coo(n, torch.from_numpy(src.view(np.int32)).cuda(), torch.from_numpy(dst.view(np.int32)).cuda(),
                                  None if sym else torch.from_numpy(w.view(np.int32)).cuda(), symmetrize=sym)
    rpd, cold, _ = tigr.tigr_graph_export_csr(gd)
    assert np.array_equal(rpd, rp) and np.array_equal(cold, col)


def test_host_input_sorted_runs_skewed(tigr):
    """Host arc lists of more than one copy chunk are sorted chunk by chunk as they land and the
    sorted runs are merged into the rows (sort.cu build_sorted_runs): three chunks (the last
    ragged), unweighted, with hub sources whose rows span every chunk and nodes without arcs,
    must give the oracle's stable CSR; an id >= n in the last chunk is rejected (EINVAL)."""
    n, m = (1 << 22) + 3, 2 * (1 << 24) + 4099
    rng = np.random.default_rng(17)
    src = np.minimum((n * rng.random(m) ** 6).astype(np.uint32), n - 1)  # heavy skew toward 0
    dst = rng.integers(0, n, m, dtype=np.uint32)
    g = tigr.tigr_graph_from_coo(n, src, dst, None)
    rp, col, _ = tigr.tigr_graph_export_csr(g)
    o = oracle.csr_build(n, src, dst)
    assert np.array_equal(rp, o.row_ptr) and np.array_equal(col, o.col)
    # PageRank's in-degree sketch is collected on the same chunked path
    vg = tigr.tigr_virtualize(g, 8)
    assert float(np.abs(tigr.tigr_run(vg, "pr") - oracle.pagerank(o, 20)).max()) <= 1e-6
    bad = dst.copy()
    bad[-1] = n
    with pytest.raises(tigr.TigrError) as ei:
        tigr.tigr_graph_from_coo(n, src, bad, None)
    assert ei.value.status == tigr.TIGR_EINVAL


@pytest.mark.parametrize("n", [1, 2, 300])
def test_host_input_sorted_runs_tiny_n(tigr, n):
    """Sorted runs with one-pass keys: n = 1 (every arc a self-loop of node 0, one run per chunk
    holding a single row), n = 2 and n = 300 (one 8-bit or 9-bit-in-two-passes key), two copy
    chunks, weighted; CSR and SSSP against the oracle."""
    m = (1 << 24) + 5
    rng = np.random.default_rng(n)
    src = rng.integers(0, n, m, dtype=np.uint32)
    dst = rng.integers(0, n, m, dtype=np.uint32)
    w = rng.integers(1, 65, m, dtype=np.uint32)
    g = tigr.tigr_graph_from_coo(n, src, dst, w)
    rp, col, ww = tigr.tigr_graph_export_csr(g)
    o = oracle.csr_build(n, src, dst, w)
    assert np.array_equal(rp, o.row_ptr) and np.array_equal(col, o.col) and np.array_equal(ww, o.wt)
    assert np.array_equal(tigr.tigr_run(tigr.tigr_virtualize(g, 8), "sssp", 0), oracle.sssp(o, 0))


def test_host_input_partitioned_multi_chunk(tigr):
    """tigr_graph_from_coo_part with host arrays of two copy chunks (the multi-GPU e2e path: the
    filtered first pass, chunked copies overlapped with the arc-list scan): every rank's CSR
    equals the oracle's CSR restricted to the rank's source range."""
    n, m = 1 << 20, (1 << 24) + 777
    rng = np.random.default_rng(23)
    src = np.minimum((n * rng.random(m) ** 3).astype(np.uint32), n - 1)
    dst = rng.integers(0, n, m, dtype=np.uint32)
    w = rng.integers(1, 65, m, dtype=np.uint32)
    o = oracle.csr_build(n, src, dst, w)
    cuts = [0, n // 3, n]
    for r in range(2):
        lo, hi = cuts[r], cuts[r + 1]
        g = tigr.tigr_graph_from_coo_part(n, src, dst, w, src_lo=lo, src_hi=hi)
        rp, col, ww = tigr.tigr_graph_export_csr(g)
        a, b = o.row_ptr[lo], o.row_ptr[hi]
        want_rp = np.concatenate([np.zeros(lo, np.int64), o.row_ptr[lo:hi + 1] - a,
                                  np.full(n - hi, b - a, np.int64)])
        assert np.array_equal(rp, want_rp)
        assert np.array_equal(col, o.col[a:b]) and np.array_equal(ww, o.wt[a:b])


def test_vgraph_pr_profile(tigr):
    """tigr_vgraph_pr_profile: the push PageRank relax's arcs split into shared-memory hot slots
    and global float64 reductions.  cfg1 (n < hot slots): no global reduction at all; cfg2 (2^20
    nodes): every arc counted once, n_in = nodes with in-arcs, and the global reductions at least
    the arcs outside the true top-hot_slots in-degrees; a rank of two counts its range's arcs."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    p = tigr.tigr_vgraph_pr_profile(tigr.tigr_virtualize(tigr.tigr_graph_from_coo(rec.n, src, dst, w), 8))
    assert p["arcs"] == rec.m and p["global_reds"] == 0 and p["hot_slots"] >= rec.n
    rec = graphgen.recipe("cfg2")
    src, dst, _ = graphgen.generate(rec, weighted=False)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, None)
    vg = tigr.tigr_virtualize(g, 8)
    p = tigr.tigr_vgraph_pr_profile(vg)
    indeg = np.bincount(dst, minlength=rec.n)
    assert p["arcs"] == rec.m and p["n_in"] == int((indeg > 0).sum())
    top = int(np.sort(indeg)[::-1][:p["hot_slots"]].sum())
    assert rec.m - top <= p["global_reds"] < rec.m
    tigr.tigr_vgraph_partition(vg, 2, 0)
    vp, _ = tigr.tigr_vgraph_export(vg)
    lo, hi = vg.info()["lo"], vg.info()["hi"]
    deg = np.bincount(src, minlength=rec.n)
    mine = (vp[:-1] >= lo) & (vp[:-1] < hi) & (deg > 0)
    assert tigr.tigr_vgraph_pr_profile(vg)["arcs"] == int(deg[mine].sum())


def test_bytes_alg_byte_model(tigr):
    """tigr_stats.bytes_alg is SURVEY §8(d)'s byte model, computed in the library: PageRank per
    relax launch 20 B/arc + 4 B/virtual node + 20 B per node with arcs (apply fused in), over
    this rank's range after tigr_vgraph_partition; frontier algorithms with collect_stats from the
    device counters (0 without them)."""
    rec = graphgen.recipe("cfg1")
    src, dst, w = graphgen.generate(rec)
    deg = np.bincount(src, minlength=rec.n)
    g = tigr.tigr_graph_from_coo(rec.n, src, dst, w)
    vg = tigr.tigr_virtualize(g, 8)
    nv = vg.info()["nv"]
    _, st = tigr.tigr_run(vg, "pr", return_stats=True)
    assert st["bytes_alg"] == 20 * (rec.m * 20 + nv * 4 + int((deg > 0).sum()) * 20)
    assert abs(st["ms_kernels"] - (st["ms_total"] - st["ms_exchange"])) < 1e-9
    # one rank of two: its node range's arcs, virtual nodes and nodes with arcs
    vp, _ = tigr.tigr_vgraph_export(vg)
    rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    lo, hi = tigr.tigr_partition_ranges(rp, vp, 2)
    for r in range(2):
        tigr.tigr_vgraph_partition(vg, 2, r)
        info = vg.info()
        assert (info["lo"], info["hi"]) == (lo[r], hi[r])
        nodes = np.flatnonzero((vp[:-1] >= lo[r]) & (vp[:-1] < hi[r]) & (deg > 0))
        _, st = tigr.tigr_run(vg, "pr", return_stats=True, pr_iters=3)
        assert st["bytes_alg"] == 3 * (int(deg[nodes].sum()) * 20 + (int(hi[r]) - int(lo[r])) * 4 + len(nodes) * 20)
    tigr.tigr_vgraph_partition(vg, 1, 0)
    _, st = tigr.tigr_run(vg, "bfs", 0, return_stats=True)
    assert st["bytes_alg"] == 0
    _, st = tigr.tigr_run(vg, "bfs", 0, return_stats=True, collect_stats=1)
    assert st["bytes_alg"] == (st["edges_processed"] * 8 + st["updates"] * 4 + st["active_vnodes"] * 4
                               + st["active_nodes"] * 12 + st["iterations"] * 2 * rec.n)
